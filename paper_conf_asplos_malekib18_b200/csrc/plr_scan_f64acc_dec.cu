// plr_scan_f64acc_dec.cu -- scan kernel instantiations: fp32 data, fp64 accumulation, DECAY.
#include "plr_scan_inst.cuh"

namespace plr {
cudaError_t launch_scan_f64acc_dec(const Tables<float, double>& tab, const LaunchArgs& la, int k, int p) {
    return inst::launch<float, double, inst::CfgDec64>(tab, la, k, p);
}
}  // namespace plr
