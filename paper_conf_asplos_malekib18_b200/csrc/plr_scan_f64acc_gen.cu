// plr_scan_f64acc_gen.cu -- scan kernel instantiations: fp32 data, fp64 accumulation, non-decaying.
#include "plr_scan_inst.cuh"

namespace plr {
cudaError_t launch_scan_f64acc_gen(const Tables<float, double>& tab, const LaunchArgs& la, int k, int p) {
    return inst::launch<float, double, inst::CfgGen>(tab, la, k, p);
}
}  // namespace plr
