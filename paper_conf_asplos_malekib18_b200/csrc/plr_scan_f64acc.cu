// plr_scan_f64acc.cu -- scan kernel instantiations: fp32 data, fp64 accumulation (ill-conditioned float signatures).
#include "plr_scan_inst.cuh"

namespace plr {
cudaError_t launch_scan_f64acc(const Tables<float, double>& tab, const LaunchArgs& la, int k, int p) {
    return inst::launch<float, double>(tab, la, k, p);
}
}  // namespace plr
