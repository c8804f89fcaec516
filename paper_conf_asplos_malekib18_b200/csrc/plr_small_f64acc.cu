// plr_small_f64acc.cu -- small-n kernel instantiations: fp32 data, fp64 accumulation.
#include "plr_small_inst.cuh"

namespace plr {
cudaError_t launch_small_f64acc(const Tables<float, double>& tab, const LaunchArgs& la, int k, int p) {
    return small_inst::launch<float, double>(tab, la, k, p);
}
}  // namespace plr
