// plr_reduce_f64acc.cu -- reduce-only kernel instantiations: fp32 data, fp64 accumulation (FLOAT class).
#include "plr_reduce_inst.cuh"

namespace plr {
cudaError_t launch_reduce_f64acc(const Tables<float, double>& tab, const LaunchArgs& la, int k, int p) {
    return reduce_inst::launch<float, double>(tab, la, k, p);
}
}  // namespace plr
