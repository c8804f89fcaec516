// plr_small_f32.cu -- small-n kernel instantiations: fp32 data, fp32 accumulation.
#include "plr_small_inst.cuh"

namespace plr {
cudaError_t launch_small_f32(const Tables<float, float>& tab, const LaunchArgs& la, int k, int p) {
    return small_inst::launch<float, float>(tab, la, k, p);
}
}  // namespace plr
