// plr_small_i32.cu -- small-n kernel instantiations: int32 data, Z/2^32 ring.
#include "plr_small_inst.cuh"

namespace plr {
cudaError_t launch_small_i32(const Tables<uint32_t, uint32_t>& tab, const LaunchArgs& la, int k, int p) {
    return small_inst::launch<uint32_t, uint32_t>(tab, la, k, p);
}
}  // namespace plr
