// plr_reduce_i32.cu -- reduce-only kernel instantiations: int32 data, Z/2^32 ring.
#include "plr_reduce_inst.cuh"

namespace plr {
cudaError_t launch_reduce_i32(const Tables<uint32_t, uint32_t>& tab, const LaunchArgs& la, int k, int p) {
    return reduce_inst::launch<uint32_t, uint32_t>(tab, la, k, p);
}
}  // namespace plr
