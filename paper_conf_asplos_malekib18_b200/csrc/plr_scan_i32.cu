// plr_scan_i32.cu -- scan kernel instantiations: int32 data, Z/2^32 ring (never DECAY).
#include "plr_scan_inst.cuh"

namespace plr {
cudaError_t launch_scan_i32(const Tables<uint32_t, uint32_t>& tab, const LaunchArgs& la, int k, int p) {
    return inst::launch<uint32_t, uint32_t, inst::CfgGen>(tab, la, k, p);
}
}  // namespace plr
