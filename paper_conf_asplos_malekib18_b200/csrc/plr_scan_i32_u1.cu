// plr_scan_i32_u1.cu -- scan kernel instantiations with look-back units of one tile
// (small-n launches, plr_api.cu); otherwise as plr_scan_i32.cu.
#include "plr_scan_inst.cuh"

namespace plr {
cudaError_t launch_scan_i32_u1(const Tables<uint32_t, uint32_t>& tab, const LaunchArgs& la, int k, int p) {
    return inst::launch<uint32_t, uint32_t, inst::CfgGen1>(tab, la, k, p);
}
}  // namespace plr
