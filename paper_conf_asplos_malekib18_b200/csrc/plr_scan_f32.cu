// plr_scan_f32.cu -- scan kernel instantiations: fp32 data, fp32 accumulation (DECAY plans; non-decaying float plans accumulate in fp64).
#include "plr_scan_inst.cuh"

namespace plr {
cudaError_t launch_scan_f32(const Tables<float, float>& tab, const LaunchArgs& la, int k, int p) {
    return inst::launch<float, float, inst::CfgDec>(tab, la, k, p);
}
}  // namespace plr
