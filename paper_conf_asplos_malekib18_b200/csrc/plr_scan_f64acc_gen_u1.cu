// plr_scan_f64acc_gen_u1.cu -- scan kernel instantiations with look-back units of one tile
// (small-n launches, plr_api.cu); otherwise as plr_scan_f64acc_gen.cu.
#include "plr_scan_inst.cuh"

namespace plr {
cudaError_t launch_scan_f64acc_gen_u1(const Tables<float, double>& tab, const LaunchArgs& la, int k, int p) {
    return inst::launch<float, double, inst::CfgGen1>(tab, la, k, p);
}
}  // namespace plr
