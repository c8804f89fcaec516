// plr_dispatch.cu -- dtype / accumulation / pipeline-config dispatch and tile geometry.
#include "plr_scan_inst.cuh"

namespace plr {

Geometry class_geometry(bool decay) {
    // x elements per thread (odd: conflict-free strided smem access) and W
    // compute warps per config; the ring depth is reported by scan_stages()
    if (decay) return Geometry{inst::CfgDec::X, inst::CfgDec::W, inst::CfgDec::S, 1};
    if (PLR_GEN_TMEM) return Geometry{PLR_TM_X, PLR_TM_W, PLR_TM_SL, PLR_TM_G};
    return Geometry{inst::CfgGen::X, inst::CfgGen::W, inst::CfgGen::S, 1};
}

int scan_stages(const PlanTables& pt) {
    if (pt.decay_flag) return inst::CfgDec::S;
    return PLR_GEN_TMEM ? PLR_TM_SL : inst::CfgGen::S;
}

cudaError_t launch_scan(const PlanTables& pt, const LaunchArgs& la) {
    if (pt.dtype == PLR_INT32) return launch_scan_i32(pt.ti, la, pt.k, pt.p);
    if (pt.acc64) return pt.decay_flag ? launch_scan_f64acc_dec(pt.td, la, pt.k, pt.p)
                                       : launch_scan_f64acc_gen(pt.td, la, pt.k, pt.p);
    if (!pt.decay_flag) return cudaErrorInvalidValue;    // planner forces fp64 accumulation
    return launch_scan_f32(pt.tf, la, pt.k, pt.p);
}

cudaError_t scan_occupancy(const PlanTables& pt, int* ctas_per_sm) {
    LaunchArgs la{};
    la.store = true;
    la.occupancy_out = ctas_per_sm;
    return launch_scan(pt, la);
}

}  // namespace plr
