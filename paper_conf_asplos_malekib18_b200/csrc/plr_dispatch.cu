// plr_dispatch.cu -- dtype / accumulation / pipeline-config dispatch and tile geometry.
#include "plr_scan_inst.cuh"

namespace plr {

Geometry default_geometry(plr_dtype, int, int) {
    // x = 15 elements per thread (odd: conflict-free strided smem access),
    // 8 compute warps: m = 3840 elements = 15 KB per tile.  The ring depth
    // depends on the class (scan_stages()).
    return Geometry{inst::kX, inst::kW, 0};
}

int scan_stages(const PlanTables& pt) {
    return pt.decay_flag ? inst::CfgDec::S : inst::CfgGen::S;
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
