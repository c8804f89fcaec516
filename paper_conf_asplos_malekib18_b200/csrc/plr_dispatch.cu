// plr_dispatch.cu -- dtype / accumulation dispatch and tile geometry.
#include "plr_launch.h"

namespace plr {

#ifndef PLR_STAGES
#define PLR_STAGES 5
#endif

Geometry default_geometry(plr_dtype, int, int) {
    // x = 15 elements per thread (odd: conflict-free strided smem access),
    // 8 compute warps, PLR_STAGES-stage TMA ring: m = 3840 elements = 15 KB per tile.
    return Geometry{15, 8, PLR_STAGES};
}

cudaError_t launch_scan(const PlanTables& pt, const LaunchArgs& la) {
    if (pt.dtype == PLR_INT32) return launch_scan_i32(pt.ti, la, pt.k, pt.p);
    if (pt.acc64) return launch_scan_f64acc(pt.td, la, pt.k, pt.p);
    return launch_scan_f32(pt.tf, la, pt.k, pt.p);
}

cudaError_t scan_occupancy(const PlanTables& pt, int* ctas_per_sm) {
    LaunchArgs la{};
    la.store = true;
    la.occupancy_out = ctas_per_sm;
    return launch_scan(pt, la);
}

}  // namespace plr
