// plr_dispatch.cu -- dtype dispatch and tile geometry.
#include "plr_launch.h"

namespace plr {

Geometry default_geometry(plr_dtype, int, int) {
    // x = 15 elements per thread (odd: conflict-free strided smem access),
    // 8 compute warps, 4-stage TMA ring: m = 3840 elements = 15 KB per tile.
    return Geometry{15, 8, 4};
}

cudaError_t launch_scan(const PlanTables& pt, const LaunchArgs& la) {
    return pt.dtype == PLR_INT32 ? launch_scan_i32(pt, la) : launch_scan_f32(pt, la);
}

cudaError_t scan_occupancy(const PlanTables& pt, int* ctas_per_sm) {
    return pt.dtype == PLR_INT32 ? occupancy_i32(pt, ctas_per_sm) : occupancy_f32(pt, ctas_per_sm);
}

}  // namespace plr
