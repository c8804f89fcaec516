// plr_dispatch.cu -- dtype / accumulation / pipeline-config dispatch and tile geometry.
#include "plr_scan_inst.cuh"

namespace plr {

Geometry class_geometry(bool decay, int k, bool acc64) {
    // x elements per thread (odd: conflict-free strided smem access) and W
    // compute warps per config; the ring depth is reported by scan_stages()
    if (decay && acc64) return Geometry{inst::CfgDec64::X, inst::CfgDec64::W, inst::CfgDec64::S, 1};
    if (decay) return Geometry{inst::CfgDec::X, inst::CfgDec::W, inst::CfgDec::S, 1};
    switch (inst::gen_kind(k)) {
        case 2: return Geometry{PLR_RR_X, PLR_RR_W, PLR_RR_SA + PLR_RR_SB, PLR_RR_G};
        case 1: return Geometry{PLR_TM_X, PLR_TM_W, PLR_TM_SL + PLR_TM_ST, PLR_TM_G};
    }
    return Geometry{inst::CfgGen::X, inst::CfgGen::W, inst::CfgGen::S, 1};
}

int scan_stages(const PlanTables& pt) { return pt.geo.S; }

int kernel_kind(const PlanTables& pt) {
    if (pt.decay_flag) return (pt.acc64 ? inst::CfgDec64::DT : inst::CfgDec::DT) ? 4 : 0;
    const int kind = inst::gen_kind(pt.k);
    return kind == 0 ? 3 : kind;
}

cudaError_t launch_scan(const PlanTables& pt, const LaunchArgs& la) {
    if (pt.dtype == PLR_INT32)
        return la.unit1 ? launch_scan_i32_u1(pt.ti1, la, pt.k, pt.p) : launch_scan_i32(pt.ti, la, pt.k, pt.p);
    if (pt.acc64) {
        if (pt.decay_flag) return launch_scan_f64acc_dec(pt.td, la, pt.k, pt.p);
        return la.unit1 ? launch_scan_f64acc_gen_u1(pt.td1, la, pt.k, pt.p) : launch_scan_f64acc_gen(pt.td, la, pt.k, pt.p);
    }
    if (!pt.decay_flag) return cudaErrorInvalidValue;    // planner forces fp64 accumulation
    return launch_scan_f32(pt.tf, la, pt.k, pt.p);
}

cudaError_t launch_small(const PlanTables& pt, const LaunchArgs& la) {
    if (pt.dtype == PLR_INT32) return launch_small_i32(pt.tis, la, pt.k, pt.p);
    if (pt.acc64) return launch_small_f64acc(pt.tds, la, pt.k, pt.p);
    return launch_small_f32(pt.tfs, la, pt.k, pt.p);
}

cudaError_t launch_reduce(const PlanTables& pt, const LaunchArgs& la) {
    if (pt.dtype == PLR_INT32) return launch_reduce_i32(pt.tr, la, pt.k, pt.p);
    if (pt.acc64) return launch_reduce_f64acc(pt.trd, la, pt.k, pt.p);
    return cudaErrorInvalidValue;                       // fp32-accumulation plans are DECAY: no reduce pass
}

cudaError_t reduce_occupancy(const PlanTables& pt, int* ctas_per_sm) {
    LaunchArgs la{};
    la.occupancy_out = ctas_per_sm;
    return launch_reduce(pt, la);
}

cudaError_t small_occupancy(const PlanTables& pt, int* ctas_per_sm) {
    LaunchArgs la{};
    la.occupancy_out = ctas_per_sm;
    return launch_small(pt, la);
}

cudaError_t small_cluster_occupancy(const PlanTables& pt, int* clusters) {
    LaunchArgs la{};
    la.occupancy_out = clusters;
    la.cluster = true;
    la.ntiles = 1;
    return launch_small(pt, la);
}

cudaError_t scan_occupancy(const PlanTables& pt, int* ctas_per_sm) {
    LaunchArgs la{};
    la.store = true;
    la.occupancy_out = ctas_per_sm;
    return launch_scan(pt, la);
}

}  // namespace plr
