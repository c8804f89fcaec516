// plr_launch.h -- host-side launch interface between the ABI and the
// templated scan kernels (instantiated per dtype in plr_scan_{i32,f32}.cu).
#pragma once
#include <cuda_runtime.h>

#include "plr_internal.h"

namespace plr {

struct LaunchArgs {
    const void* x;
    void* y;
    uint64_t n;
    uint64_t ntiles;
    unsigned long long* ticket;
    unsigned long long* status;
    uint32_t status_mask;
    int decay;
    uint32_t dec_mask = 0x3f;
    const void* x_hist;
    const void* y_hist;
    void* y_tail;
    const void* lane_T;
    unsigned long long* stats = nullptr;
    int grid;
    int sig = 0;                        // compile-time signature id (plr_constsig.cuh), 0 = runtime tables
    bool store;
    bool unit1 = false;                 // look-back units of one tile (small n): the *_u1 kernels
    bool reverse = false;               // the anticausal recurrence (REV kernels: small-n, DECAY)
    bool cluster = false;               // small-n kernel: clusters of kSmallC tiles (cluster look-back)
    int lag = 0;                        // re-read kernel: phase-B lag in tiles (0: NS-1)
    cudaStream_t stream;
    int* occupancy_out = nullptr;       // non-null: only report CTAs/SM of the kernel
};

// ScanParams of one launch from the plan's tables and the launch arguments
template <typename T, typename A>
inline ScanParams<T, A> make_params(const Tables<T, A>& tab, const LaunchArgs& la) {
    ScanParams<T, A> prm;
    prm.x = static_cast<const T*>(la.x);
    prm.y = static_cast<T*>(la.y);
    prm.n = la.n;
    prm.ntiles = la.ntiles;
    prm.ticket = la.ticket;
    prm.status = la.status;
    prm.status_mask = la.status_mask;
    prm.decay = la.decay;
    prm.dec_mask = la.dec_mask;
    prm.x_hist = static_cast<const T*>(la.x_hist);
    prm.y_hist = static_cast<const T*>(la.y_hist);
    prm.y_tail = static_cast<T*>(la.y_tail);
    prm.lane_T = static_cast<const A*>(la.lane_T);
    prm.stats = la.stats;
    prm.lag = la.lag;
    prm.tab = tab;
    return prm;
}

// Tile geometry of the DECAY / generic kernel configs.
// (fp64-accumulation DECAY plans have their own config)
Geometry class_geometry(bool decay, int k, bool acc64 = false);

cudaError_t launch_scan(const PlanTables& pt, const LaunchArgs& la);
// the small-n kernel (plr_kernels_small.cuh): one CTA per tile of the plan's
// geo_s, grid = ntiles (la.grid ignored); la.y == nullptr: reduce-only
cudaError_t launch_small(const PlanTables& pt, const LaunchArgs& la);
cudaError_t small_occupancy(const PlanTables& pt, int* ctas_per_sm);
cudaError_t small_cluster_occupancy(const PlanTables& pt, int* clusters);   // co-resident clusters of kSmallC
// the reduce-only kernel (plr_kernels_reduce.cuh): la.status = per-CTA record
// scratch (kStatusMaxBytes each), la.grid CTAs over contiguous tile ranges of
// kRedX * kRedW * 32 elements, la.y_tail = the K end-state outputs
cudaError_t launch_reduce(const PlanTables& pt, const LaunchArgs& la);
// the Scan comparator (plr_blelloch.cuh); tmp == nullptr: size query
cudaError_t blelloch_i32(const uint32_t* x, uint32_t* y, long long n, const uint32_t* c, int k, const uint32_t* alpha,
                         int p, void* tmp, size_t& tmp_bytes, cudaStream_t s);
cudaError_t blelloch_f32(const float* x, float* y, long long n, const float* c, int k, const float* alpha, int p,
                         void* tmp, size_t& tmp_bytes, cudaStream_t s);
cudaError_t reduce_occupancy(const PlanTables& pt, int* ctas_per_sm);
cudaError_t launch_reduce_i32(const Tables<uint32_t, uint32_t>& tab, const LaunchArgs& la, int k, int p);
cudaError_t launch_reduce_f64acc(const Tables<float, double>& tab, const LaunchArgs& la, int k, int p);
cudaError_t launch_small_i32(const Tables<uint32_t, uint32_t>& tab, const LaunchArgs& la, int k, int p);
cudaError_t launch_small_f32(const Tables<float, float>& tab, const LaunchArgs& la, int k, int p);
cudaError_t launch_small_f64acc(const Tables<float, double>& tab, const LaunchArgs& la, int k, int p);
cudaError_t scan_occupancy(const PlanTables& pt, int* ctas_per_sm);

// per-(data, accumulation) type entry points (plr_scan_*.cu)
cudaError_t launch_scan_i32(const Tables<uint32_t, uint32_t>& tab, const LaunchArgs& la, int k, int p);
cudaError_t launch_scan_f32(const Tables<float, float>& tab, const LaunchArgs& la, int k, int p);
cudaError_t launch_scan_f64acc_dec(const Tables<float, double>& tab, const LaunchArgs& la, int k, int p);
cudaError_t launch_scan_f64acc_gen(const Tables<float, double>& tab, const LaunchArgs& la, int k, int p);
cudaError_t launch_scan_i32_u1(const Tables<uint32_t, uint32_t>& tab, const LaunchArgs& la, int k, int p);
cudaError_t launch_scan_f64acc_gen_u1(const Tables<float, double>& tab, const LaunchArgs& la, int k, int p);
// ring depth of the config a plan launches with (plan info)
int scan_stages(const PlanTables& pt);
// plr_plan_info.kernel_kind of a plan
int kernel_kind(const PlanTables& pt);

}  // namespace plr
