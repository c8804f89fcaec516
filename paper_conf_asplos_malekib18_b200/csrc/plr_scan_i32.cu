// plr_scan_i32.cu -- instantiations of the single-pass scan kernel for
// PLR_INT32 (ring Z/2^32, as uint32_t).
#include "plr_kernels.cuh"
#include "plr_launch.h"

namespace plr {
namespace {

using T = uint32_t;
constexpr int kX = 15, kW = 8, kS = 4;   // see default_geometry()

template <int K, int P, bool STORE>
cudaError_t launch_kps(const PlanTables& pt, const LaunchArgs& la) {
    auto kern = &dev::plr_scan_kernel<T, K, P, kX, kW, kS, STORE>;
    const size_t smem = dev::Smem<kX, kW, kS>::bytes;
    static bool configured = false;
    if (!configured) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        configured = true;
    }
    if (la.occupancy_out != nullptr)    // occupancy query (see occupancy_*)
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(la.occupancy_out, kern, (kW + 1) * 32, smem);
    ScanParams<T> prm;
    prm.x = static_cast<const T*>(la.x);
    prm.y = static_cast<T*>(la.y);
    prm.n = la.n;
    prm.ntiles = la.ntiles;
    prm.ticket_base = la.ticket_base;
    prm.ticket = la.ticket;
    prm.status = la.status;
    prm.epoch = la.epoch;
    prm.decay = la.decay;
    prm.x_hist = static_cast<const T*>(la.x_hist);
    prm.y_hist = static_cast<const T*>(la.y_hist);
    prm.y_tail = static_cast<T*>(la.y_tail);
    prm.lane_T = static_cast<const T*>(la.lane_T);
    prm.tab = pt.ti;
    kern<<<la.grid, (kW + 1) * 32, smem, la.stream>>>(prm);
    return cudaGetLastError();
}

template <int K, int P>
cudaError_t launch_kp(const PlanTables& pt, const LaunchArgs& la) {
    return la.store ? launch_kps<K, P, true>(pt, la) : launch_kps<K, P, false>(pt, la);
}

template <int K>
cudaError_t launch_k(const PlanTables& pt, const LaunchArgs& la) {
    switch (pt.p) {
        case 0: return launch_kp<K, 0>(pt, la);
        case 1: return launch_kp<K, 1>(pt, la);
        case 2: return launch_kp<K, 2>(pt, la);
        case 3: return launch_kp<K, 3>(pt, la);
    }
    return cudaErrorInvalidValue;
}

}  // namespace

cudaError_t launch_scan_i32(const PlanTables& pt, const LaunchArgs& la) {
    switch (pt.k) {
        case 1: return launch_k<1>(pt, la);
        case 2: return launch_k<2>(pt, la);
        case 3: return launch_k<3>(pt, la);
        case 4: return launch_k<4>(pt, la);
    }
    return cudaErrorInvalidValue;
}

cudaError_t occupancy_i32(const PlanTables& pt, int* ctas_per_sm) {
    LaunchArgs la{};
    la.store = true;
    la.occupancy_out = ctas_per_sm;     // query mode: report occupancy, do not launch
    return launch_scan_i32(pt, la);
}

}  // namespace plr
