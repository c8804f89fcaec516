// plr_scan_inst.cuh -- host-side launch of the scan kernel for one
// (data type T, accumulation type A); included by the per-type .cu files so
// the instantiations compile in parallel.
#pragma once
#include "plr_kernels.cuh"
#include "plr_launch.h"

namespace plr {
namespace inst {

#ifndef PLR_STAGES
#define PLR_STAGES 5
#endif
#ifndef PLR_LAG
#define PLR_LAG 2
#endif
#ifndef PLR_NL
#define PLR_NL 2
#endif
constexpr int kX = 15, kW = 8, kS = PLR_STAGES, kD = PLR_LAG, kNL = PLR_NL;   // see default_geometry()

template <typename T, typename A, int K, int P, bool STORE>
cudaError_t launch_kps(const Tables<T, A>& tab, const LaunchArgs& la) {
    auto kern = &dev::plr_scan_kernel<T, A, K, P, kX, kW, kS, kD, kNL, STORE>;
    const size_t smem = dev::Layout<T, A, K, kX, kW, kS, kD>::bytes;
    static bool configured = false;
    if (!configured) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        configured = true;
    }
    if (la.occupancy_out != nullptr)    // occupancy query: report CTAs/SM, do not launch
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(la.occupancy_out, kern, (kW + 1 + kNL) * 32, smem);
    ScanParams<T, A> prm;
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
    prm.lane_T = static_cast<const A*>(la.lane_T);
    prm.stats = la.stats;
    prm.tab = tab;
    kern<<<la.grid, (kW + 1 + kNL) * 32, smem, la.stream>>>(prm);
    return cudaGetLastError();
}

template <typename T, typename A, int K>
cudaError_t launch_k(const Tables<T, A>& tab, const LaunchArgs& la, int p) {
    switch (p) {
        case 0: return la.store ? launch_kps<T, A, K, 0, true>(tab, la) : launch_kps<T, A, K, 0, false>(tab, la);
        case 1: return la.store ? launch_kps<T, A, K, 1, true>(tab, la) : launch_kps<T, A, K, 1, false>(tab, la);
        case 2: return la.store ? launch_kps<T, A, K, 2, true>(tab, la) : launch_kps<T, A, K, 2, false>(tab, la);
        case 3: return la.store ? launch_kps<T, A, K, 3, true>(tab, la) : launch_kps<T, A, K, 3, false>(tab, la);
    }
    return cudaErrorInvalidValue;
}

template <typename T, typename A>
cudaError_t launch(const Tables<T, A>& tab, const LaunchArgs& la, int k, int p) {
    switch (k) {
        case 1: return launch_k<T, A, 1>(tab, la, p);
        case 2: return launch_k<T, A, 2>(tab, la, p);
        case 3: return launch_k<T, A, 3>(tab, la, p);
        case 4: return launch_k<T, A, 4>(tab, la, p);
    }
    return cudaErrorInvalidValue;
}

}  // namespace inst
}  // namespace plr
