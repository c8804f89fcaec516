// plr_small_inst.cuh -- host-side launch of the small-n kernel for one (data,
// accumulation) type; included by plr_small_{i32,f32,f64acc}.cu.
#pragma once
#include "plr_kernels_small.cuh"
#include "plr_launch.h"

namespace plr {
namespace small_inst {

template <typename T, typename A, int K, int P>
cudaError_t launch_kp(const Tables<T, A>& tab, const LaunchArgs& la) {
    using L = dev::LayoutS<T, A, K, kSmallX, kSmallW>;
    void (*kern)(const ScanParams<T, A>) = la.reverse ? &dev::plr_small_kernel<T, A, K, P, kSmallX, kSmallW, true>
                                                      : &dev::plr_small_kernel<T, A, K, P, kSmallX, kSmallW, false>;
    static_assert(L::bytes <= 48 * 1024, "small-n kernel needs no dynamic shared memory opt-in");
    if (la.cluster) {                       // clusters of kSmallC tiles (forward, resident)
        void (*kc)(const ScanParams<T, A>) = &dev::plr_small_kernel<T, A, K, P, kSmallX, kSmallW, false, kSmallC>;
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3((unsigned)((la.ntiles + kSmallC - 1) / kSmallC * kSmallC), 1, 1);
        cfg.blockDim = dim3(kSmallW * 32, 1, 1);
        cfg.dynamicSmemBytes = L::bytes;
        cfg.stream = la.stream;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = kSmallC;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        if (la.occupancy_out != nullptr) return cudaOccupancyMaxActiveClusters(la.occupancy_out, kc, &cfg);
        const ScanParams<T, A> prm = make_params(tab, la);
        return cudaLaunchKernelEx(&cfg, kc, prm);
    }
    if (la.occupancy_out != nullptr)
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(la.occupancy_out, kern, kSmallW * 32, L::bytes);
    const ScanParams<T, A> prm = make_params(tab, la);
    kern<<<(unsigned)la.ntiles, kSmallW * 32, L::bytes, la.stream>>>(prm);
    return cudaGetLastError();
}

template <typename T, typename A, int K>
cudaError_t launch_k(const Tables<T, A>& tab, const LaunchArgs& la, int p) {
    switch (p) {
        case 0: return launch_kp<T, A, K, 0>(tab, la);
        case 1: return launch_kp<T, A, K, 1>(tab, la);
        case 2: return launch_kp<T, A, K, 2>(tab, la);
        case 3: return launch_kp<T, A, K, 3>(tab, la);
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

}  // namespace small_inst
}  // namespace plr
