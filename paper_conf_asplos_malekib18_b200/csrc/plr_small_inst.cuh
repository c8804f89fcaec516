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
