// plr_reduce_inst.cuh -- host-side launch of the reduce-only kernel for one
// (data, accumulation) type; included by plr_reduce_{i32,f64acc}.cu.
#pragma once
#include "plr_kernels_reduce.cuh"
#include "plr_launch.h"
#include <atomic>

namespace plr {
namespace reduce_inst {

template <typename T, typename A, int K, int P>
cudaError_t launch_kp(const Tables<T, A>& tab, const LaunchArgs& la) {
    using L = dev::LayoutRd<T, A, K, kRedX, kRedW, kRedS>;
    void (*kern)(const ScanParams<T, A>) = &dev::plr_reduce_kernel<T, A, K, P, kRedX, kRedW, kRedS>;
    constexpr int threads = (kRedW + 1) * 32;
    static std::atomic<unsigned long long> configured{0};        // per-device smem opt-in
    int dev = 0;
    if (cudaError_t e = cudaGetDevice(&dev); e != cudaSuccess) return e;
    const unsigned long long bit = 1ull << (dev & 63);
    if (!(configured.load(std::memory_order_acquire) & bit)) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)L::bytes);
        if (e != cudaSuccess) return e;
        configured.fetch_or(bit, std::memory_order_acq_rel);
    }
    if (la.occupancy_out != nullptr)
        return cudaOccupancyMaxActiveBlocksPerMultiprocessor(la.occupancy_out, kern, threads, L::bytes);
    const ScanParams<T, A> prm = make_params(tab, la);
    kern<<<la.grid, threads, L::bytes, la.stream>>>(prm);
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

}  // namespace reduce_inst
}  // namespace plr
