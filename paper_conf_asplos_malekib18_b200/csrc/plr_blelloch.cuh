// plr_blelloch.cuh -- the "Scan" comparator of the paper (SURVEY.md §8(f)
// row 3): Blelloch's formulation of a linear recurrence as a prefix scan
// whose elements are (k x k matrix, k-vector) pairs with the associative
// operator (A2, u2) o (A1, u1) = (A2 A1, A2 u1 + u2) (P:230-234,
// P:381-390), evaluated with CUB's DeviceScan (decoupled
// look-back, the library path the paper benchmarks against, P:853,
// P:967-970).  It is a comparison baseline for bench/ablation tooling, NOT
// the PLR path: every element carries k^2 + k words through the scan and
// every combine costs k^3 + k^2 multiply-adds (the work the paper charges
// Scan with), where PLR's hierarchy carries k words per chunk.
// Element i is (M, e0 t_i) with M the companion matrix of (1: c) and t_i the
// map output (Eq. 2, computed on the fly from x); the scan's inclusive
// prefix is (M^{i+1}, S_i), S_i = (y_i, ..., y_{i-k+1}).  Inputs and outputs
// stream through transform iterators (O(n) memory; the paper's Scan
// materialised the O(n k^2) pairs).
#pragma once
#include <cub/device/device_scan.cuh>
#include <thrust/iterator/counting_iterator.h>
#include <thrust/iterator/transform_iterator.h>
#include <thrust/iterator/transform_output_iterator.h>

#include "plr_internal.h"

namespace plr {
namespace blelloch {

template <typename A, int K>
struct Affine {
    A M[K * K];
    A v[K];
};

template <typename A>
__device__ __forceinline__ A fma_(A a, A b, A c) { return a * b + c; }
template <>
__device__ __forceinline__ float fma_<float>(float a, float b, float c) { return __fmaf_rn(a, b, c); }

// (A2, u2) o (A1, u1): first 1, then 2
template <typename A, int K>
struct Combine {
    __device__ __forceinline__ Affine<A, K> operator()(const Affine<A, K>& a, const Affine<A, K>& b) const {
        Affine<A, K> c;
#pragma unroll
        for (int q = 0; q < K; q++) {
#pragma unroll
            for (int r = 0; r < K; r++) {
                A s = A(0);
#pragma unroll
                for (int t = 0; t < K; t++) s = fma_(b.M[q * K + t], a.M[t * K + r], s);
                c.M[q * K + r] = s;
            }
            A s = b.v[q];
#pragma unroll
            for (int t = 0; t < K; t++) s = fma_(b.M[q * K + t], a.v[t], s);
            c.v[q] = s;
        }
        return c;
    }
};

template <typename A, int K>
struct Element {
    const A* x;
    A c[K];
    A alpha[kMaxP + 1];
    int p;
    __device__ Affine<A, K> operator()(long long i) const {
        Affine<A, K> e;
#pragma unroll
        for (int q = 0; q < K * K; q++) e.M[q] = A(0);
#pragma unroll
        for (int r = 0; r < K; r++) e.M[r] = c[r];
#pragma unroll
        for (int q = 1; q < K; q++) e.M[q * K + q - 1] = A(1);
        A t = alpha[0] * x[i];
        for (int j = 1; j <= p; j++)
            if (i - j >= 0) t = fma_(alpha[j], x[i - j], t);
        e.v[0] = t;
#pragma unroll
        for (int q = 1; q < K; q++) e.v[q] = A(0);
        return e;
    }
};

template <typename A, int K>
struct First {
    __device__ __forceinline__ A operator()(const Affine<A, K>& e) const { return e.v[0]; }
};

template <typename A, int K>
cudaError_t scan(const A* x, A* y, long long n, const A* c, const A* alpha, int p, void* tmp, size_t& tmp_bytes,
                 cudaStream_t stream) {
    Element<A, K> g;
    g.x = x;
    g.p = p;
    for (int r = 0; r < K; r++) g.c[r] = c[r];
    for (int j = 0; j <= kMaxP; j++) g.alpha[j] = j <= p ? alpha[j] : A(0);
    auto in = thrust::make_transform_iterator(thrust::counting_iterator<long long>(0), g);
    auto out = thrust::make_transform_output_iterator(y, First<A, K>());
    return cub::DeviceScan::InclusiveScan(tmp, tmp_bytes, in, out, Combine<A, K>(), n, stream);
}

}  // namespace blelloch
}  // namespace plr
