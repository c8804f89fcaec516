// plr_kernels.cuh -- sm_100a kernels of the PLR hot path.
//
// One persistent single-pass kernel evaluates Eq. (1):
//   a1 load + fused FIR map (Eq. (2))
//   a2 per-thread sequential chunk of X elements with zero state
//      (the serial loop of P:206-214; work-efficient replacement of the
//      element-level doubling of Phase 1)
//   a3 warp carry propagation: Kogge-Stone over the 32 lanes with
//      T(X*2^s), shuffles
//   a4 block propagation of warp aggregates through shared memory
//   a5 grid: decoupled look-back of the k carries with epoch-tagged status
//      words (Phase 2; carry precomputation P:527-556;
//      chunk ticket P:651-653; publish/wait P:668-683)
//   a6 carry-in distribution + correction y_u = l_u + sum_r S_r h^(r)_u
//
//   a7 store
// Data movement: one producer warp issues TMA bulk copies
// (cp.async.bulk, mbarrier complete_tx) of whole tiles into an S-stage
// shared-memory ring and TMA bulk stores of the finished tiles; compute warps
// only touch shared memory (odd X => conflict-free strided access).
#pragma once
#include <cuda_runtime.h>
#include <cstdint>

#include "plr_internal.h"

namespace plr {
namespace dev {

// ---------------------------------------------------------------- PTX ------
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint64_t* bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.release.cta.shared::cta.b64 _, [%0], %1;"
                 ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
    return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    while (!mbar_try_wait(bar, parity)) { }
}
// TMA 1D bulk copy global -> shared, completion on an mbarrier (UBLKCP).
__device__ __forceinline__ void bulk_load(void* sdst, const void* gsrc, uint32_t bytes, uint64_t* bar,
                                          uint64_t policy) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
        ::"r"(smem_u32(sdst)), "l"(gsrc), "r"(bytes), "r"(smem_u32(bar)), "l"(policy) : "memory");
}
// TMA 1D bulk copy shared -> global, bulk-group completion.
__device__ __forceinline__ void bulk_store(void* gdst, const void* ssrc, uint32_t bytes, uint64_t policy) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;"
                 ::"l"(gdst), "r"(smem_u32(ssrc)), "r"(bytes), "l"(policy) : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group %0;" ::"n"(N) : "memory"); }
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ void named_sync(int id, int nthreads) {
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}
__device__ __forceinline__ void st_relaxed(unsigned long long* p, unsigned long long v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ unsigned long long ld_relaxed(const unsigned long long* p) {
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

// ------------------------------------------------------------- ring ops ----
__device__ __forceinline__ uint32_t mad(uint32_t a, uint32_t b, uint32_t c) { return a * b + c; }
__device__ __forceinline__ float mad(float a, float b, float c) { return __fmaf_rn(a, b, c); }
__device__ __forceinline__ uint32_t bits(uint32_t v) { return v; }
__device__ __forceinline__ uint32_t bits(float v) { return __float_as_uint(v); }
template <typename T> __device__ __forceinline__ T from_bits(uint32_t b);
template <> __device__ __forceinline__ uint32_t from_bits<uint32_t>(uint32_t b) { return b; }
template <> __device__ __forceinline__ float from_bits<float>(uint32_t b) { return __uint_as_float(b); }

// v[q] += sum_r Tm[q][r] * o[r]
template <typename T, int K>
__device__ __forceinline__ void matvec_acc(T (&v)[K], const T* Tm, const T (&o)[K]) {
    T r_[K];
#pragma unroll
    for (int q = 0; q < K; q++) {
        T acc = v[q];
#pragma unroll
        for (int r = 0; r < K; r++) acc = mad(Tm[q * kMaxK + r], o[r], acc);
        r_[q] = acc;
    }
#pragma unroll
    for (int q = 0; q < K; q++) v[q] = r_[q];
}

// ------------------------------------------------------ the scan kernel ----
template <int X, int W, int S>
struct Smem {
    static constexpr int M = 32 * W * X;
    static constexpr int SW = M + kHalo;                       // words per stage
    static constexpr size_t stage_bytes = (size_t)S * SW * 4;
    static constexpr size_t bytes = stage_bytes + 2 * S * 8 /*bars*/ + S * 8 /*tile ids*/ +
                                    (W * kMaxK + kMaxK) * 4 + 16;
};

template <typename T, int K, int P, int X, int W, int S, bool STORE>
__global__ void __launch_bounds__((W + 1) * 32)
plr_scan_kernel(const __grid_constant__ ScanParams<T> prm) {
    using SM = Smem<X, W, S>;
    constexpr int M = SM::M;
    constexpr int SW = SM::SW;
    constexpr int NC = W * 32;
    constexpr int LOGW = (W >= 16) ? 4 : (W >= 8) ? 3 : (W >= 4) ? 2 : (W >= 2) ? 1 : 0;
    static_assert((1 << LOGW) == W, "W must be a power of two");
    static_assert(X >= K && X <= kMaxX && (X & 1), "X must be odd and >= K");
    static_assert(P <= kHalo, "halo");

    extern __shared__ __align__(128) unsigned char smem_raw[];
    T* stages = reinterpret_cast<T*>(smem_raw);
    uint64_t* full_bar = reinterpret_cast<uint64_t*>(smem_raw + SM::stage_bytes);
    uint64_t* done_bar = full_bar + S;
    long long* tile_of = reinterpret_cast<long long*>(done_bar + S);
    T* wagg = reinterpret_cast<T*>(tile_of + S);               // [W][K]
    T* bcast = wagg + W * kMaxK;                               // [K]

    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    const long long ntiles = (long long)prm.ntiles;
    const unsigned long long n = prm.n;
    const bool last_ragged = (n % (unsigned long long)M) != 0;

    if (tid == 0) {
        for (int s = 0; s < S; s++) { mbar_init(&full_bar[s], 1); mbar_init(&done_bar[s], NC); }
        fence_mbar_init();
    }
    __syncthreads();

    // ===================================================== producer warp ===
    if (warp == W) {
        if (lane != 0) return;
        const uint64_t pol = policy_evict_first();
        bool done = false;
        auto fill = [&](int s) {
            const long long j = (long long)(atomicAdd(prm.ticket, 1ull) - prm.ticket_base);
            tile_of[s] = j;
            if (j >= ntiles) { done = true; mbar_arrive(&full_bar[s]); return; }
            if (j == ntiles - 1 && last_ragged) { mbar_arrive(&full_bar[s]); return; }   // consumers load it
            T* st = stages + (size_t)s * SW;
            if (j == 0) {
#pragma unroll
                for (int q = 0; q < kHalo; q++)
                    st[q] = (q >= kHalo - P && prm.x_hist != nullptr) ? prm.x_hist[q - (kHalo - P)] : T(0);
                mbar_arrive_tx(&full_bar[s], M * sizeof(T));
                bulk_load(st + kHalo, prm.x, M * sizeof(T), &full_bar[s], pol);
            } else {
                mbar_arrive_tx(&full_bar[s], SW * sizeof(T));
                bulk_load(st, prm.x + (size_t)j * M - kHalo, SW * sizeof(T), &full_bar[s], pol);
            }
        };
        for (int s = 0; s < S && !done; s++) fill(s);
        for (int it = 0;; it++) {
            const int s = it % S;
            const long long j = tile_of[s];
            if (j >= ntiles) break;
            mbar_wait(&done_bar[s], (uint32_t)((it / S) & 1));
            bool stored = false;
            if (STORE && !(j == ntiles - 1 && last_ragged)) {
                bulk_store(prm.y + (size_t)j * M, stages + (size_t)s * SW + kHalo, M * sizeof(T), pol);
                bulk_commit();
                stored = true;
            }
            if (it >= 1 && !done) {
                if (stored) bulk_wait_read<1>(); else bulk_wait_read<0>();
                fill((it - 1) % S);
            }
        }
        bulk_wait_all<0>();
        return;
    }

    // ===================================================== compute warps ===
    const Tables<T>& tb = prm.tab;
    T Tl[K * K];                                                // T(X*lane)
#pragma unroll
    for (int e = 0; e < K * K; e++) Tl[e] = prm.lane_T[e * 32 + lane];
    const uint32_t tagA = 2u * prm.epoch, tagI = 2u * prm.epoch + 1u;

    for (int it = 0;; it++) {
        const int s = it % S;
        mbar_wait(&full_bar[s], (uint32_t)((it / S) & 1));
        const long long j = tile_of[s];
        if (j >= ntiles) break;
        const bool ragged = (j == ntiles - 1) && last_ragged;
        T* st = stages + (size_t)s * SW;
        const long long g0 = j * (long long)M + (long long)tid * X;   // global index of my first element

        // ---- a1: load my X elements (+ P halo) and apply the FIR map -----
        T xv[X + P];
        if (!ragged) {
            const T* base = st + kHalo + tid * X;
#pragma unroll
            for (int q = 0; q < P; q++) xv[q] = base[q - P];
#pragma unroll
            for (int u = 0; u < X; u++) xv[P + u] = base[u];
        } else {
#pragma unroll
            for (int q = 0; q < X + P; q++) {
                const long long i = g0 - P + q;
                T v = T(0);
                if (i >= 0 && (unsigned long long)i < n) v = prm.x[i];
                else if (i < 0 && i >= -P && prm.x_hist != nullptr) v = prm.x_hist[P + i];
                xv[q] = v;
            }
        }
        // ---- a2: sequential local recurrence with zero state --------------
        T l[X];
#pragma unroll
        for (int u = 0; u < X; u++) {
            T acc = tb.alpha[0] * xv[P + u];
#pragma unroll
            for (int q = 1; q <= P; q++) acc = mad(tb.alpha[q], xv[P + u - q], acc);
#pragma unroll
            for (int r = 1; r <= K; r++)
                if (u - r >= 0) acc = mad(tb.c[r - 1], l[u - r], acc);
            l[u] = acc;
        }
        // local carry A = (l_{X-1}, ..., l_{X-K})
        T v[K];
#pragma unroll
        for (int q = 0; q < K; q++) v[q] = l[X - 1 - q];

        // ---- a3: warp inclusive scan with T(X * 2^s) ----------------------
#pragma unroll
        for (int s2 = 0; s2 < 5; s2++) {
            T o[K];
#pragma unroll
            for (int q = 0; q < K; q++) o[q] = __shfl_up_sync(0xffffffffu, v[q], 1 << s2);
            if (lane >= (1 << s2)) matvec_acc<T, K>(v, tb.Twarp[s2], o);
        }
        T E[K];                                                  // warp-exclusive prefix
#pragma unroll
        for (int q = 0; q < K; q++) {
            T t = __shfl_up_sync(0xffffffffu, v[q], 1);
            E[q] = lane == 0 ? T(0) : t;
        }
        if (lane == 31) {
#pragma unroll
            for (int q = 0; q < K; q++) wagg[warp * kMaxK + q] = v[q];
        }
        named_sync(1, NC);

        // ---- a4: scan of the W warp aggregates with T(32X * 2^s) ----------
        T u_[K];
#pragma unroll
        for (int q = 0; q < K; q++) u_[q] = lane < W ? wagg[lane * kMaxK + q] : T(0);
#pragma unroll
        for (int s2 = 0; s2 < LOGW; s2++) {
            T o[K];
#pragma unroll
            for (int q = 0; q < K; q++) o[q] = __shfl_up_sync(0xffffffffu, u_[q], 1 << s2);
            if (lane >= (1 << s2)) matvec_acc<T, K>(u_, tb.Tblk[s2], o);
        }
        T Pw[K], At[K];
#pragma unroll
        for (int q = 0; q < K; q++) {
            T t = __shfl_sync(0xffffffffu, u_[q], (warp + 31) & 31);
            Pw[q] = warp == 0 ? T(0) : t;
            At[q] = __shfl_sync(0xffffffffu, u_[q], W - 1);     // tile aggregate
        }

        // ---- a5: decoupled look-back (warp 0) -----------------------------
        if (warp == 0) {
            T Gp[K];
            unsigned long long* stj = prm.status + (size_t)j * kStatusWords;
            auto publish = [&](const T (&val)[K], uint32_t tag) {
                T mine = T(0);
#pragma unroll
                for (int q = 0; q < K; q++) if (lane == q) mine = val[q];
                if (lane < K) st_relaxed(stj + lane, ((unsigned long long)tag << 32) | bits(mine));
            };
            if (j == 0) {
#pragma unroll
                for (int q = 0; q < K; q++) Gp[q] = prm.y_hist != nullptr ? prm.y_hist[K - 1 - q] : T(0);
                T G[K];
#pragma unroll
                for (int q = 0; q < K; q++) G[q] = At[q];
                matvec_acc<T, K>(G, tb.Tlb[0], Gp);
                publish(G, tagI);
            } else if (prm.decay) {
                // T(m) == 0: the inclusive carry equals the aggregate, publish
                // it at once; the look-back is a single hop.
                publish(At, tagI);
                const unsigned long long* sp = prm.status + (size_t)(j - 1) * kStatusWords;
                uint32_t word = 0;
                if (lane < K) {
                    unsigned long long w;
                    do { w = ld_relaxed(sp + lane); } while ((uint32_t)(w >> 32) != tagI);
                    word = (uint32_t)w;
                }
#pragma unroll
                for (int q = 0; q < K; q++) Gp[q] = from_bits<T>(__shfl_sync(0xffffffffu, word, q));
            } else {
                publish(At, tagA);
                T acc[K];
                T Tacc[K * kMaxK];
#pragma unroll
                for (int q = 0; q < K; q++) {
                    acc[q] = T(0);
#pragma unroll
                    for (int r = 0; r < kMaxK; r++) Tacc[q * kMaxK + r] = (q == r) ? T(1) : T(0);
                }
                long long base = j - 1;
                for (;;) {
                    const long long jj = base - lane;
                    int stt = 2;                                   // jj < 0: never needed
                    T val[K];
#pragma unroll
                    for (int q = 0; q < K; q++) val[q] = T(0);
                    if (jj >= 0) {
                        const unsigned long long* sp = prm.status + (size_t)jj * kStatusWords;
                        unsigned long long w[K];
#pragma unroll
                        for (int q = 0; q < K; q++) w[q] = ld_relaxed(sp + q);
                        bool allI = true, allA = true;
#pragma unroll
                        for (int q = 0; q < K; q++) {
                            const uint32_t tg = (uint32_t)(w[q] >> 32);
                            allI = allI && tg == tagI;
                            allA = allA && tg == tagA;
                            val[q] = from_bits<T>((uint32_t)w[q]);
                        }
                        stt = allI ? 2 : (allA ? 1 : 0);
                    }
                    const unsigned incl = __ballot_sync(0xffffffffu, stt == 2);
                    const int d = incl ? (__ffs(incl) - 1) : 32;
                    const unsigned need = d >= 31 ? 0xffffffffu : ((2u << d) - 1u);
                    const unsigned notready = __ballot_sync(0xffffffffu, stt == 0);
                    if (notready & need) continue;                 // re-poll the window
                    if (lane > d) {
#pragma unroll
                        for (int q = 0; q < K; q++) val[q] = T(0);
                    }
                    // fold: R = sum_{l<=d} T(l*m) val_l  (tree over lanes)
#pragma unroll
                    for (int s2 = 0; s2 < 5; s2++) {
                        T o[K];
#pragma unroll
                        for (int q = 0; q < K; q++) o[q] = __shfl_down_sync(0xffffffffu, val[q], 1 << s2);
                        matvec_acc<T, K>(val, tb.Tlb[s2], o);
                    }
                    T R[K];
#pragma unroll
                    for (int q = 0; q < K; q++) R[q] = __shfl_sync(0xffffffffu, val[q], 0);
                    matvec_acc<T, K>(acc, Tacc, R);
                    if (d < 32) break;
                    // the next window is 32 tiles further back: Tacc *= T(32m)
                    T nt[K * kMaxK];
#pragma unroll
                    for (int q = 0; q < K; q++)
#pragma unroll
                        for (int r = 0; r < K; r++) {
                            T a2 = T(0);
#pragma unroll
                            for (int t = 0; t < K; t++) a2 = mad(Tacc[q * kMaxK + t], tb.Tlb[5][t * kMaxK + r], a2);
                            nt[q * kMaxK + r] = a2;
                        }
#pragma unroll
                    for (int e = 0; e < K * kMaxK; e++) Tacc[e] = nt[e];
                    base -= 32;
                }
#pragma unroll
                for (int q = 0; q < K; q++) Gp[q] = acc[q];
                T G[K];
#pragma unroll
                for (int q = 0; q < K; q++) G[q] = At[q];
                matvec_acc<T, K>(G, tb.Tlb[0], Gp);
                publish(G, tagI);
            }
            if (lane < K) {
                T mine = T(0);
#pragma unroll
                for (int q = 0; q < K; q++) if (lane == q) mine = Gp[q];
                bcast[lane] = mine;
            }
        }
        named_sync(1, NC);

        // ---- a6: carry-in and correction ----------------------------------
        T Gp[K];
#pragma unroll
        for (int q = 0; q < K; q++) Gp[q] = bcast[q];
        T Win[K];
#pragma unroll
        for (int q = 0; q < K; q++) Win[q] = Pw[q];
        matvec_acc<T, K>(Win, tb.Twin[warp], Gp);              // warp carry-in
        T Sst[K];
#pragma unroll
        for (int q = 0; q < K; q++) {                           // thread carry-in
            T acc = E[q];
#pragma unroll
            for (int r = 0; r < K; r++) acc = mad(Tl[q * K + r], Win[r], acc);
            Sst[q] = acc;
        }
#pragma unroll
        for (int u = 0; u < X; u++) {
            T acc = l[u];
#pragma unroll
            for (int r = 0; r < K; r++) acc = mad(tb.H[u][r], Sst[r], acc);
            l[u] = acc;
        }

        // ---- a7: write back ----------------------------------------------
        if (!ragged) {
            if (STORE) {
                T* base = st + kHalo + tid * X;
#pragma unroll
                for (int u = 0; u < X; u++) base[u] = l[u];
            }
        } else if (STORE) {
#pragma unroll
            for (int u = 0; u < X; u++) {
                const long long i = g0 + u;
                if ((unsigned long long)i < n) prm.y[i] = l[u];
            }
        }
        if (prm.y_tail != nullptr) {
            const long long lo = (long long)n - K;
            if (g0 + X > lo && g0 < (long long)n) {
#pragma unroll
                for (int u = 0; u < X; u++) {
                    const long long i = g0 + u;
                    if (i >= lo && i < (long long)n) prm.y_tail[i - lo] = l[u];
                }
            }
        }
        fence_proxy_async();
        mbar_arrive(&done_bar[s]);
    }
}

}  // namespace dev
}  // namespace plr
