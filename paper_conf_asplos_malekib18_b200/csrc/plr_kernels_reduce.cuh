// plr_kernels_reduce.cuh -- the reduce-only pass of the sharded schedule for
// non-decaying signatures (the end state E_r of a segment
// with zero history, read n, write nothing).
//
// A segment's end state needs no look-back: with zero history it is the
// ordered fold of the tile aggregates, E = sum_j T((J-1-j) m) A_j (the carry
// algebra of P:527-542 applied to the whole segment), so every CTA streams a
// CONTIGUOUS range of tiles, folds its aggregates in order
// (acc = T(m) acc + A_j), and the last CTA to finish folds the CTAs' records
// (E = T(L_c) E + acc_c).  Phase A of the scan (a1 map, a2 zero-state chunk,
// a3 lane scan, a4 warp-aggregate scan) is all the per-tile work; loads are
// TMA bulk copies into an S-stage ring, so the pass runs at the read
// roofline instead of the single-pass kernels' look-back pipeline.
//
// The last tile of a ragged segment is evaluated as a virtual tile ending at
// element n whose map outputs before the tile start are zero (a zero input
// leaves a zero state unchanged), and folded with T(r), r = its length.
#pragma once
#include "plr_kernels.cuh"

namespace plr {
namespace dev {

template <typename T, typename A, int K, int X, int W, int S>
struct LayoutRd {
    static constexpr int M = 32 * W * X;
    static constexpr int SW = M + kHalo;
    static constexpr size_t off_stage = 0;                                        // S x SW (T)
    static constexpr size_t off_wagg = ((size_t)S * SW * sizeof(T) + 15) & ~(size_t)15;   // [2][W][kMaxK] A
    static constexpr size_t off_acc = off_wagg + 2 * (size_t)W * kMaxK * sizeof(A);  // [kMaxK] A: the CTA's fold
    static constexpr size_t off_bar = (off_acc + kMaxK * sizeof(A) + 15) & ~(size_t)15;
    static constexpr size_t bytes = off_bar + 2 * S * 8 + 16;                     // full[S], empty[S], flag
};

// per-CTA record in the plan's status array (stride kStatusMaxBytes):
// K accumulation-type words, then the range length in elements
template <typename A>
__device__ __forceinline__ unsigned long long* rd_record(unsigned long long* status, int c) {
    return status + (size_t)c * (kStatusMaxBytes / 8);
}

// M^L for the companion matrix of (1: c) (A ring), square-and-multiply
template <typename A, int K>
__device__ void companion_pow(const A* c, unsigned long long L, A* R) {
    A B[kMaxK * kMaxK], P[kMaxK * kMaxK];
    for (int e = 0; e < kMaxK * kMaxK; e++) { R[e] = A(0); B[e] = A(0); }
    for (int q = 0; q < K; q++) R[q * kMaxK + q] = A(1);
    for (int r = 0; r < K; r++) B[r] = c[r];
    for (int q = 1; q < K; q++) B[q * kMaxK + q - 1] = A(1);
    auto mul = [&](const A* X1, const A* Y1, A* Z) {
        for (int q = 0; q < K; q++)
            for (int r = 0; r < K; r++) {
                A acc = A(0);
                for (int t = 0; t < K; t++) acc = mad(X1[q * kMaxK + t], Y1[t * kMaxK + r], acc);
                P[q * kMaxK + r] = acc;
            }
        for (int e = 0; e < kMaxK * kMaxK; e++) Z[e] = P[e];
    };
    while (L) {
        if (L & 1) mul(R, B, R);
        L >>= 1;
        if (L) mul(B, B, B);
    }
}

template <typename T, typename A, int K, int P, int X, int W, int S>
__global__ void __launch_bounds__((W + 1) * 32, 2)
plr_reduce_kernel(const __grid_constant__ ScanParams<T, A> prm) {
    using L = LayoutRd<T, A, K, X, W, S>;
    constexpr int M = L::M;
    constexpr int SW = L::SW;
    constexpr int NC = 32 * W;
    constexpr int LOGW = (W >= 16) ? 4 : (W >= 8) ? 3 : (W >= 4) ? 2 : 0;
    static_assert((1 << LOGW) == W && W >= 4, "W must be a power of two >= 4");
    static_assert(X >= K && X <= kMaxX && (X & 1), "X must be odd and >= K");
    static_assert(P <= kHalo, "halo");
    static_assert(K * sizeof(A) + 8 <= kStatusMaxBytes, "record");

    extern __shared__ __align__(128) unsigned char smem[];
    T* stages = reinterpret_cast<T*>(smem + L::off_stage);
    A* wagg = reinterpret_cast<A*>(smem + L::off_wagg);
    A* sacc = reinterpret_cast<A*>(smem + L::off_acc);
    uint64_t* full = reinterpret_cast<uint64_t*>(smem + L::off_bar);
    uint64_t* empty = full + S;
    int* s_last = reinterpret_cast<int*>(empty + S);

    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    const unsigned long long n = prm.n;
    const long long ntiles = (long long)prm.ntiles;
    const bool last_ragged = (n % (unsigned long long)M) != 0;
    const Tables<T, A>& tb = prm.tab;
    const int grid = (int)gridDim.x;
    const long long q = (ntiles + grid - 1) / grid;              // tiles per CTA (contiguous)
    const long long t0 = (long long)blockIdx.x * q;
    const long long t1 = t0 + q < ntiles ? t0 + q : ntiles;
    const int nt = t1 > t0 ? (int)(t1 - t0) : 0;

    // launch state (read before this CTA's one grab at the end)
    const unsigned long long tbase = ld_volatile_u64(prm.ticket + 1);
    const uint32_t epoch = (uint32_t)ld_volatile_u64(prm.ticket + 2) + 1u;
    if (tid == 0) {
        for (int s = 0; s < S; s++) { mbar_init(&full[s], 1); mbar_init(&empty[s], NC); }
        fence_mbar_init();
    }
    (void)__syncthreads_or((int)(tbase == 0ull && epoch == 0u));

    if (warp == W) {                                             // producer: TMA loads of the CTA's range
        if (lane == 0) {
            const uint64_t pol = policy_evict_first();
            for (int f = 0; f < nt; f++) {
                const int s = f % S;
                if (f >= S) mbar_wait_poll(&empty[s], (uint32_t)(((f / S) - 1) & 1));
                const long long j = t0 + f;
                if (j == ntiles - 1 && last_ragged) { mbar_arrive(&full[s]); continue; }   // compute loads it
                T* st = stages + (size_t)s * SW;
                if (j == 0) {
#pragma unroll
                    for (int e = 0; e < kHalo; e++)
                        st[e] = (e >= kHalo - P && prm.x_hist != nullptr) ? prm.x_hist[e - (kHalo - P)] : T(0);
                    mbar_arrive_tx(&full[s], M * sizeof(T));
                    bulk_load(st + kHalo, prm.x, M * sizeof(T), &full[s], pol);
                } else {
                    mbar_arrive_tx(&full[s], SW * sizeof(T));
                    bulk_load(st, prm.x + (size_t)j * M - kHalo, SW * sizeof(T), &full[s], pol);
                }
            }
        }
    } else {
        // the fold of the CTA's tile aggregates lives in sacc; tile f's warp-
        // aggregate scan and fold run in warp f mod W (ordered after tile
        // f-1's fold by tile f's named barrier), so no warp idles the others
        if (tid == 0) {
#pragma unroll
            for (int e = 0; e < K; e++) sacc[e] = A(0);
        }
        for (int f = 0; f < nt; f++) {
            const int s = f % S;
            const long long j = t0 + f;
            const bool ragged = j == ntiles - 1 && last_ragged;
            mbar_wait(&full[s], (uint32_t)((f / S) & 1));
            // a1: inputs; the ragged tile is the virtual tile [n - M, n) with
            // map outputs before j M set to zero
            T xv[X + P];
            long long gv = 0;                                    // global index of xv[P]
            if (!ragged) {
                const T* base = stages + (size_t)s * SW + kHalo + tid * X;
#pragma unroll
                for (int e = 0; e < P; e++) xv[e] = base[e - P];
#pragma unroll
                for (int u = 0; u < X; u++) xv[P + u] = base[u];
            } else {
                gv = (long long)n - M + (long long)tid * X;
#pragma unroll
                for (int e = 0; e < X + P; e++) {
                    const long long i = gv - P + e;
                    T v = T(0);
                    if (i >= 0 && (unsigned long long)i < n) v = prm.x[i];
                    else if (i < 0 && i >= -P && prm.x_hist != nullptr) v = prm.x_hist[P + i];
                    xv[e] = v;
                }
            }
            mbar_arrive(&empty[s]);
            // a2: zero-state chunk end state
            A v[K];
#pragma unroll
            for (int r = 0; r < K; r++) v[r] = A(0);
#pragma unroll
            for (int u = 0; u < X; u++) {
                T t = tb.alpha[0] * xv[P + u];
#pragma unroll
                for (int e = 1; e <= P; e++) t = mad(tb.alpha[e], xv[P + u - e], t);
                if (ragged && gv + u < j * (long long)M) t = T(0);
                A a_ = cvt<A, T>(t);
#pragma unroll
                for (int r = K; r >= 1; r--)
                    if (u - r >= 0) a_ = mad(tb.c[r - 1], v[r - 1], a_);
#pragma unroll
                for (int r = K - 1; r >= 1; r--) v[r] = v[r - 1];
                v[0] = a_;
            }
            // a3: lane scan with T(X 2^s)
#pragma unroll
            for (int s2 = 0; s2 < 5; s2++) {
                A o[K];
#pragma unroll
                for (int e = 0; e < K; e++) o[e] = shfl_up(v[e], 1 << s2);
                if (lane >= (1 << s2)) matvec_acc<A, K>(v, tb.Twarp[s2], o);
            }
            A* wg = wagg + (size_t)(f & 1) * W * kMaxK;
            if (lane == 31) {
#pragma unroll
                for (int e = 0; e < K; e++) wg[warp * kMaxK + e] = v[e];
            }
            named_sync(1, NC);
            // a4 (warp f mod W): tile aggregate, folded in order: acc = T(L) acc + A_tile
            if (warp == f % W) {
                A acc[K];
#pragma unroll
                for (int e = 0; e < K; e++) acc[e] = sacc[e];
                A u_[K];
#pragma unroll
                for (int e = 0; e < K; e++) u_[e] = lane < W ? wg[lane * kMaxK + e] : A(0);
#pragma unroll
                for (int s2 = 0; s2 < LOGW; s2++) {
                    A o[K];
#pragma unroll
                    for (int e = 0; e < K; e++) o[e] = shfl_up(u_[e], 1 << s2);
                    if (lane >= (1 << s2)) matvec_acc<A, K>(u_, tb.Tblk[s2], o);
                }
                A At[K];
#pragma unroll
                for (int e = 0; e < K; e++) At[e] = shfl_idx(u_[e], W - 1);
                if (!ragged) {
                    matvec_acc<A, K>(At, tb.Tm, acc);
                } else {                                         // the virtual tile: fold with T(r)
                    A Tr[kMaxK * kMaxK];
                    companion_pow<A, K>(tb.c, n - (unsigned long long)j * M, Tr);
                    matvec_acc<A, K>(At, Tr, acc);
                }
                __syncwarp();
                if (lane == 0) {
#pragma unroll
                    for (int e = 0; e < K; e++) sacc[e] = At[e];
                }
            }
        }
        named_sync(1, NC);                                       // the last fold is in sacc
        // the CTA's record: its fold and its length in elements
        if (warp == 0 && lane == 0) {
            unsigned long long* rec = rd_record<A>(prm.status, blockIdx.x);
            A* ra = reinterpret_cast<A*>(rec);
#pragma unroll
            for (int e = 0; e < K; e++) ra[e] = sacc[e];
            const unsigned long long len = nt == 0 ? 0ull
                : (t1 == ntiles ? n - (unsigned long long)t0 * M : (unsigned long long)nt * M);
            rec[(kStatusMaxBytes / 8) - 1] = len;
            __threadfence();
            const long long rel = (long long)(atomicAdd(prm.ticket, 1ull) - tbase);
            launch_state_advance(prm.ticket, rel, (unsigned long long)grid, tbase, epoch);
            *s_last = rel == grid - 1;
        }
    }
    __syncthreads();
    // the last CTA folds the records in order: E = T(L_c) E + acc_c.  Every
    // thread first copies records tid, tid + blockDim, ... into the (now idle)
    // stage ring, so the grid's records cost one L2 round trip, not one per
    // record (a serial chain of dependent loads was ~0.3 us x grid)
    if (!*s_last) return;
    constexpr int RW = kMaxK;                                     // values per copied record
    static_assert(L::off_wagg >= (size_t)kRedMaxGrid * (8 + RW * sizeof(A)), "record copy fits the stage ring");
    unsigned long long* slen = reinterpret_cast<unsigned long long*>(smem + L::off_stage);
    A* srec = reinterpret_cast<A*>(slen + grid);
    __threadfence();
    for (int c = tid; c < grid; c += (int)blockDim.x) {
        const volatile unsigned long long* rec = rd_record<A>(prm.status, c);
        const volatile A* ra = reinterpret_cast<const volatile A*>(rec);
        slen[c] = rec[(kStatusMaxBytes / 8) - 1];
#pragma unroll
        for (int e = 0; e < K; e++) srec[(size_t)c * RW + e] = ra[e];
    }
    __syncthreads();
    if (tid == 0) {
        A E[K];
#pragma unroll
        for (int e = 0; e < K; e++) E[e] = A(0);
        A Tq[kMaxK * kMaxK];
        companion_pow<A, K>(tb.c, (unsigned long long)q * M, Tq);
        for (int c = 0; c < grid; c++) {
            const unsigned long long len = slen[c];
            if (len == 0) continue;
            A a_[K];
#pragma unroll
            for (int e = 0; e < K; e++) a_[e] = srec[(size_t)c * RW + e];
            if (len == (unsigned long long)q * M) {
                matvec_acc<A, K>(a_, Tq, E);
            } else {
                A Tl2[kMaxK * kMaxK];
                companion_pow<A, K>(tb.c, len, Tl2);
                matvec_acc<A, K>(a_, Tl2, E);
            }
#pragma unroll
            for (int e = 0; e < K; e++) E[e] = a_[e];
        }
        if (prm.y_tail != nullptr) {                            // y_{n-K} .. y_{n-1}
#pragma unroll
            for (int e = 0; e < K; e++) prm.y_tail[K - 1 - e] = cvt<T, A>(E[e]);
        }
    }
}

}  // namespace dev
}  // namespace plr
