// plr_kernels_small.cuh -- the small-n scan kernel.
//
// At n <= a few million elements the persistent, warp-specialised kernels
// pay a fixed cost per launch (deep TMA rings, TMEM allocation, producer /
// storer / look-back roles, multi-tile look-back units) that no tile count
// amortises: 2^20 elements are ~140 tiles, one per SM, and the critical path
// is one load, one look-back and one store (profiles/r02p_small_n_trace.md).
// The paper concedes this regime to an auto-tuned code and lists "better
// heuristics to boost the performance on small inputs" as future work
// (P:951-955); its chunk-size heuristic picks smaller chunks
// for small inputs.
//
// This kernel is the same hierarchy with none of the pipeline:
// one CTA per tile of m = 32 W X elements (all tiles of a small launch are
// resident at once), the tile index from a ticket (so waiting
// CTAs never block an unscheduled predecessor), one TMA bulk load and one
// TMA bulk store, and every intermediate of a thread kept in registers
// between phase A and phase B:
//   a1 map, a2 zero-state chunk, a3 lane scan T(X 2^s), a4 warp-aggregate
//   scan (one warp), a5 decoupled look-back of the k carries by warp 0 (the
//   single hop of DECAY plans, T(m) = 0), a6 seeded serial recurrence from
//   the true incoming state, a7 store.
// When every tile of the launch is resident at once (the host checks
// ntiles <= SMs x CTAs per SM: ScanParams::dec_mask bit 8) the tile index is
// blockIdx.x -- the load is issued at entry, not after a contended ticket
// (1.5 us for 273 CTAs, profiles/r03c_trace_small.jsonl) -- and each CTA's
// one ticket is taken at its END, only to advance the launch state.
//
// REV: the anticausal recurrence y_i = sum_j a_j x_{i+j} + sum_j b_j y_{i+j}
// (zero beyond the end): the causal one over the reversed sequence, the
// other half of a forward-backward (zero-phase) filter pair (P:809-811,
// P:866-868).  Ticket j processes ORIGINAL tile o = ntiles-1-j, read back to
// front, so tiles stay 16-byte aligned; the ragged last tile comes first,
// as a full virtual tile whose positions beyond n are zero (zero inputs
// before the start leave the zero state unchanged), and the map's halo
// lies after the tile instead of before it.
//
// C > 1 (non-decaying signatures, forward, every tile resident): thread-block
// clusters of C CTAs (C consecutive tiles) exchange their tile aggregates
// through distributed shared memory, so the decoupled look-back runs over
// CLUSTER records (one per C tiles): each CTA folds its in-cluster
// predecessors' aggregates read over DSMEM (E_r), the cluster's rank 0
// publishes the cluster aggregate and, after the look-back, its inclusive
// carry, and tile r of cluster c enters with E_r + T(r m) G_{c-1}.  At 2^20
// elements (273 tiles) the per-tile look-back read up to 272 records at once
// from every CTA (a 3.3 us critical path, profiles/r03m_trace_small.jsonl);
// with clusters of 4 (71 co-resident on B200; clusters of 8 fit only 33,
// GPC fragmentation) the look-back reads at most 70.  The carry algebra is P:527-542
// applied to units of C tiles; padding CTAs beyond the last tile have zero
// input (zero state), load and store nothing.
#pragma once
#include "plr_kernels.cuh"

namespace plr {
namespace dev {

// ---- thread-block cluster / distributed shared memory ----------------------
__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_arrive_release() { asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory"); }
__device__ __forceinline__ void cluster_arrive_relaxed() { asm volatile("barrier.cluster.arrive.relaxed.aligned;" ::: "memory"); }
__device__ __forceinline__ void cluster_wait_acquire() { asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory"); }
// value of type A at shared address p of CTA `rank` of this cluster
template <typename A>
__device__ __forceinline__ A ld_dsmem(const A* p, uint32_t rank) {
    uint32_t a;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(a) : "r"(smem_u32(p)), "r"(rank));
    if constexpr (sizeof(A) == 8) {
        unsigned long long v;
        asm volatile("ld.shared::cluster.u64 %0, [%1];" : "=l"(v) : "r"(a) : "memory");
        A out;
        memcpy(&out, &v, 8);
        return out;
    } else {
        uint32_t v;
        asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
        A out;
        memcpy(&out, &v, 4);
        return out;
    }
}

// PLR_TRACE builds: globaltimer stamps of the launch's LAST tile (the end of
// its critical path) into stats words 9..15 (plan made with PLR_STATS=1)
#ifdef PLR_TRACE
#define PLR_STAMP_LAST(i) do { if (prm.stats != nullptr && j == ntiles - 1) { unsigned long long t_; \
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_)); prm.stats[i] = t_; } } while (0)
#else
#define PLR_STAMP_LAST(i) do { } while (0)
#endif

template <typename T, typename A, int K, int X, int W>
struct LayoutS {
    static constexpr int M = 32 * W * X;
    static constexpr size_t off_stage = 0;                                           // kHalo + M words (T)
    static constexpr size_t off_wagg = ((size_t)(kHalo + M) * sizeof(T) + 15) & ~(size_t)15;   // [W][kMaxK] A
    static constexpr size_t off_Pw = off_wagg + (size_t)W * kMaxK * sizeof(A);       // [W][kMaxK] A
    static constexpr size_t off_G = off_Pw + (size_t)W * kMaxK * sizeof(A);          // [kMaxK] A
    static constexpr size_t off_Ac = off_G + kMaxK * sizeof(A);                     // [kMaxK] A: tile aggregate (DSMEM)
    static constexpr size_t off_bar = (off_Ac + kMaxK * sizeof(A) + 15) & ~(size_t)15;
    static constexpr size_t off_tile = off_bar + 8;
    static constexpr size_t bytes = off_tile + 8;
};

template <typename T, typename A, int K, int P, int X, int W, bool REV = false, int C = 1>
__global__ void __launch_bounds__(W * 32, W >= 16 ? 1 : 2)
plr_small_kernel(const __grid_constant__ ScanParams<T, A> prm) {
    using L = LayoutS<T, A, K, X, W>;
    constexpr int LOGC = C >= 8 ? 3 : C >= 4 ? 2 : C >= 2 ? 1 : 0;
    static_assert((1 << LOGC) == C && C <= 8, "cluster of 1, 2, 4 or 8 tiles");
    static_assert(C == 1 || !REV, "cluster launches are forward only");
    constexpr int M = L::M;
    constexpr int LOGW = (W >= 16) ? 4 : (W >= 8) ? 3 : (W >= 4) ? 2 : (W >= 2) ? 1 : 0;
    static_assert((1 << LOGW) == W, "W must be a power of two");
    static_assert(X >= K && X <= kMaxX && (X & 1), "X must be odd and >= K");
    static_assert(P <= kHalo, "halo");
    constexpr bool DECF = false;                     // status layout flag (layout is DEC-independent)

    extern __shared__ __align__(128) unsigned char smem[];
    T* stage = reinterpret_cast<T*>(smem + L::off_stage);
    A* wagg = reinterpret_cast<A*>(smem + L::off_wagg);
    A* sPw = reinterpret_cast<A*>(smem + L::off_Pw);
    A* sG = reinterpret_cast<A*>(smem + L::off_G);
    uint64_t* bar = reinterpret_cast<uint64_t*>(smem + L::off_bar);
    long long* s_tile = reinterpret_cast<long long*>(smem + L::off_tile);

    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    const long long ntiles = (long long)prm.ntiles;
    const unsigned long long n = prm.n;
    const Tables<T, A>& tb = prm.tab;
    const bool decay = prm.decay != 0;               // T(m) == 0: inclusive == aggregate, one-hop look-back

    // launch state (dev::launch_state_advance): one ticket per CTA, so the
    // grab with relative index ntiles - 1 is this launch's last; every CTA
    // reads the base before its own grab
    __shared__ uint32_t s_epoch;
#ifdef PLR_TRACE
    unsigned long long t_entry;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_entry));
#endif
    const bool resident = (prm.dec_mask & 0x100u) != 0;     // all tiles resident: tile = blockIdx.x
    __shared__ unsigned long long s_tbase;
    // one TMA bulk load of tile j (+ halo); the ragged tile is loaded by the
    // compute threads element by element
    auto issue_load = [&](long long j) {
        mbar_init(bar, 1);
        fence_mbar_init();
        const bool ragged_ = REV ? (j == 0 && n % (unsigned long long)M != 0) : (unsigned long long)(j + 1) * M > n;
        if (ragged_) return;
        const uint64_t pol = policy_evict_first();
        if (REV) {                                   // original tile o, halo after it (zero beyond n)
            const long long o = ntiles - 1 - j;
            mbar_arrive_tx(bar, M * sizeof(T));
            bulk_load(stage, prm.x + (size_t)o * M, M * sizeof(T), bar, pol);
#pragma unroll
            for (int q = 0; q < kHalo; q++) {
                const unsigned long long i = (unsigned long long)(o + 1) * M + q;
                stage[M + q] = (q < P && i < n) ? prm.x[i] : T(0);
            }
        } else if (j == 0) {
            mbar_arrive_tx(bar, M * sizeof(T));
            bulk_load(stage + kHalo, prm.x, M * sizeof(T), bar, pol);
#pragma unroll
            for (int q = 0; q < kHalo; q++)
                stage[q] = (q >= kHalo - P && prm.x_hist != nullptr) ? prm.x_hist[q - (kHalo - P)] : T(0);
        } else {
            mbar_arrive_tx(bar, (M + kHalo) * sizeof(T));
            bulk_load(stage, prm.x + (size_t)j * M - kHalo, (M + kHalo) * sizeof(T), bar, pol);
        }
    };
    if (tid == 0) {
        // resident: the tile is known at entry, so its load is issued before
        // the launch state is read (an L2 round trip, ~0.5 us)
        if (resident) issue_load((long long)blockIdx.x);
        const unsigned long long tbase = ld_volatile_u64(prm.ticket + 1);
        const uint32_t epoch = (uint32_t)ld_volatile_u64(prm.ticket + 2) + 1u;
        long long j;
        if (resident) {
            j = (long long)blockIdx.x;
            s_tbase = tbase;
        } else {
            j = (long long)(atomicAdd(prm.ticket, 1ull) - tbase);
            launch_state_advance(prm.ticket, j, (unsigned long long)ntiles, tbase, epoch);
            issue_load(j);
        }
#ifdef PLR_TRACE
        if (prm.stats != nullptr && j == ntiles - 1) prm.stats[9] = t_entry;
#endif
        PLR_STAMP_LAST(10);
        *s_tile = j;
        s_epoch = epoch;
    }
    __syncthreads();
    const long long j = *s_tile;
    const uint32_t epoch = s_epoch;
    const uint32_t tagA = 2u * epoch, tagI = 2u * epoch + 1u;
    const bool ragged = REV ? (j == 0 && n % (unsigned long long)M != 0) : (unsigned long long)(j + 1) * M > n;
    const long long g0 = j * (long long)M + (long long)tid * X;
    // REV: tile position v (processing order) is original element oM + M-1-v
    const long long oM = REV ? (ntiles - 1 - j) * (long long)M : 0;
    const int v0 = tid * X;

    // a1: my X inputs (+ P halo) and the map t (Eq. 2)
    T xv[X + P];
    if (REV) {
        if (!ragged) {
            mbar_wait(bar, 0);
            if (tid == 0) PLR_STAMP_LAST(11);
#pragma unroll
            for (int q = 0; q < X + P; q++) xv[q] = stage[M - 1 - (v0 - P + q)];
        } else {
#pragma unroll
            for (int q = 0; q < X + P; q++) {
                const unsigned long long i = (unsigned long long)(oM + M - 1 - (v0 - P + q));
                xv[q] = i < n ? prm.x[i] : T(0);
            }
        }
    } else if (!ragged) {
        mbar_wait(bar, 0);
        if (tid == 0) PLR_STAMP_LAST(11);
        const T* base = stage + kHalo + tid * X;
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
    T tv[X];
#pragma unroll
    for (int u = 0; u < X; u++) {
        T t = tb.alpha[0] * xv[P + u];
#pragma unroll
        for (int q = 1; q <= P; q++) t = mad(tb.alpha[q], xv[P + u - q], t);
        tv[u] = t;
    }
    // a2: zero-state chunk end state (only the last K values are needed)
    A v[K];
#pragma unroll
    for (int r = 0; r < K; r++) v[r] = A(0);
#pragma unroll
    for (int u = 0; u < X; u++) {
        A acc = cvt<A, T>(tv[u]);
#pragma unroll
        for (int r = K; r >= 1; r--)
            if (u - r >= 0) acc = mad(tb.c[r - 1], v[r - 1], acc);
#pragma unroll
        for (int r = K - 1; r >= 1; r--) v[r] = v[r - 1];
        v[0] = acc;
    }
    // a3: lane scan with T(X 2^s); DECAY skips negligible steps (dec_mask)
#pragma unroll
    for (int s2 = 0; s2 < 5; s2++) {
        if (decay && !((prm.dec_mask >> s2) & 1u)) continue;
        A o[K];
#pragma unroll
        for (int q = 0; q < K; q++) o[q] = shfl_up(v[q], 1 << s2);
        if (lane >= (1 << s2)) matvec_acc<A, K>(v, tb.Twarp[s2], o);
    }
    A e[K];                                          // warp-exclusive prefix of this thread
#pragma unroll
    for (int q = 0; q < K; q++) {
        const A t = shfl_up(v[q], 1);
        e[q] = lane == 0 ? A(0) : t;
    }
    if (lane == 31) {
#pragma unroll
        for (int q = 0; q < K; q++) wagg[warp * kMaxK + q] = v[q];
    }
    __syncthreads();                                 // wagg complete; every stage read done
    if (tid == 0) PLR_STAMP_LAST(12);

    // a4 + a5 (warp 0): warp-aggregate scan, publish, look back, publish
    if (warp == 0) {
        A u_[K];
#pragma unroll
        for (int q = 0; q < K; q++) u_[q] = lane < W ? wagg[lane * kMaxK + q] : A(0);
        const bool blk = !decay || (prm.dec_mask & 32u);
        if (blk) {
#pragma unroll
            for (int s2 = 0; s2 < LOGW; s2++) {
                A o[K];
#pragma unroll
                for (int q = 0; q < K; q++) o[q] = shfl_up(u_[q], 1 << s2);
                if (lane >= (1 << s2)) matvec_acc<A, K>(u_, tb.Tblk[s2], o);
            }
        }
        // (DECAY with T(32X d) == 0: a warp's exclusive prefix is the previous
        // warp's aggregate and the tile aggregate the last warp's)
        A At[K];
#pragma unroll
        for (int q = 0; q < K; q++) {
            const A pw = shfl_up(u_[q], 1);
            if (lane < W) sPw[lane * kMaxK + q] = lane == 0 ? A(0) : pw;
            At[q] = shfl_idx(u_[q], W - 1);
        }
        if constexpr (C > 1) {
            if (lane == 0) {
                A* sAc = reinterpret_cast<A*>(smem + L::off_Ac);
#pragma unroll
                for (int q = 0; q < K; q++) sAc[q] = At[q];
            }
        }
      if constexpr (C == 1) {
        A Gp[K];                                     // carries entering the tile
        if (j == 0) {
#pragma unroll
            for (int q = 0; q < K; q++) Gp[q] = prm.y_hist != nullptr ? A(prm.y_hist[K - 1 - q]) : A(0);
        } else if (decay) {
            publish_status<A, K, DECF>(prm.status, prm.status_mask, j, At, tagI, lane);
            A g[K];
            if (lane == 0) {
                int ns = 32;
                SpinGuard guard;
                while (read_status<A, K, DECF>(prm.status, prm.status_mask, j - 1, g, tagA, tagI) != 2) {
                    guard(9);
                    __nanosleep(ns);
                    ns = ns < 128 ? 2 * ns : ns;
                }
            }
#pragma unroll
            for (int q = 0; q < K; q++) Gp[q] = shfl_idx(lane == 0 ? g[q] : A(0), 0);
        } else {
            publish_status<A, K, DECF>(prm.status, prm.status_mask, j, At, tagA, lane);
            __shared__ unsigned long long s_lbst[kLbStatWords];   // debug counters (PLR_STATS=1)
            const LbStats lbs{s_lbst};
            lbs.init(lane);
            __syncwarp();
            // every predecessor publishes at about the same time: the widest
            // window from the start, short flat sleeps
            lookback_generic<T, A, K, DECF>(prm, tb, j, lane, tagA, tagI, Gp, lbs, 0, 0, 64, true);
            __syncwarp();
            lbs.flush(prm.stats, lane);
        }
        if (lane == 0) PLR_STAMP_LAST(13);
        if (!decay || j == 0) {
            A G[K];
#pragma unroll
            for (int q = 0; q < K; q++) G[q] = At[q];
            matvec_acc<A, K>(G, tb.Tm, Gp);          // G_j = A_j + T(m) G_{j-1}
            publish_status<A, K, DECF>(prm.status, prm.status_mask, j, G, tagI, lane);
        }
        if (lane == 0) {
#pragma unroll
            for (int q = 0; q < K; q++) sG[q] = Gp[q];
        }
      }
    }
    if constexpr (C > 1) {
        // every CTA's aggregate is in its shared memory (barrier #1); warp 0
        // reads the cluster's C aggregates, then arrives on barrier #2 (its
        // shared memory may go once every CTA is past its DSMEM reads: the
        // wait is at the end of the kernel)
        __syncwarp();
        cluster_arrive_release();
        cluster_wait_acquire();
        if (warp == 0) {
            const uint32_t r = cluster_rank();               // == j mod C (tile = blockIdx.x)
            A am[K];
            const A* sAc = reinterpret_cast<const A*>(smem + L::off_Ac);
#pragma unroll
            for (int q = 0; q < K; q++) am[q] = lane < C ? ld_dsmem<A>(sAc + q, (uint32_t)lane) : A(0);
            __syncwarp();
            cluster_arrive_relaxed();
            // E_r = sum_{i<r} T((r-1-i) m) A_i (zero carry into the cluster),
            // Ac = the cluster aggregate; every lane folds redundantly
            A E[K], Er[K];
#pragma unroll
            for (int q = 0; q < K; q++) { E[q] = A(0); Er[q] = A(0); }
#pragma unroll
            for (int i = 0; i < C; i++) {
                A ai[K];
#pragma unroll
                for (int q = 0; q < K; q++) ai[q] = shfl_idx(am[q], i);
                if ((uint32_t)i == r) {
#pragma unroll
                    for (int q = 0; q < K; q++) Er[q] = E[q];
                }
                matvec_acc<A, K>(ai, tb.Tm, E);              // E <- A_i + T(m) E
#pragma unroll
                for (int q = 0; q < K; q++) E[q] = ai[q];
            }
            const long long c = j / C;
            A Gc[K];                                          // carries entering cluster c
            if (c == 0) {
#pragma unroll
                for (int q = 0; q < K; q++) Gc[q] = prm.y_hist != nullptr ? A(prm.y_hist[K - 1 - q]) : A(0);
            } else {
                if (r == 0) publish_status<A, K, DECF>(prm.status, prm.status_mask, c, E, tagA, lane);
                __shared__ unsigned long long s_lbst[kLbStatWords];   // debug counters (PLR_STATS=1)
                const LbStats lbs{s_lbst};
                lbs.init(lane);
                __syncwarp();
                lookback_generic<T, A, K, DECF, LOGC>(prm, tb, c, lane, tagA, tagI, Gc, lbs, 0, 0, 64, true);
                __syncwarp();
                lbs.flush(prm.stats, lane);
            }
            if (lane == 0) PLR_STAMP_LAST(13);
            if (r == 0) {                                     // G_c = Ac + T(C m) G_{c-1}
                A G[K];
#pragma unroll
                for (int q = 0; q < K; q++) G[q] = E[q];
                matvec_acc<A, K>(G, tb.Tpow[LOGC], Gc);
                publish_status<A, K, DECF>(prm.status, prm.status_mask, c, G, tagI, lane);
            }
            // carry entering tile j: E_r + T(r m) G_{c-1}, T(r m) from the binary powers T(2^b m)
#pragma unroll
            for (int b = 0; b < LOGC; b++) {
                if ((r >> b) & 1u) {
                    A t2[K];
#pragma unroll
                    for (int q = 0; q < K; q++) t2[q] = A(0);
                    matvec_acc<A, K>(t2, tb.Tpow[b], Gc);
#pragma unroll
                    for (int q = 0; q < K; q++) Gc[q] = t2[q];
                }
            }
            if (lane == 0) {
#pragma unroll
                for (int q = 0; q < K; q++) sG[q] = Er[q] + Gc[q];
            }
        } else {
            __syncwarp();
            cluster_arrive_relaxed();
        }
    }
    __syncthreads();

    // a6: carry-in of the warp and of the thread, then the serial recurrence
    // of P:206-214 over the thread's X elements seeded with it
    A Gp[K], Win[K], S[K];
#pragma unroll
    for (int q = 0; q < K; q++) {
        Gp[q] = sG[q];
        Win[q] = sPw[warp * kMaxK + q];
    }
    if (decay && !(prm.dec_mask & 32u)) {            // T(32X w) == 0 for w >= 1
        if (warp == 0) {
#pragma unroll
            for (int q = 0; q < K; q++) Win[q] = Gp[q];
        }
    } else {
        matvec_acc<A, K>(Win, tb.Twin[warp], Gp);
    }
#pragma unroll
    for (int q = 0; q < K; q++) {
        A acc = e[q];
#pragma unroll
        for (int r = 0; r < K; r++) acc = mad(prm.lane_T[(q * K + r) * 32 + lane], Win[r], acc);
        S[q] = acc;
    }
    T yv[X];
#pragma unroll
    for (int u = 0; u < X; u++) {
        A acc = cvt<A, T>(tv[u]);
#pragma unroll
        for (int r = K; r >= 1; r--) acc = mad(tb.c[r - 1], S[r - 1], acc);
#pragma unroll
        for (int r = K - 1; r >= 1; r--) S[r] = S[r - 1];
        S[0] = acc;
        yv[u] = cvt<T, A>(acc);
    }
    // a7: y into the stage and one TMA bulk store (ragged tile: direct stores)
    const bool store = prm.y != nullptr;
    if (REV) {
        if (!ragged) {
#pragma unroll
            for (int u = 0; u < X; u++) stage[M - 1 - (v0 + u)] = yv[u];
        } else {
#pragma unroll
            for (int u = 0; u < X; u++) {
                const unsigned long long i = (unsigned long long)(oM + M - 1 - (v0 + u));
                if (i < n) prm.y[i] = yv[u];
            }
        }
    } else if (!ragged) {
        if (store) {
            T* base = stage + kHalo + tid * X;
#pragma unroll
            for (int u = 0; u < X; u++) base[u] = yv[u];
        }
    } else if (store) {
#pragma unroll
        for (int u = 0; u < X; u++) {
            const long long i = g0 + u;
            if ((unsigned long long)i < n) prm.y[i] = yv[u];
        }
    }
    if (!REV && prm.y_tail != nullptr) {
        const long long lo = (long long)n - K;
        if (g0 + X > lo && g0 < (long long)n) {
#pragma unroll
            for (int u = 0; u < X; u++) {
                const long long i = g0 + u;
                if (i >= lo && i < (long long)n) prm.y_tail[i - lo] = yv[u];
            }
        }
    }
    if (!ragged && store) {
        fence_proxy_async();
        __syncthreads();
        if (tid == 0) PLR_STAMP_LAST(14);
        if (tid == 0) {
            if (REV) bulk_store(prm.y + (size_t)oM, stage, M * sizeof(T), policy_evict_first());
            else bulk_store(prm.y + (size_t)j * M, stage + kHalo, M * sizeof(T), policy_evict_first());
            bulk_commit();
            bulk_wait_read<0>();                     // smem stays valid until the store has read it
            PLR_STAMP_LAST(15);
        }
    }
    if (resident && tid == 0) {                      // the CTA's one ticket: the last one advances the state
        const long long rel = (long long)(atomicAdd(prm.ticket, 1ull) - s_tbase);
        launch_state_advance(prm.ticket, rel, (unsigned long long)gridDim.x, s_tbase, epoch);
    }
    if constexpr (C > 1) cluster_wait_acquire();     // barrier #2: no CTA of the cluster reads this smem any more
}

}  // namespace dev
}  // namespace plr
