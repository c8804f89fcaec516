// plr_kernels_tmem.cuh -- generic-class (multi-tile look-back) scan kernel
// that parks each tile's chunk values in tensor memory (TMEM) between
// phase A (load, FIR, chunk recurrence, warp/block propagation: a1-a4) and
// phase B (carry-in + correction + store: a6-a7).
//
// Why: for non-decaying signatures the carry of a tile is known only after
// a look-back over its predecessors, an L2 round trip
// of ~1 us under full HBM load.  Hiding it needs several tiles between
// phase A and phase B per CTA; keeping them in shared memory caps the lead at
// one tile for large tiles.  TMEM (256 KB/SM, unused by this bandwidth-bound
// path) holds the per-thread chunk values l_u and warp-exclusive carries of
// up to NT tiles, so shared memory only holds TMA load stages (released as
// soon as phase A has read them) and TMA store stages.
//
//   warps 0..W-1   compute: phase A of tile i, then phase B of tile i-D
//                  (D = NT-1); tcgen05.st / tcgen05.ld move the parked data
//   warp W lane 0  loader: tickets + cp.async.bulk loads
//   warp W lane 1  storer: cp.async.bulk stores of finished tiles
//   warps W+1..    look-back (a5), taking turns over the CTA's tiles
#pragma once
#include "plr_constsig.cuh"
#include "plr_kernels.cuh"

namespace plr {
namespace dev {

// ---------------------------------------------------------------- TMEM -----
__device__ __forceinline__ void tmem_alloc(uint32_t* smem_dst, uint32_t ncols) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;"
                 ::"r"(smem_u32(smem_dst)), "r"(ncols) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_dealloc(uint32_t taddr, uint32_t ncols) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols) : "memory");
}
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

// store / load N consecutive 32-bit columns of this thread's TMEM lane
template <int N>
__device__ __forceinline__ void tmem_st(uint32_t taddr, const uint32_t* v);
template <>
__device__ __forceinline__ void tmem_st<1>(uint32_t taddr, const uint32_t* v) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(taddr), "r"(v[0]) : "memory");
}
template <>
__device__ __forceinline__ void tmem_st<2>(uint32_t taddr, const uint32_t* v) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x2.b32 [%0], {%1, %2};" ::"r"(taddr), "r"(v[0]), "r"(v[1]) : "memory");
}
template <>
__device__ __forceinline__ void tmem_st<4>(uint32_t taddr, const uint32_t* v) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x4.b32 [%0], {%1, %2, %3, %4};"
                 ::"r"(taddr), "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]) : "memory");
}
template <>
__device__ __forceinline__ void tmem_st<8>(uint32_t taddr, const uint32_t* v) {
    asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};"
                 ::"r"(taddr), "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]),
                 "r"(v[7]) : "memory");
}
template <int N>
__device__ __forceinline__ void tmem_ld(uint32_t taddr, uint32_t* v);
template <>
__device__ __forceinline__ void tmem_ld<1>(uint32_t taddr, uint32_t* v) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x1.b32 {%0}, [%1];" : "=r"(v[0]) : "r"(taddr) : "memory");
}
template <>
__device__ __forceinline__ void tmem_ld<2>(uint32_t taddr, uint32_t* v) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x2.b32 {%0, %1}, [%2];" : "=r"(v[0]), "=r"(v[1]) : "r"(taddr) : "memory");
}
template <>
__device__ __forceinline__ void tmem_ld<4>(uint32_t taddr, uint32_t* v) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]) : "r"(taddr) : "memory");
}
template <>
__device__ __forceinline__ void tmem_ld<8>(uint32_t taddr, uint32_t* v) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
                 : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
                 : "r"(taddr) : "memory");
}
// N arbitrary columns as a sum of power-of-two pieces (compile-time)
template <int N>
__device__ __forceinline__ void tmem_st_n(uint32_t taddr, const uint32_t* v) {
    if constexpr (N >= 8) { tmem_st<8>(taddr, v); tmem_st_n<N - 8>(taddr + 8, v + 8); }
    else if constexpr (N >= 4) { tmem_st<4>(taddr, v); tmem_st_n<N - 4>(taddr + 4, v + 4); }
    else if constexpr (N >= 2) { tmem_st<2>(taddr, v); tmem_st_n<N - 2>(taddr + 2, v + 2); }
    else if constexpr (N == 1) { tmem_st<1>(taddr, v); }
}
template <int N>
__device__ __forceinline__ void tmem_ld_n(uint32_t taddr, uint32_t* v) {
    if constexpr (N >= 8) { tmem_ld<8>(taddr, v); tmem_ld_n<N - 8>(taddr + 8, v + 8); }
    else if constexpr (N >= 4) { tmem_ld<4>(taddr, v); tmem_ld_n<N - 4>(taddr + 4, v + 4); }
    else if constexpr (N >= 2) { tmem_ld<2>(taddr, v); tmem_ld_n<N - 2>(taddr + 2, v + 2); }
    else if constexpr (N == 1) { tmem_ld<1>(taddr, v); }
}

template <typename V> __device__ __forceinline__ uint32_t lo_word(V v);
template <> __device__ __forceinline__ uint32_t lo_word<uint32_t>(uint32_t v) { return v; }
template <> __device__ __forceinline__ uint32_t lo_word<float>(float v) { return __float_as_uint(v); }
template <typename V> __device__ __forceinline__ V from_word(uint32_t w);
template <> __device__ __forceinline__ uint32_t from_word<uint32_t>(uint32_t w) { return w; }
template <> __device__ __forceinline__ float from_word<float>(uint32_t w) { return __uint_as_float(w); }

// A value <-> TMEM words (1 word for 32-bit types, 2 for double)
template <typename A> struct AWords { static constexpr int N = sizeof(A) / 4; };
template <typename A>
__device__ __forceinline__ void a_to_words(A v, uint32_t* w) {
    if constexpr (sizeof(A) == 8) {
        const unsigned long long b = __double_as_longlong(v);
        w[0] = (uint32_t)b;
        w[1] = (uint32_t)(b >> 32);
    } else {
        w[0] = lo_word<A>(v);
    }
}
template <typename A>
__device__ __forceinline__ A a_from_words(const uint32_t* w) {
    if constexpr (sizeof(A) == 8) {
        return __longlong_as_double((long long)(((unsigned long long)w[1] << 32) | w[0]));
    } else {
        return from_word<A>(w[0]);
    }
}

// ------------------------------------------------------ shared memory ------
template <typename T, typename A, int K, int X, int W, int SL, int ST, int NT>
struct LayoutT {
    static constexpr int M = 32 * W * X;
    static constexpr int NC = 32 * W;
    static constexpr int SWL = M + kHalo;                                       // words per load stage
    static constexpr size_t off_load = 0;
    static constexpr size_t off_store = (size_t)SL * SWL * sizeof(T);           // ST x M
    static constexpr size_t off_Pw = off_store + (size_t)ST * M * sizeof(T);    // [NT][W][K] A
    static constexpr size_t off_At = off_Pw + (size_t)NT * W * K * sizeof(A);   // [NT][kMaxK]
    static constexpr size_t off_G = off_At + (size_t)NT * kMaxK * sizeof(A);    // [NT][kMaxK]
    static constexpr size_t off_wagg = off_G + (size_t)NT * kMaxK * sizeof(A);  // [NT][W][kMaxK]
    static constexpr size_t off_bar = (off_wagg + (size_t)NT * W * kMaxK * sizeof(A) + 15) & ~(size_t)15;
    // bars: full_L[SL], empty_L[SL], full_T[ST], empty_T[ST], agg[NT], carry[NT]
    static constexpr size_t off_ids = off_bar + (size_t)(2 * SL + 2 * ST + 2 * NT) * 8;
    // ids: tile_of[SL], store_tile[ST], slot_tile[NT] (long long), tmem base (u32),
    // stop position (pipeline index of the compute warps' stop marker)
    static constexpr size_t off_tmem = off_ids + (size_t)(SL + ST + NT) * 8;
    static constexpr size_t off_stop = off_tmem + 4;
    static constexpr size_t off_drain = off_tmem + 8;                           // tickets exhausted (int)
    static constexpr size_t off_lbstat = off_tmem + 16;                         // [kMaxNL][kLbStatWords]
    static constexpr size_t bytes = off_lbstat + kMaxNL * kLbStatWords * 8;
};

// TMEM columns per warp per parked tile: X chunk values + K carries (A words)
template <typename A, int K, int X>
struct TmemCols { static constexpr int CW = X + K * AWords<A>::N; };

// REV: the anticausal recurrence (plr_kernels_small.cuh): ticket j is
// original tile ntiles-1-j read back to front, the ragged tile first (a
// virtual full tile, zero beyond n), the map's halo after the tile (load
// stage layout [tile][halo]); y goes into the store ring in original order.
template <typename T, typename A, int K, int P, int X, int W, int SL, int ST, int NT, int NL, int G, bool STORE,
          int SIG, bool REV = false>
__global__ void __launch_bounds__((W + 1 + NL) * 32, 1)
plr_scan_tmem_kernel(const __grid_constant__ ScanParams<T, A> prm) {
    using L = LayoutT<T, A, K, X, W, SL, ST, NT>;
    constexpr int M = L::M;
    constexpr int SWL = L::SWL;
    constexpr int NC = L::NC;
    constexpr int D = NT - 1;                                    // phase-B lag in tiles
    constexpr int WQ = W / 4;                                    // warps sharing a TMEM lane quarter
    constexpr int CW = TmemCols<A, K, X>::CW;
    constexpr int AWN = AWords<A>::N;
    constexpr int LOGW = (W >= 16) ? 4 : (W >= 8) ? 3 : (W >= 4) ? 2 : 0;
    static_assert((1 << LOGW) == W && W >= 4, "W must be a power of two >= 4");
    static_assert(X >= K && X <= kMaxX && (X & 1), "X must be odd and >= K");
    static_assert(NT >= 2 && NT * WQ * CW <= 512, "TMEM columns");
    static_assert(P <= kHalo, "halo");
    static_assert(G >= 1 && G <= kMaxG && G + 1 <= NT, "look-back unit of G tiles needs G+1 parked tiles");
    // (NL-1) G >= NT used to hang (profiles/r02d_unit_size_hangs.txt): see
    // wait_agg's chained waits and DESIGN.md §10
    constexpr bool DEC = false;

    extern __shared__ __align__(128) unsigned char smem[];
    T* lstage = reinterpret_cast<T*>(smem + L::off_load);
    T* tstage = reinterpret_cast<T*>(smem + L::off_store);
    A* sPw = reinterpret_cast<A*>(smem + L::off_Pw);
    A* sAt = reinterpret_cast<A*>(smem + L::off_At);
    A* sG = reinterpret_cast<A*>(smem + L::off_G);
    A* wagg = reinterpret_cast<A*>(smem + L::off_wagg);
    uint64_t* full_L = reinterpret_cast<uint64_t*>(smem + L::off_bar);
    uint64_t* empty_L = full_L + SL;
    uint64_t* full_T = empty_L + SL;
    uint64_t* empty_T = full_T + ST;
    uint64_t* agg_bar = empty_T + ST;
    uint64_t* carry_bar = agg_bar + NT;
    long long* tile_of = reinterpret_cast<long long*>(smem + L::off_ids);
    long long* store_tile = tile_of + SL;
    long long* slot_tile = store_tile + ST;
    uint32_t* tmem_base_p = reinterpret_cast<uint32_t*>(smem + L::off_tmem);
    volatile int* stop_pos = reinterpret_cast<volatile int*>(smem + L::off_stop);
    volatile int* draining = reinterpret_cast<volatile int*>(smem + L::off_drain);

    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    const long long ntiles = (long long)prm.ntiles;
    const unsigned long long n = prm.n;
    const bool last_ragged = (n % (unsigned long long)M) != 0;
    static_assert(!REV || STORE, "the anticausal pass always stores");
    // the tile the compute warps load element by element (REV: the first)
    auto is_ragged = [&](long long j) -> bool { return last_ragged && j == (REV ? 0 : ntiles - 1); };
    // first element of tile j in the arrays (REV: original tile ntiles-1-j)
    auto tile_start = [&](long long j) -> long long { return (REV ? ntiles - 1 - j : j) * (long long)M; };
    // SIG != 0: the signature's tables are compile-time constants (plr_constsig.cuh)
    constexpr Tables<T, A> kTab = const_tables<T, A>(SIG, X, W, G);
    static_assert(SIG == 0 || const_sig_k(SIG) == K, "signature order");
    const Tables<T, A>& tb = SIG != 0 ? kTab : prm.tab;

    // launch state from device memory (tickets, epoch); the barrier consumes
    // the loads, so they complete before this CTA's first ticket grab
    const unsigned long long tbase = ld_volatile_u64(prm.ticket + 1);
    const uint32_t epoch = (uint32_t)ld_volatile_u64(prm.ticket + 2) + 1u;
    (void)__syncthreads_or((int)(tbase == 0ull && epoch == 0u));

    if (tid == 0) {
        for (int s = 0; s < SL; s++) { mbar_init(&full_L[s], 1); mbar_init(&empty_L[s], NC); }
        for (int s = 0; s < ST; s++) { mbar_init(&full_T[s], NC); mbar_init(&empty_T[s], 1); }
        for (int s = 0; s < NT; s++) { mbar_init(&agg_bar[s], 1); mbar_init(&carry_bar[s], 1); }
        *stop_pos = 1 << 30;
        // few units per CTA (small n): every stop-aware wait polls from the start
        *draining = (long long)((ntiles + G - 1) / G) <= 2LL * gridDim.x ? 1 : 0;
        fence_mbar_init();
    }
    if (warp == 0) tmem_alloc(tmem_base_p, 512);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_base_p;

    // ===================================================== producer warp ===
    if (warp == W) {
        const uint64_t pol = policy_evict_first();
        if (lane == 0) {                                            // loader
            long long unit = 0;
            for (int f = 0;; f++) {
                const int s = f % SL;
                if (f >= SL) mbar_wait_poll(&empty_L[s], (uint32_t)(((f / SL) - 1) & 1));
                // one ticket per look-back unit of G consecutive tiles
                if (f % G == 0) unit = (long long)(atomicAdd(prm.ticket, 1ull) - tbase);
                long long j = unit * G + f % G;
                if (j >= ntiles) j = ntiles;
                tile_of[s] = j;
                if (j >= ntiles) {
                    // the CTA that ends inside the last (partial) unit still makes
                    // its one failing grab: the host counts nunits + grid tickets
                    const long long rel = f % G != 0 ? (long long)(atomicAdd(prm.ticket, 1ull) - tbase) : unit;
                    launch_state_advance(prm.ticket, rel, (unsigned long long)((ntiles + G - 1) / G) + gridDim.x,
                                         tbase, epoch);
                    *draining = 1;                                  // the stop is SL..NT tiles away
                    mbar_arrive(&full_L[s]);
                    break;
                }
                if (is_ragged(j)) { mbar_arrive(&full_L[s]); continue; }
                T* st = lstage + (size_t)s * SWL;
                if (REV) {                                      // the tile, its halo after it (zero beyond n)
                    const long long o = tile_start(j);
#pragma unroll
                    for (int q = 0; q < kHalo; q++) {
                        const unsigned long long i = (unsigned long long)(o + M + q);
                        st[M + q] = (q < P && i < n) ? prm.x[i] : T(0);
                    }
                    mbar_arrive_tx(&full_L[s], M * sizeof(T));
                    bulk_load(st, prm.x + (size_t)o, M * sizeof(T), &full_L[s], pol);
                } else if (j == 0) {
#pragma unroll
                    for (int q = 0; q < kHalo; q++)
                        st[q] = (q >= kHalo - P && prm.x_hist != nullptr) ? prm.x_hist[q - (kHalo - P)] : T(0);
                    mbar_arrive_tx(&full_L[s], M * sizeof(T));
                    bulk_load(st + kHalo, prm.x, M * sizeof(T), &full_L[s], pol);
                } else {
                    mbar_arrive_tx(&full_L[s], SWL * sizeof(T));
                    bulk_load(st, prm.x + (size_t)j * M - kHalo, SWL * sizeof(T), &full_L[s], pol);
                }
            }
        } else if (lane == 1) {                                     // storer
            // up to ST-1 bulk stores in flight; a stage is handed back to the
            // compute warps once the bulk store has finished reading it
            int pend[ST];
            int np = 0;
            for (int t = 0;; t++) {
                const int sT = t % ST;
                mbar_wait_poll(&full_T[sT], (uint32_t)((t / ST) & 1));
                const long long jt = store_tile[sT];
                if (jt >= ntiles) break;
                if (STORE && !is_ragged(jt)) {
                    bulk_store(prm.y + (size_t)tile_start(jt), tstage + (size_t)sT * M, M * sizeof(T), pol);
                    bulk_commit();
                    pend[np++] = sT;
                    if (np > ST - 1) {
                        bulk_wait_read<ST - 1>();                   // the oldest store has read its stage
                        mbar_arrive(&empty_T[pend[0]]);
#pragma unroll
                        for (int q = 0; q + 1 < ST; q++) pend[q] = pend[q + 1];
                        np--;
                    }
                } else {
                    mbar_arrive(&empty_T[sT]);                      // nothing read from this stage
                }
            }
            bulk_wait_all<0>();
            for (int q = 0; q < np; q++) mbar_arrive(&empty_T[pend[q]]);
        }
        return;
    }

    // ===================================================== look-back warps ==
    // Per look-back unit of G consecutive tiles (one ticket): fold the tile
    // aggregates into the unit's local inclusive prefixes L_g = A_g + T(m)
    // L_{g-1}, publish the unit aggregate, look back over the preceding units
    // for the carry G_{J-1} entering the unit, hand
    // every tile its carry-in L_{g-1} + T(g m) G_{J-1} and publish the unit's
    // inclusive carry L_{G-1} + T(G m) G_{J-1}.
    if (warp > W) {
        const uint32_t tagA = 2u * epoch, tagI = 2u * epoch + 1u;
        static_assert(NL <= kMaxNL, "look-back warps");
        const LbStats lbs{reinterpret_cast<unsigned long long*>(smem + L::off_lbstat) + (warp - W - 1) * kLbStatWords};
        lbs.init(lane);
        // aggregate of pipeline position p (false at the stop); parity waits
        // chained so none runs more than one phase ahead of its slot (as in
        // plr_kernels_rr.cuh: positions <= known were seen complete)
        int known = -1;
        auto wait_pos = [&](int q) -> bool {
            return mbar_wait_or_stop(&agg_bar[q % NT], (uint32_t)((q / NT) & 1), stop_pos, q, draining);
        };
        auto wait_agg = [&](int p) -> bool {
            while (known < p - NT) {
                if (!wait_pos(known + NT)) return false;
                known += NT;
            }
            if (!wait_pos(p)) return false;
            if (p > known) known = p;
            return slot_tile[p % NT] < ntiles;
        };
        for (int u = warp - (W + 1);; u += NL) {               // NL look-back warps take turns
            const long long c_start = clock64();
            A Lp[G][K];                                        // local inclusive prefixes
            int cnt = 0;
#pragma unroll
            for (int g = 0; g < G; g++) {
                if (g == cnt && wait_agg(u * G + g)) {
                    const int slot = (u * G + g) % NT;
#pragma unroll
                    for (int q = 0; q < K; q++) Lp[g][q] = sAt[slot * kMaxK + q];
                    if (g > 0) matvec_acc<A, K>(Lp[g], tb.Tm, Lp[g - 1]);
                    cnt++;
                }
            }
            if (cnt == 0) break;
            const long long J = slot_tile[(u * G) % NT] / G;   // unit index
            A Gp[K];                                           // G_{J-1}: carries entering the unit
            if (J == 0) {
#pragma unroll
                for (int q = 0; q < K; q++) Gp[q] = prm.y_hist != nullptr ? A(prm.y_hist[K - 1 - q]) : A(0);
            } else {
                // publish the unit aggregate at once, then look back
                A Ag[K];
#pragma unroll
                for (int q = 0; q < K; q++) Ag[q] = Lp[G - 1][q];
#pragma unroll
                for (int g = 0; g + 1 < G; g++)
                    if (g + 1 == cnt)
#pragma unroll
                        for (int q = 0; q < K; q++) Ag[q] = Lp[g][q];
                publish_status<A, K, DEC>(prm.status, prm.status_mask, J, Ag, tagA, lane);
                // stats: "agg" = idle until the unit's aggregate, "lb" = look-back
                lookback_generic<T, A, K, DEC>(prm, tb, J, lane, tagA, tagI, Gp, lbs, c_start, clock64());
            }
#pragma unroll
            for (int g = 0; g < G; g++) {
                if (g < cnt) {
                    const int slot = (u * G + g) % NT;
                    A C[K];                                    // carry entering tile g
#pragma unroll
                    for (int q = 0; q < K; q++) C[q] = g == 0 ? A(0) : Lp[g > 0 ? g - 1 : 0][q];
                    matvec_acc<A, K>(C, tb.Tsub[g], Gp);
                    if (lane == 0) {
#pragma unroll
                        for (int q = 0; q < K; q++) sG[slot * kMaxK + q] = C[q];
                    }
                }
            }
            __syncwarp();
            if (lane == 0)
                for (int g = 0; g < cnt; g++) mbar_arrive(&carry_bar[(u * G + g) % NT]);
            if (cnt < G) break;                                // the CTA's last (partial) unit
            A Gi[K];
#pragma unroll
            for (int q = 0; q < K; q++) Gi[q] = Lp[G - 1][q];
            matvec_acc<A, K>(Gi, tb.Tpow[0], Gp);              // G_J = L_{G-1} + T(G m) G_{J-1}
            publish_status<A, K, DEC>(prm.status, prm.status_mask, J, Gi, tagI, lane);
        }
        lbs.flush(prm.stats, lane);
        return;
    }

    // ===================================================== compute warps ===
    A Tl[K * K];                                                // T(X*lane)
#pragma unroll
    for (int e = 0; e < K * K; e++) Tl[e] = prm.lane_T[e * 32 + lane];
    // this warp's TMEM lanes (quarter warp%4) and column block
    const uint32_t tmem_w = tmem_base + ((uint32_t)(32 * (warp & 3)) << 16) + (uint32_t)((warp >> 2) * CW);

    auto phaseA = [&](int it) -> long long {
        const int s = it % SL;
        const int slot = it % NT;
        mbar_wait(&full_L[s], (uint32_t)((it / SL) & 1));
        const long long j = tile_of[s];
        if (j >= ntiles) {
            if (tid == 0) { slot_tile[slot] = j; *stop_pos = it; mbar_arrive(&agg_bar[slot]); }
            return j;
        }
        const bool ragged = is_ragged(j);
        const T* st = lstage + (size_t)s * SWL;
        const long long g0 = j * (long long)M + (long long)tid * X;
        // a1: my X elements (+ P halo)
        T xv[X + P];
        if (REV) {                                              // positions v: element o + M-1-v
            const int v0 = tid * X - P;
            if (!ragged) {
#pragma unroll
                for (int q = 0; q < X + P; q++) xv[q] = st[M - 1 - (v0 + q)];
            } else {
                const long long o = tile_start(j);
#pragma unroll
                for (int q = 0; q < X + P; q++) {
                    const unsigned long long i = (unsigned long long)(o + M - 1 - (v0 + q));
                    xv[q] = i < n ? prm.x[i] : T(0);
                }
            }
        } else if (!ragged) {
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
        mbar_arrive(&empty_L[s]);                               // the load stage may be refilled
        // a2: FIR + sequential chunk recurrence with zero state
        uint32_t w[CW];
        A hist[K];
#pragma unroll
        for (int r = 0; r < K; r++) hist[r] = A(0);
#pragma unroll
        for (int u = 0; u < X; u++) {
            T t = tb.alpha[0] * xv[P + u];
#pragma unroll
            for (int q = 1; q <= P; q++) t = mad(tb.alpha[q], xv[P + u - q], t);
            A acc = cvt<A, T>(t);
#pragma unroll
            for (int r = K; r >= 1; r--)
                if (u - r >= 0) acc = mad(tb.c[r - 1], hist[r - 1], acc);
#pragma unroll
            for (int r = K - 1; r >= 1; r--) hist[r] = hist[r - 1];
            hist[0] = acc;
            w[u] = lo_word<T>(cvt<T, A>(acc));
        }
        A v[K];
#pragma unroll
        for (int q = 0; q < K; q++) v[q] = hist[q];
        // a3: warp inclusive scan with T(X * 2^s)
#pragma unroll
        for (int s2 = 0; s2 < 5; s2++) {
            A o[K];
#pragma unroll
            for (int q = 0; q < K; q++) o[q] = shfl_up(v[q], 1 << s2);
            if (lane >= (1 << s2)) matvec_acc<A, K>(v, tb.Twarp[s2], o);
        }
#pragma unroll
        for (int q = 0; q < K; q++) {
            const A e = shfl_up(v[q], 1);
            a_to_words<A>(lane == 0 ? A(0) : e, &w[X + q * AWN]);   // warp-exclusive prefix
        }
        // park chunk values + carries in TMEM for phase B (D tiles later)
        tmem_st_n<CW>(tmem_w + (uint32_t)(slot * WQ * CW), w);
        if (lane == 31) {
#pragma unroll
            for (int q = 0; q < K; q++) wagg[(slot * W + warp) * kMaxK + q] = v[q];
        }
        named_sync(1, NC);
        // a4: scan of the W warp aggregates with T(32X * 2^s)
        A u_[K];
#pragma unroll
        for (int q = 0; q < K; q++) u_[q] = lane < W ? wagg[(slot * W + lane) * kMaxK + q] : A(0);
#pragma unroll
        for (int s2 = 0; s2 < LOGW; s2++) {
            A o[K];
#pragma unroll
            for (int q = 0; q < K; q++) o[q] = shfl_up(u_[q], 1 << s2);
            if (lane >= (1 << s2)) matvec_acc<A, K>(u_, tb.Tblk[s2], o);
        }
        A At[K];
#pragma unroll
        for (int q = 0; q < K; q++) {
            const A pw = shfl_idx(u_[q], (warp + 31) & 31);
            At[q] = shfl_idx(u_[q], W - 1);                     // tile aggregate
            if (lane == 0) sPw[(slot * W + warp) * K + q] = warp == 0 ? A(0) : pw;
            if (tid == 0) sAt[slot * kMaxK + q] = At[q];
        }
        // the look-back warp folds the tile aggregate into its unit's
        tmem_wait_st();
        __syncwarp();
        if (tid == 0) { slot_tile[slot] = j; mbar_arrive(&agg_bar[slot]); }
        return j;
    };

    auto phaseB = [&](int it) {
        const int slot = it % NT;
        const int sT = it % ST;
        mbar_wait(&carry_bar[slot], (uint32_t)((it / NT) & 1));
        // tile id read after the carry wait (tid 0 wrote it before agg_bar,
        // which the carry is ordered after; no barrier follows a stop)
        const long long j = slot_tile[slot];
        const bool ragged = is_ragged(j);
        const long long g0 = j * (long long)M + (long long)tid * X;
        uint32_t w[CW];
        tmem_ld_n<CW>(tmem_w + (uint32_t)(slot * WQ * CW), w);
        A Gp[K], Win[K], Sst[K];
#pragma unroll
        for (int q = 0; q < K; q++) {
            Gp[q] = sG[slot * kMaxK + q];
            Win[q] = sPw[(slot * W + warp) * K + q];
        }
        matvec_acc<A, K>(Win, prm.tab.Twin[warp], Gp);         // warp carry-in (runtime index: parameter tables)
        tmem_wait_ld();
#pragma unroll
        for (int q = 0; q < K; q++) {                           // thread carry-in
            A acc = a_from_words<A>(&w[X + q * AWN]);
#pragma unroll
            for (int r = 0; r < K; r++) acc = mad(Tl[q * K + r], Win[r], acc);
            Sst[q] = acc;
        }
        T Sd[K];
#pragma unroll
        for (int q = 0; q < K; q++) Sd[q] = cvt<T, A>(Sst[q]);
        T yv[X];
#pragma unroll
        for (int u = 0; u < X; u++) {
            T acc = from_word<T>(w[u]);
#pragma unroll
            for (int r = 0; r < K; r++) acc = mad(tb.H[u][r], Sd[r], acc);
            yv[u] = acc;
        }
        mbar_wait(&empty_T[sT], (uint32_t)(((it / ST) & 1) ^ 1));   // store stage free
        if (!ragged) {
            if (STORE) {
                T* stt = tstage + (size_t)sT * M;
#pragma unroll
                for (int u = 0; u < X; u++) stt[REV ? M - 1 - (tid * X + u) : tid * X + u] = yv[u];
            }
        } else if (STORE) {
#pragma unroll
            for (int u = 0; u < X; u++) {
                const long long i = REV ? tile_start(j) + M - 1 - (tid * X + u) : g0 + u;
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
        if (tid == 0) store_tile[sT] = j;
        fence_proxy_async();
        mbar_arrive(&full_T[sT]);
    };

    // phase B of tile nb reads its id from slot_tile[nb % NT]: written at the
    // end of phase A(nb), overwritten only by phase A(nb + NT)
    int na = 0, nb = 0;                                         // phases A / B done
    for (; na < D; na++)
        if (phaseA(na) >= ntiles) break;
    for (bool stop = na < D; !stop;) {
        const long long j = phaseA(na);
        phaseB(nb);
        nb++;
        if (j >= ntiles) stop = true; else na++;
    }
    for (; nb < na; nb++) phaseB(nb);                           // drain
    // stop markers: the storer, and look-back warps waiting beyond the stop
    {
        // STORE = false: the storer releases every stage at once, so it may
        // not have consumed position nb - ST yet; arriving early would
        // complete full_T[sT] a phase ahead of its parity wait (a hang), so
        // wait for the stage as phase B of position nb would.  STORE = true:
        // phase B(nb-1)'s own wait implies the storer consumed position
        // nb-2 >= nb-ST, and waiting here would deadlock: the storer keeps
        // up to ST-1 stages until a further arrival (a ragged last tile is
        // released out of that order), which is this marker's.
        const int sT = nb % ST;
        if constexpr (!STORE) mbar_wait(&empty_T[sT], (uint32_t)(((nb / ST) & 1) ^ 1));
        if (tid == 0) store_tile[sT] = ntiles;
        mbar_arrive(&full_T[sT]);
    }
    // look-back warps waiting beyond the stop see *stop_pos (set by phase A)
    tc_fence_before();
    named_sync(1, NC);
    if (warp == 0) {
        tc_fence_after();
        tmem_dealloc(tmem_base, 512);
    }
}

}  // namespace dev
}  // namespace plr
