// plr_kernels_rr.cuh -- generic-class (multi-tile look-back) scan kernel with
// a long phase-A / phase-B lag: phase B re-reads its tile from L2 and
// recomputes the chunk from the true carry-in instead of correcting parked
// chunk values.
//
// Why: for non-decaying signatures a tile's carry is known only after a
// look-back over the preceding units, ~2-4 L2 round
// trips of 1.5 us each under full HBM load.  Hiding that needs a lag of many
// tiles between phase A (carry production) and phase B (output).  Parking the
// chunk values of every tile in flight (TMEM, 256 KB/SM) caps the lag at ~6
// tiles; here only the k-word warp-exclusive carry of each thread is parked
// in TMEM, the input tile is fetched again from L2 for phase B (it was read
// from HBM by phase A NS-1 tiles earlier: ~NS x 4.5 MB of traffic ago, far
// below the 126 MB L2), and phase B evaluates the serial recurrence of
// P:206-214 seeded with the thread's true incoming state.  HBM traffic stays
// one read and one write per element; L2 serves the second read.
//
//   warps 0..W-1   compute: phase A of tile i (a1-a4: load, FIR, zero-state
//                  chunk end state, warp / block carry scans), then phase B
//                  of tile i-(NS-1) (a6-a7: carry-in, seeded recurrence, y)
//   warp W lane 0  loader A: tickets (one per unit of G tiles) +
//                  cp.async.bulk loads of x for phase A (HBM)
//   warp W lane 1  loader B: cp.async.bulk re-loads of x for phase B (L2)
//   warp W lane 2  storer: cp.async.bulk stores of y from the phase-B stage
//   warps W+1..    look-back (a5) per unit of G tiles, taking turns
#pragma once
#include "plr_constsig.cuh"
#include "plr_kernels.cuh"
#include "plr_kernels_tmem.cuh"

namespace plr {
namespace dev {

__device__ __forceinline__ uint64_t policy_evict_last() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ uint64_t policy_evict_normal() {
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}

// ------------------------------------------------------ shared memory ------
template <typename T, typename A, int K, int X, int W, int SA, int SB, int NS>
struct LayoutR {
    static constexpr int M = 32 * W * X;
    static constexpr int SWL = M + kHalo;                                       // words per stage
    static constexpr size_t off_A = 0;                                          // SA x SWL
    static constexpr size_t off_B = (size_t)SA * SWL * sizeof(T);               // SB x SWL
    static constexpr size_t off_Pw = off_B + (size_t)SB * SWL * sizeof(T);      // [NS][W][K] A
    static constexpr size_t off_At = off_Pw + (size_t)NS * W * K * sizeof(A);   // [NS][kMaxK]
    static constexpr size_t off_G = off_At + (size_t)NS * kMaxK * sizeof(A);    // [NS][kMaxK]
    static constexpr size_t off_wagg = off_G + (size_t)NS * kMaxK * sizeof(A);  // [NS][W][kMaxK]
    static constexpr size_t off_bar = (off_wagg + (size_t)NS * W * kMaxK * sizeof(A) + 15) & ~(size_t)15;
    // bars: fullA[SA], emptyA[SA], fullB[SB], emptyB[SB], yfull[SB], agg[NS], carry[NS]
    static constexpr size_t off_ids = off_bar + (size_t)(2 * SA + 3 * SB + 2 * NS) * 8;
    // ids: tileA[SA], slot_tile[NS], store_tile[SB] (long long)
    static constexpr size_t off_tmem = off_ids + (size_t)(SA + NS + SB) * 8;
    static constexpr size_t off_stop = off_tmem + 4;
    static constexpr size_t off_drain = off_tmem + 8;                           // tickets exhausted (int)
    static constexpr size_t off_lbstat = off_tmem + 16;                         // [kMaxNL][kLbStatWords]
    static constexpr size_t bytes = off_lbstat + kMaxNL * kLbStatWords * 8;
};

// TMEM columns per warp per slot: the K-word warp-exclusive carry (A words)
template <typename A, int K>
struct RrCols { static constexpr int CW = K * AWords<A>::N; };

// REV: the anticausal recurrence (plr_kernels_small.cuh): ticket j is
// original tile ntiles-1-j read back to front, the ragged tile first (a
// virtual full tile, zero beyond n), the map's halo after the tile (stage
// layout [tile][halo]); phase B writes y into the stage in original order.
// The REV paths are separate `if constexpr` branches, so the forward kernel's
// code is the one measured before they existed (a shared formulation cost
// tuple2 1.5 %, profiles/r04o_ab_rr.txt).
template <typename T, typename A, int K, int P, int X, int W, int SA, int SB, int NS, int NL, int G, bool STORE,
          int SIG, bool REV = false>
__global__ void __launch_bounds__((W + 1 + NL) * 32, 1)
plr_scan_rr_kernel(const __grid_constant__ ScanParams<T, A> prm) {
    using L = LayoutR<T, A, K, X, W, SA, SB, NS>;
    constexpr int M = L::M;
    constexpr int SWL = L::SWL;
    constexpr int NC = 32 * W;
    constexpr int D = NS - 1;                                    // phase-B lag in tiles
    constexpr int WQ = W / 4;                                    // warps sharing a TMEM lane quarter
    constexpr int CW = RrCols<A, K>::CW;
    constexpr int AWN = AWords<A>::N;
    constexpr int LOGW = (W >= 16) ? 4 : (W >= 8) ? 3 : (W >= 4) ? 2 : 0;
    static_assert((1 << LOGW) == W && W >= 4, "W must be a power of two >= 4");
    static_assert(X >= K && X <= kMaxX && (X & 1), "X must be odd and >= K");
    static_assert(NS * WQ * CW <= 512, "TMEM columns");
    constexpr uint32_t TCOLS = NS * WQ * CW <= 32 ? 32 : NS * WQ * CW <= 64 ? 64 : NS * WQ * CW <= 128 ? 128
                             : NS * WQ * CW <= 256 ? 256 : 512;   // power-of-two allocation
    static_assert(P <= kHalo, "halo");
    static_assert(G >= 1 && G <= kMaxG && G + 1 <= NS, "look-back unit of G tiles needs G+1 slots");
    // (NL-1) G >= NS used to hang (profiles/r02d_unit_size_hangs.txt): a
    // look-back warp's first agg wait of its next unit ran more than one
    // phase ahead of its slot; wait_agg now chains its waits
    static_assert(SB >= 2 && SA >= 1, "stages");
    constexpr bool DEC = false;

    extern __shared__ __align__(128) unsigned char smem[];
    T* stA = reinterpret_cast<T*>(smem + L::off_A);
    T* stB = reinterpret_cast<T*>(smem + L::off_B);
    A* sPw = reinterpret_cast<A*>(smem + L::off_Pw);
    A* sAt = reinterpret_cast<A*>(smem + L::off_At);
    A* sG = reinterpret_cast<A*>(smem + L::off_G);
    A* wagg = reinterpret_cast<A*>(smem + L::off_wagg);
    uint64_t* fullA = reinterpret_cast<uint64_t*>(smem + L::off_bar);
    uint64_t* emptyA = fullA + SA;
    uint64_t* fullB = emptyA + SA;
    uint64_t* emptyB = fullB + SB;
    uint64_t* yfull = emptyB + SB;
    uint64_t* agg_bar = yfull + SB;
    uint64_t* carry_bar = agg_bar + NS;
    long long* tileA = reinterpret_cast<long long*>(smem + L::off_ids);
    long long* slot_tile = tileA + SA;
    long long* store_tile = slot_tile + NS;                     // tile id of each phase-B stage
    uint32_t* tmem_base_p = reinterpret_cast<uint32_t*>(smem + L::off_tmem);
    volatile int* stop_pos = reinterpret_cast<volatile int*>(smem + L::off_stop);
    volatile int* draining = reinterpret_cast<volatile int*>(smem + L::off_drain);

    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    const long long ntiles = (long long)prm.ntiles;
    const unsigned long long n = prm.n;
    const bool last_ragged = (n % (unsigned long long)M) != 0;
    static_assert(!REV || STORE, "the anticausal pass always stores");
    // REV: first element of tile j in the arrays (original tile ntiles-1-j)
    auto rev_start = [&](long long j) -> long long { return (ntiles - 1 - j) * (long long)M; };
    // SIG != 0: the signature's tables are compile-time constants (plr_constsig.cuh)
    constexpr Tables<T, A> kTab = const_tables<T, A>(SIG, X, W, G);
    static_assert(SIG == 0 || const_sig_k(SIG) == K, "signature order");
    const Tables<T, A>& tb = SIG != 0 ? kTab : prm.tab;

    if (threadIdx.x == 0) PLR_STAMP(10);
    // launch state from device memory (tickets, epoch); the barrier consumes
    // the loads, so they complete before this CTA's first ticket grab
    const unsigned long long tbase = ld_volatile_u64(prm.ticket + 1);
    const uint32_t epoch = (uint32_t)ld_volatile_u64(prm.ticket + 2) + 1u;
    (void)__syncthreads_or((int)(tbase == 0ull && epoch == 0u));

    if (tid == 0) {
        for (int s = 0; s < SA; s++) { mbar_init(&fullA[s], 1); mbar_init(&emptyA[s], NC); }
        for (int s = 0; s < SB; s++) { mbar_init(&fullB[s], 1); mbar_init(&emptyB[s], 1); mbar_init(&yfull[s], NC); }
        for (int s = 0; s < NS; s++) { mbar_init(&agg_bar[s], 1); mbar_init(&carry_bar[s], 1); }
        *stop_pos = 1 << 30;
        // few units per CTA (small n): every stop-aware wait polls from the start
        *draining = (long long)((ntiles + G - 1) / G) <= 2LL * gridDim.x ? 1 : 0;
        fence_mbar_init();
    }
    if (warp == 0) tmem_alloc(tmem_base_p, TCOLS);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_base_p;
    if (tid == 0) PLR_STAMP(9);

    // phase B is needed for every tile when y is stored, else only for the
    // tiles that hold y_{n-K} .. y_{n-1} (the end state the reduce returns)
    auto covers_tail = [&](long long jj) -> bool {
        return STORE || n < (unsigned long long)K || (unsigned long long)(jj + 1) * M > n - K;
    };
    // TMA load of tile j (with its P-word halo) into stage st, completion on bar
    auto load_tile = [&](T* st, long long j, uint64_t* bar, uint64_t pol) {
        if constexpr (REV) {                                    // the tile, its halo after it (zero beyond n)
            const long long o = rev_start(j);
#pragma unroll
            for (int q = 0; q < kHalo; q++) {
                const unsigned long long i = (unsigned long long)(o + M + q);
                st[M + q] = (q < P && i < n) ? prm.x[i] : T(0);
            }
            mbar_arrive_tx(bar, M * sizeof(T));
            bulk_load(st, prm.x + (size_t)o, M * sizeof(T), bar, pol);
        } else if (j == 0) {
#pragma unroll
            for (int q = 0; q < kHalo; q++)
                st[q] = (q >= kHalo - P && prm.x_hist != nullptr) ? prm.x_hist[q - (kHalo - P)] : T(0);
            mbar_arrive_tx(bar, M * sizeof(T));
            bulk_load(st + kHalo, prm.x, M * sizeof(T), bar, pol);
        } else {
            mbar_arrive_tx(bar, SWL * sizeof(T));
            bulk_load(st, prm.x + (size_t)j * M - kHalo, SWL * sizeof(T), bar, pol);
        }
    };

    // ===================================================== producer warp ===
    if (warp == W) {
        if (lane == 0) {                                            // loader A (HBM)
#ifndef PLR_RR_APOL
#define PLR_RR_APOL 0
#endif
            // x is re-read by phase B from L2: keep it (evict_last) unless overridden
            const uint64_t pol = PLR_RR_APOL == 0 ? policy_evict_last()
                               : PLR_RR_APOL == 1 ? policy_evict_normal() : policy_evict_first();
            long long unit = 0;
            for (int f = 0;; f++) {
                const int s = f % SA;
                if (f >= SA) mbar_wait_poll(&emptyA[s], (uint32_t)(((f / SA) - 1) & 1));
                // one ticket per look-back unit of G consecutive tiles
                if (f % G == 0) unit = (long long)(atomicAdd(prm.ticket, 1ull) - tbase);
                long long j = unit * G + f % G;
                if (j >= ntiles) j = ntiles;
                tileA[s] = j;
                if (j >= ntiles) {
                    // the CTA that ends inside the last (partial) unit still makes
                    // its one failing grab: the host counts nunits + grid tickets
                    const long long rel = f % G != 0 ? (long long)(atomicAdd(prm.ticket, 1ull) - tbase) : unit;
                    launch_state_advance(prm.ticket, rel, (unsigned long long)((ntiles + G - 1) / G) + gridDim.x,
                                         tbase, epoch);
                    *draining = 1;                                  // the stop is SA..NS tiles away
                    mbar_arrive(&fullA[s]);
                    break;
                }
                if (j == (REV ? 0 : ntiles - 1) && last_ragged) { mbar_arrive(&fullA[s]); continue; }   // compute loads it
                load_tile(stA + (size_t)s * SWL, j, &fullA[s], pol);
            }
        } else if (lane == 1) {                                     // loader B (L2)
#ifndef PLR_RR_BPOL
#define PLR_RR_BPOL 0
#endif
            // x is dead after the re-read: evict first (PLR_RR_BPOL=1: normal)
            const uint64_t pol = PLR_RR_BPOL == 0 ? policy_evict_first() : policy_evict_normal();
            for (int f = 0;; f++) {
                const int sb = f % SB;
                // the tile id of position f is known once its phase A is done
                const int slot = f % NS;
                const uint32_t par = (uint32_t)((f / NS) & 1);
                bool stop = false;
                SpinGuard guard;
                while (!mbar_poll(&agg_bar[slot], par)) {
                    guard(4);
                    if (*stop_pos <= f) { stop = true; break; }
                }
                const long long j = stop ? ntiles : slot_tile[slot];
                if (j >= ntiles) break;
                if (f >= SB) mbar_wait_poll(&emptyB[sb], (uint32_t)(((f / SB) - 1) & 1));
                if (j == (REV ? 0 : ntiles - 1) && last_ragged) { mbar_arrive(&fullB[sb]); continue; }
                if (!covers_tail(j)) { mbar_arrive(&fullB[sb]); continue; }   // reduce-only: phase B skipped
                load_tile(stB + (size_t)sb * SWL, j, &fullB[sb], pol);
            }
        } else if (lane == 2) {                                     // storer
            // every stage goes back to loader B as soon as its bulk store has
            // read it (the stage is the next re-load's destination)
            // PLR_RR_STQ bulk stores in flight: the stage of position t goes
            // back once the store of position t + STQ - 1 is issued and every
            // older store has read its stage (one bulk group per position,
            // empty for a ragged or unstored tile)
#ifndef PLR_RR_STQ
#define PLR_RR_STQ 1
#endif
            constexpr int STQ = PLR_RR_STQ;
            static_assert(STQ >= 1 && STQ <= SB && STQ <= 4, "stores in flight");
            const uint64_t pol = policy_evict_first();
            int t = 0;
            for (;; t++) {
                const int sb = t % SB;
                // phase B of position t wrote y into stage sb; the stop is
                // signalled through stop_pos (phase B never runs for it)
                const uint32_t par = (uint32_t)((t / SB) & 1);
                bool stop = false;
                SpinGuard guard;
                while (!mbar_poll(&yfull[sb], par)) {
                    guard(5);
                    if (*stop_pos <= t) { stop = true; break; }
                }
                if (stop) { PLR_STAMP(13); break; }
                const long long jt = store_tile[sb];
                if constexpr (REV) {
                    if (!(jt == 0 && last_ragged))
                        bulk_store(prm.y + (size_t)rev_start(jt), stB + (size_t)sb * SWL, M * sizeof(T), pol);
                } else if (STORE && !(jt == ntiles - 1 && last_ragged)) {
                    bulk_store(prm.y + (size_t)jt * M, stB + (size_t)sb * SWL + kHalo, M * sizeof(T), pol);
                }
                bulk_commit();
                bulk_wait_read<STQ - 1>();                          // stores up to t - STQ + 1 have read their stages
                if (t - (STQ - 1) >= 0) mbar_arrive(&emptyB[(t - (STQ - 1)) % SB]);
            }
            bulk_wait_read<0>();
            for (int r = t - (STQ - 1); r < t; r++)
                if (r >= 0) mbar_arrive(&emptyB[r % SB]);
            bulk_wait_all<0>();
            PLR_STAMP(14);
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
        // Aggregate of pipeline position p (false at the stop).  A parity wait
        // is exact only if the slot's previous phase (position p - NS) has
        // completed: a barrier two phases behind reports the parity of an
        // older phase as done (stale slot_tile / sAt: wrong unit or carry, a
        // hang or silent corruption).  Positions complete in order and this
        // warp saw every position <= known complete, so it first waits for
        // known + NS (exact) until p - NS <= known.
        int known = -1;
        auto wait_pos = [&](int q) -> bool {
            return mbar_wait_or_stop(&agg_bar[q % NS], (uint32_t)((q / NS) & 1), stop_pos, q, draining);
        };
        auto wait_agg = [&](int p) -> bool {
            while (known < p - NS) {
                if (!wait_pos(known + NS)) return false;
                known += NS;
            }
            if (!wait_pos(p)) return false;
            if (p > known) known = p;
            return slot_tile[p % NS] < ntiles;
        };
        for (int u = warp - (W + 1);; u += NL) {
            const long long c_start = clock64();
            A Lp[G][K];
            int cnt = 0;
#pragma unroll
            for (int g = 0; g < G; g++) {
                if (g == cnt && wait_agg(u * G + g)) {
                    const int slot = (u * G + g) % NS;
#pragma unroll
                    for (int q = 0; q < K; q++) Lp[g][q] = sAt[slot * kMaxK + q];
                    if (g > 0) matvec_acc<A, K>(Lp[g], tb.Tm, Lp[g - 1]);
                    cnt++;
                }
            }
            if (cnt == 0) break;
            const long long J = slot_tile[(u * G) % NS] / G;   // unit index
            A Gp[K];                                           // G_{J-1}: carries entering the unit
            if (J == 0) {
#pragma unroll
                for (int q = 0; q < K; q++) Gp[q] = prm.y_hist != nullptr ? A(prm.y_hist[K - 1 - q]) : A(0);
            } else {
                A Ag[K];                                       // unit aggregate: publish at once
#pragma unroll
                for (int q = 0; q < K; q++) Ag[q] = Lp[G - 1][q];
#pragma unroll
                for (int g = 0; g + 1 < G; g++)
                    if (g + 1 == cnt)
#pragma unroll
                        for (int q = 0; q < K; q++) Ag[q] = Lp[g][q];
                publish_status<A, K, DEC>(prm.status, prm.status_mask, J, Ag, tagA, lane);
                lookback_generic<T, A, K, DEC>(prm, tb, J, lane, tagA, tagI, Gp, lbs, c_start, clock64());
            }
#pragma unroll
            for (int g = 0; g < G; g++) {
                if (g < cnt) {
                    const int slot = (u * G + g) % NS;
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
                for (int g = 0; g < cnt; g++) mbar_arrive(&carry_bar[(u * G + g) % NS]);
            if (cnt < G) break;                                // the CTA's last (partial) unit
            A Gi[K];
#pragma unroll
            for (int q = 0; q < K; q++) Gi[q] = Lp[G - 1][q];
            matvec_acc<A, K>(Gi, tb.Tpow[0], Gp);              // G_J = L_{G-1} + T(G m) G_{J-1}
            publish_status<A, K, DEC>(prm.status, prm.status_mask, J, Gi, tagI, lane);
            if (u == 0 && lane == 0) PLR_STAMP(11);
        }
        if (warp == W + 1 && lane == 0) PLR_STAMP(12);
        lbs.flush(prm.stats, lane);
        return;
    }

    // ===================================================== compute warps ===
    A Tl[K * K];                                                // T(X*lane)
#pragma unroll
    for (int e = 0; e < K * K; e++) Tl[e] = prm.lane_T[e * 32 + lane];
    const uint32_t tmem_w = tmem_base + ((uint32_t)(32 * (warp & 3)) << 16) + (uint32_t)((warp >> 2) * CW);

    // this thread's X inputs (+ P halo) from a stage, or from global memory
    // for the ragged last tile
    auto read_x = [&](const T* st, long long j, bool ragged, T (&xv)[X + P]) {
        const long long g0 = j * (long long)M + (long long)tid * X;
        if constexpr (REV) {                                    // positions v: element o + M-1-v
            const int v0 = tid * X - P;
            if (!ragged) {
#pragma unroll
                for (int q = 0; q < X + P; q++) xv[q] = st[M - 1 - (v0 + q)];
            } else {
                const long long o = rev_start(j);
#pragma unroll
                for (int q = 0; q < X + P; q++) {
                    const unsigned long long i = (unsigned long long)(o + M - 1 - (v0 + q));
                    xv[q] = i < n ? prm.x[i] : T(0);
                }
            }
            return;
        }
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
    };
    // a1 FIR map (Eq. 2) of element u
    auto fir = [&](const T (&xv)[X + P], int u) -> T {
        T t = tb.alpha[0] * xv[P + u];
#pragma unroll
        for (int q = 1; q <= P; q++) t = mad(tb.alpha[q], xv[P + u - q], t);
        return t;
    };

    auto phaseA = [&](int it) -> long long {
        const int s = it % SA;
        const int slot = it % NS;
        mbar_wait(&fullA[s], (uint32_t)((it / SA) & 1));
        const long long j = tileA[s];
        if (j >= ntiles) {
            if (tid == 0) { slot_tile[slot] = j; *stop_pos = it; mbar_arrive(&agg_bar[slot]); }
            return j;
        }
        const bool ragged = (j == (REV ? 0 : ntiles - 1)) && last_ragged;
        T xv[X + P];
        read_x(stA + (size_t)s * SWL, j, ragged, xv);
        mbar_arrive(&emptyA[s]);                                // the stage may be refilled
        // a2: chunk end state with zero state (only the last K values matter)
        A hist[K];
#pragma unroll
        for (int r = 0; r < K; r++) hist[r] = A(0);
#pragma unroll
        for (int u = 0; u < X; u++) {
            A acc = cvt<A, T>(fir(xv, u));
#pragma unroll
            for (int r = K; r >= 1; r--)
                if (u - r >= 0) acc = mad(tb.c[r - 1], hist[r - 1], acc);
#pragma unroll
            for (int r = K - 1; r >= 1; r--) hist[r] = hist[r - 1];
            hist[0] = acc;
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
        // park the warp-exclusive carry in TMEM for phase B
        uint32_t w[CW];
#pragma unroll
        for (int q = 0; q < K; q++) {
            const A e = shfl_up(v[q], 1);
            a_to_words<A>(lane == 0 ? A(0) : e, &w[q * AWN]);
        }
        tmem_st_n<CW>(tmem_w + (uint32_t)(slot * WQ * CW), w);
        if (lane == 31) {
#pragma unroll
            for (int q = 0; q < K; q++) wagg[(slot * W + warp) * kMaxK + q] = v[q];
        }
        named_sync(1, NC);
#ifndef PLR_RR_BLK1
#define PLR_RR_BLK1 1
#endif
        // a4: scan of the W warp aggregates with T(32X * 2^s).  One warp per
        // tile (rotating) scans and writes every warp's exclusive prefix; the
        // other warps go straight on (their phase B reads sPw after the carry,
        // ordered by agg_bar -> look-back -> carry_bar).  wagg[slot] / sPw[slot]
        // are rewritten only after the named barrier of tile it+NS, which every
        // warp reaches after its phase B of tile it.
        if (!PLR_RR_BLK1 || warp == it % W) {
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
            if (PLR_RR_BLK1) {
#pragma unroll
                for (int q = 0; q < K; q++) {
                    const A pw = shfl_up(u_[q], 1);
                    if (lane < W) sPw[(slot * W + lane) * K + q] = lane == 0 ? A(0) : pw;
                    if (lane == W - 1) sAt[slot * kMaxK + q] = u_[q];   // tile aggregate
                }
            } else {
#pragma unroll
                for (int q = 0; q < K; q++) {
                    const A pw = shfl_idx(u_[q], (warp + 31) & 31);
                    const A at = shfl_idx(u_[q], W - 1);            // tile aggregate
                    if (lane == 0) sPw[(slot * W + warp) * K + q] = warp == 0 ? A(0) : pw;
                    if (tid == 0) sAt[slot * kMaxK + q] = at;
                }
            }
        }
        tmem_wait_st();
        __syncwarp();
        if (PLR_RR_BLK1 ? (warp == it % W && lane == 0) : tid == 0) { slot_tile[slot] = j; mbar_arrive(&agg_bar[slot]); }
        return j;
    };

    auto phaseB = [&](int it) {
        const int slot = it % NS;
        const int sb = it % SB;
        mbar_wait(&carry_bar[slot], (uint32_t)((it / NS) & 1));
        // the tile id is read after the carry wait: the block-scan warp of
        // phase A wrote it before agg_bar, which the carry is ordered after
        const long long j = slot_tile[slot];
        if (!covers_tail(j)) {
            // reduce-only launch (STORE = false, the sharded schedule's first
            // pass): only the tiles holding the last K outputs (y_tail) need
            // phase B; the others keep the stage protocol and do no work
            mbar_wait(&fullB[sb], (uint32_t)((it / SB) & 1));
            if (tid == 0) store_tile[sb] = j;
            mbar_arrive(&yfull[sb]);
            return;
        }
        const bool ragged = (j == (REV ? 0 : ntiles - 1)) && last_ragged;
        const long long g0 = j * (long long)M + (long long)tid * X;
        uint32_t w[CW];
        tmem_ld_n<CW>(tmem_w + (uint32_t)(slot * WQ * CW), w);
        A Gp[K], Win[K], S[K];
#pragma unroll
        for (int q = 0; q < K; q++) {
            Gp[q] = sG[slot * kMaxK + q];
            Win[q] = sPw[(slot * W + warp) * K + q];
        }
        matvec_acc<A, K>(Win, prm.tab.Twin[warp], Gp);         // warp carry-in (runtime index: parameter tables)
        tmem_wait_ld();
#pragma unroll
        for (int q = 0; q < K; q++) {                           // thread carry-in (y_{-1}, ..., y_{-K})
            A acc = a_from_words<A>(&w[q * AWN]);
#pragma unroll
            for (int r = 0; r < K; r++) acc = mad(Tl[q * K + r], Win[r], acc);
            S[q] = acc;
        }
        // a6: the serial recurrence of P:206-214 over the thread's X elements,
        // seeded with the true incoming state
        T* st = stB + (size_t)sb * SWL;
        mbar_wait(&fullB[sb], (uint32_t)((it / SB) & 1));
        T xv[X + P];
        read_x(st, j, ragged, xv);
        if constexpr (P > 0) named_sync(2, NC);                 // halo reads before y overwrites x
        T yv[X];
#pragma unroll
        for (int u = 0; u < X; u++) {
            A acc = cvt<A, T>(fir(xv, u));
#pragma unroll
            for (int r = K; r >= 1; r--) acc = mad(tb.c[r - 1], S[r - 1], acc);
#pragma unroll
            for (int r = K - 1; r >= 1; r--) S[r] = S[r - 1];
            S[0] = acc;
            yv[u] = cvt<T, A>(acc);
        }
        // a7: y into the stage (TMA store by the storer) or global (ragged)
        if constexpr (REV) {                                    // mirrored: the stage holds original order
            if (!ragged) {
#pragma unroll
                for (int u = 0; u < X; u++) st[M - 1 - (tid * X + u)] = yv[u];
            } else {
#pragma unroll
                for (int u = 0; u < X; u++) {
                    const long long i = rev_start(j) + M - 1 - (tid * X + u);
                    if ((unsigned long long)i < n) prm.y[i] = yv[u];
                }
            }
        } else if (!ragged) {
            if (STORE) {
                T* base = st + kHalo + tid * X;
#pragma unroll
                for (int u = 0; u < X; u++) base[u] = yv[u];
            }
        } else if (STORE) {
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
        if (tid == 0) store_tile[sb] = j;
        fence_proxy_async();
        mbar_arrive(&yfull[sb]);
    };

    // phase B of position nb reads its tile id from slot_tile[nb % NS]:
    // written at the end of phase A(nb), overwritten only by phase A(nb + NS)
#ifndef PLR_RR_RUNTIME_LAG
#define PLR_RR_RUNTIME_LAG 0        // experiment builds only: a runtime lag cost tuple2 0.7 % (r04m)
#endif
#if PLR_RR_RUNTIME_LAG
    // runtime lag in [max(1, G-1), NS-1] (prm.lag = 0: NS-1): phase B of a
    // unit's first tile needs phase A of its last tile, G-1 positions later,
    // and phase B of position nb runs after phase A of nb + lag, so lag >= 1
    // (lag 0 would run phase B of the stop position, which never gets a carry)
    constexpr int kMinLag = G - 1 > 1 ? G - 1 : 1;
    const int Dl = (prm.lag >= kMinLag && prm.lag < D) ? prm.lag : D;
#else
    constexpr int Dl = D;
#endif
    int na = 0, nb = 0;                                         // phases A / B done
    for (; na < Dl; na++) {
        const long long ja = phaseA(na);
        if (ja >= ntiles) break;
    }
    for (bool stop = na < Dl; !stop;) {
        const long long j = phaseA(na);
        phaseB(nb);
        nb++;
        if (j >= ntiles) stop = true; else na++;
    }
    for (; nb < na; nb++) {                                     // drain
        phaseB(nb);
    }
    // loader B, storer and look-back warps beyond the stop see *stop_pos
    tc_fence_before();
    named_sync(1, NC);
    if (tid == 0) PLR_STAMP(15);
    if (warp == 0) {
        tc_fence_after();
        tmem_dealloc(tmem_base, TCOLS);
    }
}

}  // namespace dev
}  // namespace plr
