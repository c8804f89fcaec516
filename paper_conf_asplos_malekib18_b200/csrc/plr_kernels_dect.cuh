// plr_kernels_dect.cuh -- the DECAY kernel with the tile's map outputs
// parked in tensor memory between phase A and phase B.
//
// The in-place DECAY kernel (plr_scan_kernel) keeps each tile in its
// shared-memory stage from the TMA load through phase A, phase B and the TMA
// store, so of its S stages per CTA only ~1.5 are loading at a time; with
// the fp64-accumulation geometry (3 CTAs x 4 x 16 KB stages) that is ~70 KB
// of loads in flight per SM, about what HBM latency needs at full rate, and
// the compute warps wait on the load barrier (profiles/r03d: HP3 at 0.81 of
// a copy, full-barrier waits the top stall).  Here a load stage is released
// as soon as phase A has read it: the map outputs t (X words per thread) and
// the thread's exclusive carry go to TMEM (tcgen05.st, 256 KB per SM unused
// by this bandwidth-bound path) and come back in phase B (tcgen05.ld), which
// writes y into a separate store ring.  Loads, compute and stores are three
// independent rings.
//
// Per tile: a1 load + map, a2 zero-state chunk in A, a3 lane
// scan with T(X 2^s) (DECAY mask, R17), a4 previous warp's aggregate (T(32X)
// = 0) or the warp-aggregate scan, a5 single-hop look-back (T(m) = 0,
// P:731-740), a6 the fp32 recurrence seeded with the thread's true incoming
// state, a7 TMA store.
//
//   warps 0..W-1   compute: phase A of tile i, phase B of tile i-D
//   warp W lane 0  loader: tickets + cp.async.bulk loads
//   warp W lane 1  storer: cp.async.bulk stores from the store ring
//   warp W+1       look-back (a5) of every tile of the CTA, in order
#pragma once
#include "plr_kernels.cuh"
#include "plr_kernels_tmem.cuh"

namespace plr {
namespace dev {

template <typename T, typename A, int K, int X, int W, int SL, int ST, int NT>
struct LayoutDT {
    static constexpr int M = 32 * W * X;
    static constexpr int SWL = M + kHalo;                                       // words per load stage
    static constexpr size_t off_load = 0;
    static constexpr size_t off_store = (size_t)SL * SWL * sizeof(T);           // ST x M
    static constexpr size_t off_Pw = (off_store + (size_t)ST * M * sizeof(T) + 15) & ~(size_t)15;   // [NT][W][kMaxK]
    static constexpr size_t off_At = off_Pw + (size_t)NT * W * kMaxK * sizeof(A);   // [NT][kMaxK]
    static constexpr size_t off_G = off_At + (size_t)NT * kMaxK * sizeof(A);    // [NT][kMaxK]
    static constexpr size_t off_wagg = off_G + (size_t)NT * kMaxK * sizeof(A);  // [NT][W][kMaxK]
    static constexpr size_t off_bar = (off_wagg + (size_t)NT * W * kMaxK * sizeof(A) + 15) & ~(size_t)15;
    // bars: full_L[SL], empty_L[SL], full_T[ST], empty_T[ST], agg[NT], carry[NT]
    static constexpr size_t off_ids = off_bar + (size_t)(2 * SL + 2 * ST + 2 * NT) * 8;
    // ids: tile_of[SL], store_tile[ST], slot_tile[NT]
    static constexpr size_t off_tmem = off_ids + (size_t)(SL + ST + NT) * 8;
    static constexpr size_t off_lbstat = off_tmem + 16;
    static constexpr size_t bytes = off_lbstat + kMaxNL * kLbStatWords * 8;
};

// REV: the anticausal recurrence (plr_kernels_small.cuh): ticket j is
// original tile ntiles-1-j read back to front, the ragged tile first (a
// virtual full tile, zero beyond n), the map's halo after the tile (load
// stage layout [tile][halo]); y goes into the store ring in original order.
template <typename T, typename A, int K, int P, int X, int W, int SL, int ST, int D, int MINB, bool REV = false>
__global__ void __launch_bounds__((W + 2) * 32, MINB)
plr_scan_dect_kernel(const __grid_constant__ ScanParams<T, A> prm) {
    constexpr int NT = D + 1;                                   // parked tiles (phase-B lag D)
    using L = LayoutDT<T, A, K, X, W, SL, ST, NT>;
    constexpr int M = L::M;
    constexpr int SWL = L::SWL;
    constexpr int NC = 32 * W;
    constexpr int WQ = W / 4;                                   // warps sharing a TMEM lane quarter
    constexpr int AWN = AWords<A>::N;
    constexpr int CW = X + K * AWN;                             // TMEM columns per warp per parked tile
    constexpr int LOGW = (W >= 16) ? 4 : (W >= 8) ? 3 : (W >= 4) ? 2 : 0;
    static_assert((1 << LOGW) == W && W >= 4, "W must be a power of two >= 4");
    static_assert(X >= K && X <= kMaxX && (X & 1), "X must be odd and >= K");
    static_assert(P <= kHalo, "halo");
    static_assert(NT * WQ * CW <= 512, "TMEM columns");
    constexpr uint32_t TCOLS = NT * WQ * CW <= 32 ? 32 : NT * WQ * CW <= 64 ? 64 : NT * WQ * CW <= 128 ? 128
                             : NT * WQ * CW <= 256 ? 256 : 512;
    static_assert(SL >= 2 && ST >= 1 && D >= 1, "rings");
    constexpr bool DEC = true;

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

    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    const long long ntiles = (long long)prm.ntiles;
    const unsigned long long n = prm.n;
    const bool last_ragged = (n % (unsigned long long)M) != 0;
    const Tables<T, A>& tb = prm.tab;
    // the tile the compute warps load element by element (REV: the first)
    auto is_ragged = [&](long long j) -> bool { return last_ragged && j == (REV ? 0 : ntiles - 1); };
    // first element of tile j in the arrays (REV: original tile ntiles-1-j)
    auto tile_start = [&](long long j) -> long long { return (REV ? ntiles - 1 - j : j) * (long long)M; };

    const unsigned long long tbase = ld_volatile_u64(prm.ticket + 1);
    const uint32_t epoch = (uint32_t)ld_volatile_u64(prm.ticket + 2) + 1u;
    (void)__syncthreads_or((int)(tbase == 0ull && epoch == 0u));
    if (tid == 0) {
        for (int s = 0; s < SL; s++) { mbar_init(&full_L[s], 1); mbar_init(&empty_L[s], NC); }
        for (int s = 0; s < ST; s++) { mbar_init(&full_T[s], NC); mbar_init(&empty_T[s], 1); }
        for (int s = 0; s < NT; s++) { mbar_init(&agg_bar[s], 1); mbar_init(&carry_bar[s], 1); }
        fence_mbar_init();
    }
    if (warp == 0) tmem_alloc(tmem_base_p, TCOLS);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem_base = *tmem_base_p;

    // ===================================================== producer warp ===
    if (warp == W) {
        const uint64_t pol = policy_evict_first();
        if (lane == 0) {                                            // loader
            for (int f = 0;; f++) {
                const int s = f % SL;
                if (f >= SL) mbar_wait_poll(&empty_L[s], (uint32_t)(((f / SL) - 1) & 1));
                const long long j = (long long)(atomicAdd(prm.ticket, 1ull) - tbase);
                tile_of[s] = j < ntiles ? j : ntiles;
                if (j >= ntiles) {                                  // every CTA makes one failing grab
                    launch_state_advance(prm.ticket, j, (unsigned long long)ntiles + gridDim.x, tbase, epoch);
                    mbar_arrive(&full_L[s]);
                    break;
                }
                if (is_ragged(j)) { mbar_arrive(&full_L[s]); continue; }   // compute loads it
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
            for (int t = 0;; t++) {
                const int sT = t % ST;
                mbar_wait_poll(&full_T[sT], (uint32_t)((t / ST) & 1));
                const long long jt = store_tile[sT];
                if (jt >= ntiles) break;
                if (!is_ragged(jt)) {
                    bulk_store(prm.y + (size_t)tile_start(jt), tstage + (size_t)sT * M, M * sizeof(T), pol);
                    bulk_commit();
                    bulk_wait_read<0>();                            // the store has read the stage
                }
                mbar_arrive(&empty_T[sT]);
            }
            bulk_wait_all<0>();
        }
        return;
    }

    // ===================================================== look-back warp ==
    // a5 for the CTA's tiles in order: the carry entering tile j is tile
    // j-1's inclusive carry, published at the end of j-1's phase A
    // (T(m) = 0: inclusive == aggregate), a single hop
    if (warp == W + 1) {
        const uint32_t tagA = 2u * epoch, tagI = 2u * epoch + 1u;
        for (int it = 0;; it++) {
            const int slot = it % NT;
            mbar_wait(&agg_bar[slot], (uint32_t)((it / NT) & 1));   // tile id + this tile's aggregate
            const long long j = slot_tile[slot];
            if (j >= ntiles) break;
            A Gp[K];
            if (j == 0) {
#pragma unroll
                for (int q = 0; q < K; q++) Gp[q] = prm.y_hist != nullptr ? A(prm.y_hist[K - 1 - q]) : A(0);
            } else {
                A v[K];
                if (lane == 0) {
                    int ns = 64;
                    SpinGuard guard;
                    while (read_status<A, K, DEC>(prm.status, prm.status_mask, j - 1, v, tagA, tagI) != 2) {
                        guard(8);
                        __nanosleep(ns);
                        ns = ns < 256 ? 2 * ns : ns;
                    }
                }
#pragma unroll
                for (int q = 0; q < K; q++) Gp[q] = shfl_idx(lane == 0 ? v[q] : A(0), 0);
            }
            if (lane == 0) {
#pragma unroll
                for (int q = 0; q < K; q++) sG[slot * kMaxK + q] = Gp[q];
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&carry_bar[slot]);
        }
        return;
    }

    // ===================================================== compute warps ===
    A Tl[K * K];                                                // T(X*lane)
#pragma unroll
    for (int e = 0; e < K * K; e++) Tl[e] = prm.lane_T[e * 32 + lane];
    const uint32_t tmem_w = tmem_base + ((uint32_t)(32 * (warp & 3)) << 16) + (uint32_t)((warp >> 2) * CW);

    auto phaseA = [&](int it) -> long long {
        const int s = it % SL;
        const int slot = it % NT;
        mbar_wait(&full_L[s], (uint32_t)((it / SL) & 1));
        const long long j = tile_of[s];
        if (j >= ntiles) {
            if (tid == 0) { slot_tile[slot] = j; mbar_arrive(&agg_bar[slot]); }
            return j;
        }
        const bool ragged = is_ragged(j);
        const long long g0 = j * (long long)M + (long long)tid * X;
        // a1: my X inputs (+ P halo), then the load stage goes back to the loader
        T xv[X + P];
        if (REV) {                                              // positions v: element o + M-1-v
            const int v0 = tid * X - P;
            if (!ragged) {
                const T* st = lstage + (size_t)s * SWL;
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
            const T* base = lstage + (size_t)s * SWL + kHalo + tid * X;
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
        mbar_arrive(&empty_L[s]);
        // a1 map + a2 zero-state chunk (accumulation type); t is parked
        uint32_t w[CW];
        A hist[K];
#pragma unroll
        for (int r = 0; r < K; r++) hist[r] = A(0);
#pragma unroll
        for (int u = 0; u < X; u++) {
            T t = tb.alpha[0] * xv[P + u];
#pragma unroll
            for (int q = 1; q <= P; q++) t = mad(tb.alpha[q], xv[P + u - q], t);
            w[u] = lo_word<T>(t);
            A acc = cvt<A, T>(t);
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
        // a3: lane scan with T(X 2^s), negligible steps skipped (dec_mask, R17)
#pragma unroll
        for (int s2 = 0; s2 < 5; s2++) {
            if (!((prm.dec_mask >> s2) & 1u)) continue;
            A o[K];
#pragma unroll
            for (int q = 0; q < K; q++) o[q] = shfl_up(v[q], 1 << s2);
            if (lane >= (1 << s2)) matvec_acc<A, K>(v, tb.Twarp[s2], o);
        }
#pragma unroll
        for (int q = 0; q < K; q++) {
            const A e = shfl_up(v[q], 1);
            a_to_words<A>(lane == 0 ? A(0) : e, &w[X + q * AWN]);  // warp-exclusive prefix
        }
        tmem_st_n<CW>(tmem_w + (uint32_t)(slot * WQ * CW), w);
        if (lane == 31) {
#pragma unroll
            for (int q = 0; q < K; q++) wagg[(slot * W + warp) * kMaxK + q] = v[q];
        }
        named_sync(1, NC);
        if (!(prm.dec_mask & 32u)) {
            // a4 with T(32X d) == 0, d >= 1: the exclusive warp prefix is the
            // previous warp's aggregate, the tile aggregate the last warp's
            if (lane == 0) {
#pragma unroll
                for (int q = 0; q < K; q++)
                    sPw[(slot * W + warp) * kMaxK + q] = warp == 0 ? A(0) : wagg[(slot * W + warp - 1) * kMaxK + q];
            }
            if (warp == 0) {
                A At[K];
#pragma unroll
                for (int q = 0; q < K; q++) At[q] = wagg[(slot * W + W - 1) * kMaxK + q];
                publish_status<A, K, DEC>(prm.status, prm.status_mask, j, At, 2u * epoch + 1u, lane);
            }
        } else {
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
                At[q] = shfl_idx(u_[q], W - 1);
                if (lane == 0) sPw[(slot * W + warp) * kMaxK + q] = warp == 0 ? A(0) : pw;
            }
            if (warp == 0) publish_status<A, K, DEC>(prm.status, prm.status_mask, j, At, 2u * epoch + 1u, lane);
        }
        tmem_wait_st();
        __syncwarp();
        if (tid == 0) { slot_tile[slot] = j; mbar_arrive(&agg_bar[slot]); }
        return j;
    };

    auto phaseB = [&](int it) {
        const int slot = it % NT;
        const int sT = it % ST;
        mbar_wait(&carry_bar[slot], (uint32_t)((it / NT) & 1));
        const long long j = slot_tile[slot];
        const bool ragged = is_ragged(j);
        const long long g0 = j * (long long)M + (long long)tid * X;
        uint32_t w[CW];
        tmem_ld_n<CW>(tmem_w + (uint32_t)(slot * WQ * CW), w);
        A Gp[K], Win[K];
#pragma unroll
        for (int q = 0; q < K; q++) {
            Gp[q] = sG[slot * kMaxK + q];
            Win[q] = sPw[(slot * W + warp) * kMaxK + q];
        }
        if (!(prm.dec_mask & 32u)) {                           // T(32X w) == 0 for w >= 1
            if (warp == 0) {
#pragma unroll
                for (int q = 0; q < K; q++) Win[q] = Gp[q];
            }
        } else {
            matvec_acc<A, K>(Win, prm.tab.Twin[warp], Gp);
        }
        tmem_wait_ld();
        T Sd[K];                                                // thread carry-in (y_{-1}, ..., y_{-K})
#pragma unroll
        for (int q = 0; q < K; q++) {
            A acc = a_from_words<A>(&w[X + q * AWN]);
#pragma unroll
            for (int r = 0; r < K; r++) acc = mad(Tl[q * K + r], Win[r], acc);
            Sd[q] = cvt<T, A>(acc);
        }
        // a6: the serial recurrence of P:206-214 seeded with the true state
        T yv[X];
#pragma unroll
        for (int u = 0; u < X; u++) {
            T acc = from_word<T>(w[u]);
#pragma unroll
            for (int r = K; r >= 1; r--) acc = mad(tb.cT[r - 1], Sd[r - 1], acc);
#pragma unroll
            for (int r = K - 1; r >= 1; r--) Sd[r] = Sd[r - 1];
            Sd[0] = acc;
            yv[u] = acc;
        }
        // a7: into the store ring (ragged tile: direct stores)
        mbar_wait(&empty_T[sT], (uint32_t)(((it / ST) & 1) ^ 1));
        if (!ragged) {
            T* stt = tstage + (size_t)sT * M;
#pragma unroll
            for (int u = 0; u < X; u++) stt[REV ? M - 1 - (tid * X + u) : tid * X + u] = yv[u];
        } else {
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
    {   // the storer's stop marker (it releases every stage at once: safe to wait)
        const int sT = nb % ST;
        mbar_wait(&empty_T[sT], (uint32_t)(((nb / ST) & 1) ^ 1));
        if (tid == 0) store_tile[sT] = ntiles;
        mbar_arrive(&full_T[sT]);
    }
    tc_fence_before();
    named_sync(1, NC);
    if (warp == 0) {
        tc_fence_after();
        tmem_dealloc(tmem_base, TCOLS);
    }
}

}  // namespace dev
}  // namespace plr
