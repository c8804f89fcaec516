// plr_kernels.cuh -- sm_100a kernels of the PLR hot path.
//
// One persistent, warp-specialised, single-pass kernel evaluates Eq. (1)
// (P:76-78).  Per tile of m = 32*W*X elements:
//   a1 load + fused FIR map (Eq. (2))
//   a2 per-thread sequential chunk of X elements with zero state
//      (the serial loop of P:206-214; work-efficient replacement of the
//      element-level doubling of Phase 1)
//   a3 warp carry propagation: Kogge-Stone over the 32 lanes with
//      T(X*2^s) and shuffles
//   a4 block propagation of the warp aggregates through shared memory
//
//   a5 grid: decoupled look-back of the k carries with epoch-tagged status
//      words (Phase 2; carry precomputation P:527-556; chunk
//      ticket P:651-653; publish / wait P:668-683)
//   a6 carry-in distribution + correction y_u = l_u + sum_r S_r h^(r)_u
//
//   a7 store
// Roles: warp W (producer) takes tickets and moves whole tiles with TMA bulk
// copies (cp.async.bulk + mbarrier complete_tx) into an S-stage shared-memory
// ring and back out with TMA bulk stores; warps W+1..W+NL (look-back) run a5
// for the CTA's tiles, taking turns; warps 0..W-1 (compute) run phase A
// (a1-a4) of tile i+D before phase B (a6-a7) of tile i, so the look-back
// latency of a tile overlaps D tiles of compute.
#pragma once
#include <cstdio>
#include <cuda_runtime.h>
#include <cstdint>

#include "plr_internal.h"

namespace plr {
namespace dev {

// ------------------------------------------------------ launch state -------
// ticket[0] = ticket counter, ticket[1] = this launch's ticket base,
// ticket[2] = the previous launch's epoch.  Every CTA makes exactly one
// failing grab, so a launch takes total = units + grid tickets; the grab with
// relative index total - 1 is the last one and advances the state for the
// next launch on the stream.  Nothing of a launch lives on the host, so a
// launch captured in a CUDA graph replays correctly.
__device__ __forceinline__ unsigned long long ld_volatile_u64(const unsigned long long* p) {
    return *reinterpret_cast<const volatile unsigned long long*>(p);
}
__device__ __forceinline__ void launch_state_advance(unsigned long long* tk, long long rel, unsigned long long total,
                                                     unsigned long long base, uint32_t epoch) {
    if ((unsigned long long)rel == total - 1) {
        reinterpret_cast<volatile unsigned long long*>(tk)[1] = base + total;
        reinterpret_cast<volatile unsigned long long*>(tk)[2] = epoch;
    }
}

// PLR_TRACE builds (experiment variants only): globaltimer stamps of CTA 0's
// single-tile critical path into stats words 9..15 (plan made with PLR_STATS=1)
#ifdef PLR_TRACE
#define PLR_STAMP(i) do { if (prm.stats != nullptr && blockIdx.x == 0) { unsigned long long t_; \
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_)); prm.stats[i] = t_; } } while (0)
#else
#define PLR_STAMP(i) do { } while (0)
#endif

// ------------------------------------------------------- deadlock trap ----
// PLR_DEADLOCK_TRAP builds (tests / stress variants, never the product
// library): every spin / poll loop of the kernels carries a SpinGuard that
// reads %globaltimer and, after PLR_DEADLOCK_NS of waiting at one site,
// prints the site, block and thread and executes trap -- a lost arrival or
// an unpublished status record becomes a launch error with a location
// instead of a hung GPU.  Sites: 1 mbar_wait, 2 mbar_wait_poll, 3
// mbar_wait_or_stop, 4 re-read loader B, 5 re-read storer, 6 generic
// look-back poll, 7 DECAY single-hop poll (plr_scan_kernel), 8 (dect
// kernel), 9 (small-n kernel).  Product builds: an empty struct, no code.
#ifndef PLR_DEADLOCK_NS
#define PLR_DEADLOCK_NS 2000000000ull
#endif

struct SpinGuard {
#ifdef PLR_DEADLOCK_TRAP
    unsigned long long t0 = 0;
    __device__ __forceinline__ void operator()(int site) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        if (t0 == 0) {
            t0 = t;
        } else if (t - t0 > (unsigned long long)PLR_DEADLOCK_NS) {
            printf("plr deadlock trap: site %d block %d thread %d waited %llu ns\n", site, (int)blockIdx.x,
                   (int)threadIdx.x, t - t0);
            __trap();
        }
    }
#else
    __device__ __forceinline__ void operator()(int) {}
#endif
};

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
// try_wait with a suspend-time hint: the waiting warp sleeps in hardware
// until the phase completes (or the hint, in ns, expires) instead of spinning
// through issue slots the working warps of its SM sub-partition need
__device__ __forceinline__ bool mbar_try_wait_sleep(uint64_t* bar, uint32_t parity, uint32_t hint_ns) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2, %3;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity), "r"(hint_ns) : "memory");
    return ok != 0;
}
#ifndef PLR_WAIT_HINT_NS
#define PLR_WAIT_HINT_NS 0x989680u        // 10 ms: wake on completion
#endif
#ifndef PLR_POLL_HINT_NS
#define PLR_POLL_HINT_NS 0u               // waits that also poll a stop flag (a hint measured slower)
#endif
// Stop-aware waits (loader B, storer, look-back warps): a try_wait whose
// phase does not complete suspends the warp for ~4 us whatever the hint
// (0, 200, 2000 ns measured alike, profiles/r02p_small_n_trace.md), so a
// stop set meanwhile was seen microseconds late -- the tail of every launch.
// Poll with the non-blocking test_wait and a short sleep instead.
#ifndef PLR_POLL_SLEEP_NS
#define PLR_POLL_SLEEP_NS 64
#endif
__device__ __forceinline__ bool mbar_test(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.test_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
    return ok != 0;
}
__device__ __forceinline__ bool mbar_poll(uint64_t* bar, uint32_t parity) {
    const bool ok = mbar_test(bar, parity);
    if (!ok && PLR_POLL_SLEEP_NS > 0) __nanosleep(PLR_POLL_SLEEP_NS);
    return ok;
}
// Stop-aware wait of a whole warp on a phase that may never complete (a
// pipeline position at or beyond the launch's stop): true when the phase
// completed, false once the stop position is known to be <= pos.  While
// tickets remain (*draining == 0) the warp suspends in try_wait and takes no
// issue slots from the compute warps; once the loader saw the tickets run
// out it polls (test_wait + a short sleep) so the stop is noticed at once.
// Only for warps whose lanes all wait together (the look-back warps): a
// suspended lane could hold back a diverged sibling lane of the producer
// warp that the awaited arrival depends on (those lanes use mbar_poll).
__device__ __forceinline__ bool mbar_wait_or_stop(uint64_t* bar, uint32_t parity, const volatile int* stop_pos,
                                                  int pos, const volatile int* draining) {
    SpinGuard guard;
    for (;;) {
        guard(3);
        if (mbar_test(bar, parity)) return true;
        if (*stop_pos <= pos) return false;
        if (*draining) {
            if (PLR_POLL_SLEEP_NS > 0) __nanosleep(PLR_POLL_SLEEP_NS);
        } else if (mbar_try_wait_sleep(bar, parity, PLR_WAIT_HINT_NS)) {
            return true;
        }
    }
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    SpinGuard guard;
    while (!mbar_try_wait_sleep(bar, parity, PLR_WAIT_HINT_NS)) guard(1);
}
// wait without a suspend hint, for lanes of a warp whose lanes play
// different roles (loader / storer lanes of the producer warp): a lane
// suspended for long in try_wait can hold back a diverged sibling lane that
// the awaited arrival depends on (loader B waits on the storer's emptyB)
__device__ __forceinline__ void mbar_wait_poll(uint64_t* bar, uint32_t parity) {
    SpinGuard guard;
    while (!mbar_try_wait(bar, parity)) guard(2);
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
__device__ __forceinline__ double mad(double a, double b, double c) { return __fma_rn(a, b, c); }


// conversions between the data type and the accumulation type.  fp32 values
// here come out of FTZ arithmetic (already flushed), so the plain cvt is used:
// the compiler's default under -ftz adds a flushing FMUL / DSETP+FSEL per
// conversion, one per element on the fp64-accumulation path.
template <typename To, typename From>
__device__ __forceinline__ To cvt(From v) { return To(v); }
template <>
__device__ __forceinline__ double cvt<double, float>(float v) {
    double d;
    asm("cvt.f64.f32 %0, %1;" : "=d"(d) : "f"(v));
    return d;
}
template <>
__device__ __forceinline__ float cvt<float, double>(double v) {
    float f;
    asm("cvt.rn.f32.f64 %0, %1;" : "=f"(f) : "d"(v));
    return f;
}

// v[q] += sum_r Tm[q][r] * o[r]
template <typename A, int K>
__device__ __forceinline__ void matvec_acc(A (&v)[K], const A* Tm, const A (&o)[K]) {
    A r_[K];
#pragma unroll
    for (int q = 0; q < K; q++) {
        A acc = v[q];
#pragma unroll
        for (int r = 0; r < K; r++) acc = mad(Tm[q * kMaxK + r], o[r], acc);
        r_[q] = acc;
    }
#pragma unroll
    for (int q = 0; q < K; q++) v[q] = r_[q];
}

template <typename A>
__device__ __forceinline__ A shfl_up(A v, int d) { return __shfl_up_sync(0xffffffffu, v, d); }
template <typename A>
__device__ __forceinline__ A shfl_down(A v, int d) { return __shfl_down_sync(0xffffffffu, v, d); }
template <typename A>
__device__ __forceinline__ A shfl_idx(A v, int l) { return __shfl_sync(0xffffffffu, v, l); }

// ------------------------------------------------------ status words -------
// Tile status: 2*kStatusWords 64-bit words per tile.  32-bit carries: word q
// = {tag:32 | value:32} (one single-copy-atomic store each, so a reader
// validates every component by its own tag).  fp64 carries: two words per
// component, {tag | fp32 hi} and {tag | fp32 lo} with hi = fl(v),
// lo = fl(v - hi) (a double-float split, ~48 significant bits).
template <typename A> struct StatusIO;

template <> struct StatusIO<uint32_t> {
    static constexpr int kWords = 1;
    __device__ static void pack(uint32_t v, uint32_t tag, unsigned long long* w) {
        w[0] = ((unsigned long long)tag << 32) | v;
    }
    __device__ static bool unpack(const unsigned long long* w, uint32_t tag, uint32_t& v) {
        v = (uint32_t)w[0];
        return (uint32_t)(w[0] >> 32) == tag;
    }
};
template <> struct StatusIO<float> {
    static constexpr int kWords = 1;
    __device__ static void pack(float v, uint32_t tag, unsigned long long* w) {
        w[0] = ((unsigned long long)tag << 32) | __float_as_uint(v);
    }
    __device__ static bool unpack(const unsigned long long* w, uint32_t tag, float& v) {
        v = __uint_as_float((uint32_t)w[0]);
        return (uint32_t)(w[0] >> 32) == tag;
    }
};
template <> struct StatusIO<double> {
    static constexpr int kWords = 2;   // double-float split: hi = fl(v), lo = fl(v - hi)
    __device__ static void pack(double v, uint32_t tag, unsigned long long* w) {
        const float hi = __double2float_rn(v);
        const float lo = __double2float_rn(v - (double)hi);
        w[0] = ((unsigned long long)tag << 32) | __float_as_uint(hi);
        w[1] = ((unsigned long long)tag << 32) | __float_as_uint(lo);
    }
    __device__ static bool unpack(const unsigned long long* w, uint32_t tag, double& v) {
        v = (double)__uint_as_float((uint32_t)w[0]) + (double)__uint_as_float((uint32_t)w[1]);
        return (uint32_t)(w[0] >> 32) == tag && (uint32_t)(w[1] >> 32) == tag;
    }
};

// Status records are packed at a power-of-two stride of NW 64-bit words per
// tile (NW = K words for 32-bit carries, 2K for fp64), so a window of
// consecutive tiles is one contiguous block and a warp-wide load of 32
// consecutive tiles coalesces into a few L2 requests.
// Status records: NW 64-bit words at a power-of-two stride, placed at a
// scattered slot (j * 0x9E3779B1) mod 2^c (odd multiplier: a bijection on the
// 2^c slots), so the hundreds of records that concurrent look-backs poll are
// spread over all L2 slices instead of hammering a few lines.
#ifndef PLR_STATUS_MIN_STRIDE
#define PLR_STATUS_MIN_STRIDE 4      // words: one 32-byte sector per record at least
#endif
template <typename A, int K, bool DEC>
struct StatusLayout {
    static constexpr int NW = K * StatusIO<A>::kWords;
    static constexpr int P2 = NW <= 1 ? 1 : NW <= 2 ? 2 : NW <= 4 ? 4 : 8;
    static constexpr int STRIDE = P2 > PLR_STATUS_MIN_STRIDE ? P2 : PLR_STATUS_MIN_STRIDE;
    static_assert(STRIDE * 8 <= kStatusMaxBytes, "status record stride");
};
__device__ __forceinline__ size_t status_slot(long long j, uint32_t mask) {
#ifdef PLR_STATUS_LINEAR
    (void)mask;
    return (size_t)j;
#else
    return (size_t)(((uint32_t)j * 0x9E3779B1u) & mask);
#endif
}

__device__ __forceinline__ void ld_relaxed_v2(const unsigned long long* p, unsigned long long& a,
                                              unsigned long long& b) {
    asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
}

// publish carry vector `val` of tile j with `tag`; lanes 0..NW-1 of the
// calling warp each store one 64-bit word (single-copy atomic per word)
template <typename A, int K, bool DEC>
__device__ __forceinline__ void publish_status(unsigned long long* status, uint32_t mask, long long j,
                                               const A (&val)[K], uint32_t tag, int lane) {
    using SIO = StatusIO<A>;
    using SL = StatusLayout<A, K, DEC>;
    unsigned long long* stj = status + status_slot(j, mask) * SL::STRIDE;
    unsigned long long w[SL::NW];
#pragma unroll
    for (int q = 0; q < K; q++) SIO::pack(val[q], tag, &w[q * SIO::kWords]);
#pragma unroll
    for (int e = 0; e < SL::NW; e++) if (lane == e) st_relaxed(stj + e, w[e]);
}

// read tile jj's K components: 2 inclusive, 1 aggregate, 0 not ready.  Every
// word carries its own tag, so 16-byte vector loads (two relaxed 64-bit
// accesses) are as safe as scalar ones.
template <typename A, int K, bool DEC>
__device__ __forceinline__ int read_status(const unsigned long long* status, uint32_t mask, long long jj,
                                           A (&val)[K], uint32_t tagA, uint32_t tagI) {
    using SIO = StatusIO<A>;
    using SL = StatusLayout<A, K, DEC>;
    constexpr int NW = SL::NW;
    const unsigned long long* sp = status + status_slot(jj, mask) * SL::STRIDE;
    unsigned long long w[NW + 1];
#pragma unroll
    for (int e = 0; e + 1 < NW + (NW & 1); e += 2) {
        if (e + 1 < NW) ld_relaxed_v2(sp + e, w[e], w[e + 1]);
        else w[e] = ld_relaxed(sp + e);
    }
    bool allI = true, allA = true;
#pragma unroll
    for (int q = 0; q < K; q++) {
        const bool i1 = SIO::unpack(&w[q * SIO::kWords], tagI, val[q]);
        const bool a1 = SIO::unpack(&w[q * SIO::kWords], tagA, val[q]);
        allI = allI && i1;
        allA = allA && a1;
    }
    return allI ? 2 : (allA ? 1 : 0);
}

// Split form of read_status for windows: issue every load of the window
// first, classify afterwards, so the loads of all tiles are in flight
// together (one L2 round trip per window, not one per tile).
template <typename A, int K, bool DEC>
__device__ __forceinline__ void load_status_raw(const unsigned long long* status, uint32_t mask, long long jj,
                                                unsigned long long (&w)[StatusLayout<A, K, DEC>::NW]) {
    using SL = StatusLayout<A, K, DEC>;
    constexpr int NW = SL::NW;
    const unsigned long long* sp = status + status_slot(jj, mask) * SL::STRIDE;
#pragma unroll
    for (int e = 0; e < NW; e += 2) {
        if (e + 1 < NW) ld_relaxed_v2(sp + e, w[e], w[e + 1]);
        else w[e] = ld_relaxed(sp + e);
    }
}
template <typename A, int K, bool DEC>
__device__ __forceinline__ int classify_status(const unsigned long long (&w)[StatusLayout<A, K, DEC>::NW],
                                               A (&val)[K], uint32_t tagA, uint32_t tagI) {
    using SIO = StatusIO<A>;
    bool allI = true, allA = true;
#pragma unroll
    for (int q = 0; q < K; q++) {
        const bool i1 = SIO::unpack(&w[q * SIO::kWords], tagI, val[q]);
        const bool a1 = SIO::unpack(&w[q * SIO::kWords], tagA, val[q]);
        allI = allI && i1;
        allA = allA && a1;
    }
    return allI ? 2 : (allA ? 1 : 0);
}


// look-back debug counters (PLR_STATS=1): summed per warp in registers,
// flushed with one atomic per counter when the warp exits
// in shared memory (kLbStatWords per look-back warp), flushed with one atomic
// per counter when the warp exits; registers stay free for the look-back
constexpr int kLbStatWords = 9;
constexpr int kMaxNL = 4;                              // look-back warps per CTA
struct LbStats {
    unsigned long long* v;                             // this warp's shared counters
    __device__ void init(int lane) const {
        if (lane == 0)
            for (int i = 0; i < kLbStatWords; i++) v[i] = 0;
    }
    __device__ void flush(unsigned long long* dst, int lane) const {
        if (dst != nullptr && lane == 0)
            for (int i = 0; i < kLbStatWords; i++) atomicAdd(&dst[i], v[i]);
    }
};

// Generic look-back: fold the tiles j-1, j-2, ...
// nearest first, G_{j-1} = sum_d T(d m) v_{j-1-d}, v = aggregate for "P"
// tiles and the inclusive carry of the first "I" tile.  Each poll reads a
// lane-interleaved window (all loads in flight together), folds its ready
// prefix (up to the first not-ready or first inclusive tile) and never
// re-reads folded tiles.  Called by one full warp.  LOGU: the records are
// those of units of 2^LOGU table units (T(2^LOGU U 2^s) = Tpow[s + LOGU]; the
// small-n cluster kernel's cluster records), valid while a look-back folds
// fewer than 2^(9 - LOGU) records.
template <typename T, typename A, int K, bool DEC, int LOGU = 0>
__device__ __forceinline__ void lookback_generic(const ScanParams<T, A>& prm, const Tables<T, A>& tb, long long j,
                                                 int lane, uint32_t tagA, uint32_t tagI, A (&Gp)[K],
                                                 const LbStats& lbs, long long c_start = 0, long long c_agg = 0,
                                                 int ns_cap = 512, bool wide_first = false) {
    long long c_wait = 0;
    // tiles per lane of a full window: 8 for small records, 4 when a record
    // has more than 2 words (keeps the window's registers in check)
#ifndef PLR_LB_WIDE_NW
#define PLR_LB_WIDE_NW 2
#endif
    constexpr int kT = StatusLayout<A, K, DEC>::NW <= PLR_LB_WIDE_NW ? kTPL : kTPL / 2;
    constexpr int kLogT = kT == 8 ? 3 : 2;
    A acc[K];
    A Tacc[K * kMaxK];
#pragma unroll
    for (int q = 0; q < K; q++) {
        acc[q] = A(0);
#pragma unroll
        for (int r = 0; r < kMaxK; r++) Tacc[q * kMaxK + r] = (q == r) ? A(1) : A(0);
    }
    long long o = 0;                   // distance of the first unfolded tile from j-1
#ifndef PLR_LB_LTPL0
#define PLR_LB_LTPL0 1
#endif
    int ltpl = wide_first ? kLogT : (PLR_LB_LTPL0 < kLogT ? PLR_LB_LTPL0 : kLogT);   // log2 tiles per lane, first window
#ifndef PLR_LB_NS0
#define PLR_LB_NS0 32
#endif
    int ns = PLR_LB_NS0;
    unsigned long long n_win = 0, n_wait = 0;
    SpinGuard guard;
    long long c_load = 0, c_fold = 0;
    for (;;) {
        n_win++;
        const long long cl0 = clock64();
        const int tpl = 1 << ltpl;
        // lane-interleaved window: distance d = o + 32 t + lane, t < tpl,
        // so every warp-wide load reads 32 consecutive tiles
        using SLw = StatusLayout<A, K, DEC>;
        unsigned long long raw[kT][SLw::NW];
#pragma unroll
        for (int t = 0; t < kT; t++) {             // all loads in flight together
            const long long jj = j - 1 - (o + 32LL * t + lane);
            if (t < tpl && jj >= 0) load_status_raw<A, K, DEC>(prm.status, prm.status_mask, jj, raw[t]);
        }
        A v[kT][K];
        int st[kT];
#pragma unroll
        for (int t = 0; t < kT; t++) {
            st[t] = 2;
#pragma unroll
            for (int q = 0; q < K; q++) v[t][q] = A(0);
            const long long jj = j - 1 - (o + 32LL * t + lane);
            if (t < tpl && jj >= 0) st[t] = classify_status<A, K, DEC>(raw[t], v[t], tagA, tagI);
        }
        int di = 1 << 30, dn = 1 << 30;              // lane's nearest inclusive / not-ready
#pragma unroll
        for (int t = kT - 1; t >= 0; t--) {
            if (t < tpl && st[t] == 2) di = 32 * t + lane;
            if (t < tpl && st[t] == 0) dn = 32 * t + lane;
        }
        const int dI = __reduce_min_sync(0xffffffffu, (unsigned)di);
        const int dN = __reduce_min_sync(0xffffffffu, (unsigned)dn);
        const bool found = dI < dN;
        const int e = found ? dI + 1 : (dN < (1 << 30) ? dN : 32 * tpl);   // tiles to fold now
        const long long cl1 = clock64();
        c_load += cl1 - cl0;
        if (e > 0) {
            // per-lane Horner over t (stride 32 tiles), then a tree over lanes
            A r[K];
#pragma unroll
            for (int q = 0; q < K; q++) r[q] = A(0);
#pragma unroll
            for (int t = kT - 1; t >= 0; t--) {
                if (t < tpl && 32 * t + lane < e) {
                    A nr[K];
#pragma unroll
                    for (int q = 0; q < K; q++) nr[q] = v[t][q];
                    matvec_acc<A, K>(nr, tb.Tpow[5 + LOGU], r);    // T(32 m)
#pragma unroll
                    for (int q = 0; q < K; q++) r[q] = nr[q];
                }
            }
            // R = sum_l T(l m) r_l, T(m 2^s) = Tpow[s]
#pragma unroll
            for (int s2 = 0; s2 < 5; s2++) {
                A o2[K];
#pragma unroll
                for (int q = 0; q < K; q++) o2[q] = shfl_down(r[q], 1 << s2);
                matvec_acc<A, K>(r, tb.Tpow[s2 + LOGU], o2);
            }
            A R[K];
#pragma unroll
            for (int q = 0; q < K; q++) R[q] = shfl_idx(r[q], 0);
            matvec_acc<A, K>(acc, Tacc, R);
            c_fold += clock64() - cl1;
            if (found) break;
            // skip the folded tiles: Tacc *= T(e m) (binary powers; unrolled so
            // compile-time tables fold)
#pragma unroll
            for (int s2 = 0; s2 + LOGU < 9; s2++) {
                if (!((e >> s2) & 1)) continue;
                A nt[K * kMaxK];
#pragma unroll
                for (int q = 0; q < K; q++)
#pragma unroll
                    for (int c2 = 0; c2 < K; c2++) {
                        A a2 = A(0);
#pragma unroll
                        for (int t = 0; t < K; t++) a2 = mad(Tacc[q * kMaxK + t], tb.Tpow[s2 + LOGU][t * kMaxK + c2], a2);
                        nt[q * kMaxK + c2] = a2;
                    }
#pragma unroll
                for (int q = 0; q < K; q++)
#pragma unroll
                    for (int c2 = 0; c2 < K; c2++) Tacc[q * kMaxK + c2] = nt[q * kMaxK + c2];
            }
            o += e;
            ns = PLR_LB_NS0;
            if (dN >= (1 << 30)) ltpl = kLogT;         // nothing pending: widen to the full window
        } else {
            n_wait++;                                  // nearest tile not ready yet
            guard(6);
            const long long cw = clock64();
            __nanosleep(ns);
            c_wait += clock64() - cw;
            ns = ns < ns_cap ? 2 * ns : ns;
        }
    }
    if (prm.stats != nullptr && lane == 0) {           // debug counters (shared, per warp)
        lbs.v[0] += 1;                                 // look-backs
        lbs.v[1] += n_win;                             // window polls
        lbs.v[2] += n_wait;                            // polls that folded nothing
        lbs.v[3] += (unsigned long long)(o + 1);       // depth folded (approx.)
        lbs.v[4] += (unsigned long long)(c_agg - c_start);    // cycles waiting for the own aggregate
        lbs.v[5] += (unsigned long long)(clock64() - c_agg);  // cycles looking back
        lbs.v[6] += (unsigned long long)c_wait;               // of which sleeping
        lbs.v[7] += (unsigned long long)c_load;               // loading + classifying windows
        lbs.v[8] += (unsigned long long)c_fold;               // folding
    }
#pragma unroll
    for (int q = 0; q < K; q++) Gp[q] = acc[q];
}

// ------------------------------------------------------ shared memory ------
template <typename T, typename A, int K, int X, int W, int S, int D>
struct Layout {
    static constexpr int NS = D + 1;                            // pipeline slots (tiles between A and B)
    static constexpr int M = 32 * W * X;
    static constexpr int NC = 32 * W;
    static constexpr int SW = M + kHalo;                        // words per stage
    static constexpr size_t off_stage = 0;
    static constexpr size_t off_E = (size_t)S * SW * sizeof(T);                       // [NS][K][NC] A
    static constexpr size_t off_Pw = off_E + NS * (size_t)K * NC * sizeof(A);         // [NS][W][K] A
    static constexpr size_t off_At = off_Pw + NS * (size_t)W * K * sizeof(A);         // [NS][K] A
    static constexpr size_t off_G = off_At + NS * (size_t)kMaxK * sizeof(A);          // [NS][K] A
    static constexpr size_t off_wagg = off_G + NS * (size_t)kMaxK * sizeof(A);        // [NS][W][K] A
    static constexpr size_t off_bar = (off_wagg + NS * (size_t)W * kMaxK * sizeof(A) + 15) & ~(size_t)15;
    // bars: full[S], done[S], agg[NS], carry[NS]
    static constexpr size_t off_tile = off_bar + (2 * S + 2 * NS) * 8;               // tile_of[S]
    static constexpr size_t off_aggtile = off_tile + S * 8;                           // agg_tile[NS]
    static constexpr size_t off_lbstat = off_aggtile + NS * 8;                        // [kMaxNL][kLbStatWords]
    static constexpr size_t bytes = off_lbstat + kMaxNL * kLbStatWords * 8;
};

// ------------------------------------------------------ the scan kernel ----
// SEED: phase B evaluates the serial recurrence of P:206-214 over the
// thread's X elements seeded with its true incoming state (the alternative
// of SURVEY §8(a) a6) instead of correcting parked chunk values with the
// factors h^(r)_u; the stage then holds the map outputs t (Eq. 2) between
// the phases, or x itself when p = 0 (t = a0 x is recomputed).
// REV: the anticausal recurrence (the causal one over the reversed
// sequence; see plr_kernels_small.cuh): ticket j is original tile
// ntiles-1-j read back to front, the ragged tile first (a virtual full tile,
// zero beyond n), the map's halo after the tile; stage layout [tile][halo].
template <typename T, typename A, int K, int P, int X, int W, int S, int D, int NL, bool DEC, bool STORE,
          int MINB, bool SEED = false, bool REV = false>
__global__ void __launch_bounds__((W + 1 + NL) * 32, MINB)
plr_scan_kernel(const __grid_constant__ ScanParams<T, A> prm) {
    using L = Layout<T, A, K, X, W, S, D>;
    constexpr int NS = L::NS;
    constexpr int M = L::M;
    constexpr int SW = L::SW;
    constexpr int NC = L::NC;
    constexpr int LOGW = (W >= 16) ? 4 : (W >= 8) ? 3 : (W >= 4) ? 2 : (W >= 2) ? 1 : 0;
    static_assert((1 << LOGW) == W, "W must be a power of two");
    static_assert(X >= K && X <= kMaxX && (X & 1), "X must be odd and >= K");
    static_assert(P <= kHalo, "halo");
    using SIO = StatusIO<A>;
    static_assert(K * SIO::kWords <= 2 * kStatusWords, "status words");
    static_assert(D >= 1 && S >= D + 2, "phase B of tile i runs after phase A of tile i+D: needs S >= D+2 stages");
    static_assert(NL >= 1 && NL <= S, "look-back warps");

    extern __shared__ __align__(128) unsigned char smem[];
    T* stages = reinterpret_cast<T*>(smem + L::off_stage);
    A* sE = reinterpret_cast<A*>(smem + L::off_E);
    A* sPw = reinterpret_cast<A*>(smem + L::off_Pw);
    A* sAt = reinterpret_cast<A*>(smem + L::off_At);
    A* sG = reinterpret_cast<A*>(smem + L::off_G);
    A* wagg = reinterpret_cast<A*>(smem + L::off_wagg);
    uint64_t* full_bar = reinterpret_cast<uint64_t*>(smem + L::off_bar);
    uint64_t* done_bar = full_bar + S;
    uint64_t* agg_bar = done_bar + S;
    uint64_t* carry_bar = agg_bar + NS;
    long long* tile_of = reinterpret_cast<long long*>(smem + L::off_tile);
    long long* agg_tile = reinterpret_cast<long long*>(smem + L::off_aggtile);

    const int tid = threadIdx.x;
    const int warp = tid >> 5, lane = tid & 31;
    const long long ntiles = (long long)prm.ntiles;
    const unsigned long long n = prm.n;
    const bool last_ragged = (n % (unsigned long long)M) != 0;
    const Tables<T, A>& tb = prm.tab;
    static_assert(!REV || STORE, "the anticausal pass always stores");
    // the tile the compute warps load element by element (REV: the first)
    auto is_ragged = [&](long long j) -> bool { return last_ragged && j == (REV ? 0 : ntiles - 1); };
    // first element of tile j in the arrays (REV: original tile ntiles-1-j)
    auto tile_start = [&](long long j) -> long long { return (REV ? ntiles - 1 - j : j) * (long long)M; };
    // the tile's M words inside a stage ([halo][tile], REV: [tile][halo])
    auto tile_words = [&](T* st) -> T* { return REV ? st : st + kHalo; };

    // launch state from device memory (tickets, epoch); the barrier consumes
    // the loads, so they complete before this CTA's first ticket grab
    const unsigned long long tbase = ld_volatile_u64(prm.ticket + 1);
    const uint32_t epoch = (uint32_t)ld_volatile_u64(prm.ticket + 2) + 1u;
    (void)__syncthreads_or((int)(tbase == 0ull && epoch == 0u));

    if (tid == 0) {
        for (int s = 0; s < S; s++) { mbar_init(&full_bar[s], 1); mbar_init(&done_bar[s], NC); }
        for (int s = 0; s < NS; s++) { mbar_init(&agg_bar[s], 1); mbar_init(&carry_bar[s], 1); }
        fence_mbar_init();
    }
    __syncthreads();

    // ===================================================== producer warp ===
    if (warp == W) {
        if (lane != 0) return;
        const uint64_t pol = policy_evict_first();
        int fills = 0;                                  // pipeline index of the next fill
        int stop_at = 1 << 30;                          // pipeline index of the first stop marker
        auto fill = [&]() {
            const int idx = fills++;
            const int s = idx % S;
            if (idx > stop_at) {                        // extra stop markers for the look-back warps
                tile_of[s] = ntiles;
                mbar_arrive(&full_bar[s]);
                return;
            }
            const long long j = (long long)(atomicAdd(prm.ticket, 1ull) - tbase);
            tile_of[s] = j;
            if (j >= ntiles) {
                launch_state_advance(prm.ticket, j, (unsigned long long)ntiles + gridDim.x, tbase, epoch);
                stop_at = idx; mbar_arrive(&full_bar[s]); return;
            }
            if (is_ragged(j)) { mbar_arrive(&full_bar[s]); return; }   // compute loads it
            T* st = stages + (size_t)s * SW;
            if (REV) {                                  // the tile, its halo after it (zero beyond n)
                const long long o = tile_start(j);
#pragma unroll
                for (int q = 0; q < kHalo; q++) {
                    const unsigned long long i = (unsigned long long)(o + M + q);
                    st[M + q] = (q < P && i < n) ? prm.x[i] : T(0);
                }
                mbar_arrive_tx(&full_bar[s], M * sizeof(T));
                bulk_load(st, prm.x + (size_t)o, M * sizeof(T), &full_bar[s], pol);
            } else if (j == 0) {
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
        // every look-back warp must see a stop marker: NL of them after the last tile
        auto more = [&]() { return fills < stop_at + NL; };
        for (int s = 0; s < S && more(); s++) fill();
        for (int it = 0;; it++) {
            const int s = it % S;
            const long long j = tile_of[s];
            if (j >= ntiles) break;
            mbar_wait(&done_bar[s], (uint32_t)((it / S) & 1));
            bool stored = false;
            if (STORE && !is_ragged(j)) {
                bulk_store(prm.y + (size_t)tile_start(j), tile_words(stages + (size_t)s * SW), M * sizeof(T), pol);
                bulk_commit();
                stored = true;
            }
            if (it >= 1 && more()) {
                if (stored) bulk_wait_read<1>(); else bulk_wait_read<0>();
                fill();                                 // stage (it-1) % S, pipeline index it-1+S
            }
        }
        bulk_wait_all<0>();
        return;
    }

    // ===================================================== look-back warp ==
    // Runs a5 for the CTA's tiles in ticket order.  It learns the tile id from
    // the full barrier (as soon as the tile is loaded) and walks back without
    // waiting for the tile's own aggregate, which the compute warps publish.
    if (warp > W) {
        const uint32_t tagA = 2u * epoch, tagI = 2u * epoch + 1u;
        static_assert(NL <= kMaxNL, "look-back warps");
        const LbStats lbs{reinterpret_cast<unsigned long long*>(smem + L::off_lbstat) + (warp - W - 1) * kLbStatWords};
        lbs.init(lane);
        for (int it = warp - (W + 1);; it += NL) {     // NL look-back warps take turns
            const int s = it % S;
            const int slot = it % NS;
            mbar_wait(&full_bar[s], (uint32_t)((it / S) & 1));
            const long long j = tile_of[s];
            if (j >= ntiles) break;
            A Gp[K];                                           // G_{j-1}: carries entering tile j
            if (j == 0) {
#pragma unroll
                for (int q = 0; q < K; q++) Gp[q] = prm.y_hist != nullptr ? A(prm.y_hist[K - 1 - q]) : A(0);
            } else if (DEC) {
                // T(m) == 0: every tile published inclusive == aggregate at
                // once; the look-back is a single hop.  Poll only
                // once this tile's own phase A is done: its predecessor started
                // at the same time, so it is (almost) always published by then
                // and the poll does not steal issue slots from the compute warps.
                mbar_wait(&agg_bar[slot], (uint32_t)((it / NS) & 1));
                A v[K];
                if (lane == 0) {
                    int ns = 64;
                    SpinGuard guard;
                    while (read_status<A, K, DEC>(prm.status, prm.status_mask, j - 1, v, tagA, tagI) != 2) {
                        guard(7);
                        __nanosleep(ns);
                        ns = ns < 256 ? 2 * ns : ns;
                    }
                }
#pragma unroll
                for (int q = 0; q < K; q++) Gp[q] = shfl_idx(lane == 0 ? v[q] : A(0), 0);
            } else {
                // generic look-back: fold the tiles
                // j-1, j-2, ... nearest first, G_{j-1} = sum_d T(d m) v_{j-1-d},
                // v = aggregate for "P" tiles and the inclusive carry of the
                // first "I" tile.  Each poll folds the ready prefix of its
                // window (up to the first not-ready or first inclusive tile)
                // and never re-reads folded tiles.  Start once the tile's own
                // aggregate is published: the predecessors of the same wave
                // have had the same time to publish theirs.
                const long long c_start = clock64();
                mbar_wait(&agg_bar[slot], (uint32_t)((it / NS) & 1));
#ifndef PLR_LB_START
#define PLR_LB_START 0
#endif
                if (PLR_LB_START > 0 && D > 1) {
                    // start one tile later: the CTA's next aggregate is published,
                    // so are most predecessors' (phase B of this tile is still
                    // D-1 tiles away)
                    const int nx = it + 1;
                    mbar_wait(&agg_bar[nx % NS], (uint32_t)((nx / NS) & 1));
                }
                const long long c_agg = clock64();
                lookback_generic<T, A, K, DEC>(prm, tb, j, lane, tagA, tagI, Gp, lbs, c_start, c_agg);
            }
            // the tile's own aggregate (phase A) is needed for its inclusive carry
            if (j == 0 || DEC) mbar_wait(&agg_bar[slot], (uint32_t)((it / NS) & 1));
            if (lane == 0) {
#pragma unroll
                for (int q = 0; q < K; q++) sG[slot * kMaxK + q] = Gp[q];
            }
            if (!DEC || j == 0) {
                A G[K];
#pragma unroll
                for (int q = 0; q < K; q++) G[q] = sAt[slot * kMaxK + q];
                matvec_acc<A, K>(G, tb.Tm, Gp);                // G_j = A_j + T(m) G_{j-1}
                __syncwarp();
                if (lane == 0) mbar_arrive(&carry_bar[slot]);
                publish_status<A, K, DEC>(prm.status, prm.status_mask, j, G, tagI, lane);
            } else {
                __syncwarp();
                if (lane == 0) mbar_arrive(&carry_bar[slot]);
            }
        }
        lbs.flush(prm.stats, lane);
        return;
    }

    // ===================================================== compute warps ===
    A Tl[K * K];                                                // T(X*lane)
#pragma unroll
    for (int e = 0; e < K * K; e++) Tl[e] = prm.lane_T[e * 32 + lane];

    // phase A of pipeline iteration `it`: returns the tile id (>= ntiles: stop)
    auto phaseA = [&](int it) -> long long {
        const int s = it % S;
        const int slot = it % NS;
        mbar_wait(&full_bar[s], (uint32_t)((it / S) & 1));
        const long long j = tile_of[s];
        if (j >= ntiles) {
            if (tid == 0) { agg_tile[slot] = j; mbar_arrive(&agg_bar[slot]); }
            return j;
        }
        const bool ragged = is_ragged(j);
        T* st = stages + (size_t)s * SW;
        const long long g0 = j * (long long)M + (long long)tid * X;

        // a1: my X elements (+ P halo), FIR map in the data type
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
        // a2: sequential local recurrence with zero state, in A
        // chunk values are kept in the data type (phase B corrects them;
        // SEED: the map outputs t are kept instead); only the last K live in
        // the accumulation type.  The oldest term is added first so the
        // newest value l_{u-1} is on the critical path once.
        T lf[X];
        A hist[K];                                              // hist[r-1] = l_{u-r}
#pragma unroll
        for (int r = 0; r < K; r++) hist[r] = A(0);
#pragma unroll
        for (int u = 0; u < X; u++) {
            T t = tb.alpha[0] * xv[P + u];
#pragma unroll
            for (int q = 1; q <= P; q++) t = mad(tb.alpha[q], xv[P + u - q], t);
            if constexpr (SEED) lf[u] = t;
            A acc = cvt<A, T>(t);
#pragma unroll
            for (int r = K; r >= 1; r--)
                if (u - r >= 0) acc = mad(tb.c[r - 1], hist[r - 1], acc);
#pragma unroll
            for (int r = K - 1; r >= 1; r--) hist[r] = hist[r - 1];
            hist[0] = acc;
            if constexpr (!SEED) lf[u] = cvt<T, A>(acc);
        }
        A v[K];
#pragma unroll
        for (int q = 0; q < K; q++) v[q] = hist[q];             // local carry (l_{X-1}, ..., l_{X-K})

        // a3: warp inclusive scan with T(X * 2^s); DECAY skips the steps
        // whose transfer matrix is negligible (dec_mask, uniform branch)
#pragma unroll
        for (int s2 = 0; s2 < 5; s2++) {
            if (DEC && !((prm.dec_mask >> s2) & 1u)) continue;
            A o[K];
#pragma unroll
            for (int q = 0; q < K; q++) o[q] = shfl_up(v[q], 1 << s2);
            if (lane >= (1 << s2)) matvec_acc<A, K>(v, tb.Twarp[s2], o);
        }
#pragma unroll
        for (int q = 0; q < K; q++) {
            const A e = shfl_up(v[q], 1);
            sE[(slot * K + q) * NC + tid] = lane == 0 ? A(0) : e;  // warp-exclusive prefix
        }
        if (lane == 31) {
#pragma unroll
            for (int q = 0; q < K; q++) wagg[(slot * W + warp) * kMaxK + q] = v[q];
        }
        named_sync(1, NC);                                      // all x reads and wagg writes done

        // keep the chunk values (SEED: the map outputs t) for phase B in place
        // of x (data type).  SEED with p = 0: the stage keeps x (t = a0 x is
        // recomputed), except for the ragged tile the compute warps loaded
        if (!SEED || P > 0 || ragged) {
#pragma unroll
            for (int u = 0; u < X; u++) st[REV ? M - 1 - (tid * X + u) : kHalo + tid * X + u] = lf[u];
        }

        // a4, DECAY with T(32X d) == 0 for d >= 1 (dec_mask bit 5 clear): the
        // exclusive warp prefix is the previous warp's aggregate and the tile
        // aggregate the last warp's ("only the first few warps")
        if (DEC && !(prm.dec_mask & 32u)) {
            if (lane == 0) {
#pragma unroll
                for (int q = 0; q < K; q++)
                    sPw[(slot * W + warp) * K + q] = warp == 0 ? A(0) : wagg[(slot * W + warp - 1) * kMaxK + q];
            }
            if (tid == 0) {
#pragma unroll
                for (int q = 0; q < K; q++) sAt[slot * kMaxK + q] = wagg[(slot * W + W - 1) * kMaxK + q];
            }
            if (warp == 0) {
                A At[K];
#pragma unroll
                for (int q = 0; q < K; q++) At[q] = wagg[(slot * W + W - 1) * kMaxK + q];
                publish_status<A, K, DEC>(prm.status, prm.status_mask, j, At, 2u * epoch + 1u, lane);
            }
            __syncwarp();
            if (tid == 0) { agg_tile[slot] = j; mbar_arrive(&agg_bar[slot]); }
            return j;
        }
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
#pragma unroll
        for (int q = 0; q < K; q++) {
            const A pw = shfl_idx(u_[q], (warp + 31) & 31);
            const A at = shfl_idx(u_[q], W - 1);                // tile aggregate
            if (lane == 0) sPw[(slot * W + warp) * K + q] = warp == 0 ? A(0) : pw;
            if (tid == 0) sAt[slot * kMaxK + q] = at;
        }
        // publish the tile aggregate at once: "P" for the generic
        // look-back; for DECAY the inclusive carry equals the aggregate
        if (warp == 0 && (j > 0 || DEC)) {
            A At[K];
#pragma unroll
            for (int q = 0; q < K; q++) At[q] = shfl_idx(u_[q], W - 1);
            publish_status<A, K, DEC>(prm.status, prm.status_mask, j, At, DEC ? 2u * epoch + 1u : 2u * epoch, lane);
        }
        // wagg is buffered per slot: its next writer (tile it+NS) runs after
        // every warp passed tile it+1's barrier
        __syncwarp();                                           // sPw (lane 0) visible to the warp
        if (tid == 0) { agg_tile[slot] = j; mbar_arrive(&agg_bar[slot]); }
        return j;
    };

    // phase B of pipeline iteration `it` (tile id j)
    auto phaseB = [&](int it, long long j) {
        const int s = it % S;
        const int slot = it % NS;
        mbar_wait(&carry_bar[slot], (uint32_t)((it / NS) & 1));
        const bool ragged = is_ragged(j);
        T* st = stages + (size_t)s * SW;
        // the stage word of the thread's element u (REV: mirrored, original order)
        auto at = [&](int u) -> T& { return st[REV ? M - 1 - (tid * X + u) : kHalo + tid * X + u]; };
        const long long g0 = j * (long long)M + (long long)tid * X;
        A Gp[K], Win[K], Sst[K];
#pragma unroll
        for (int q = 0; q < K; q++) {
            Gp[q] = sG[slot * kMaxK + q];
            Win[q] = sPw[(slot * W + warp) * K + q];
        }
        if (DEC && !(prm.dec_mask & 32u)) {                    // T(32X w) == 0 for w >= 1
            if (warp == 0) {
#pragma unroll
                for (int q = 0; q < K; q++) Win[q] = Gp[q];
            }
        } else {
            matvec_acc<A, K>(Win, tb.Twin[warp], Gp);          // warp carry-in
        }
#pragma unroll
        for (int q = 0; q < K; q++) {                           // thread carry-in
            A acc = sE[(slot * K + q) * NC + tid];
#pragma unroll
            for (int r = 0; r < K; r++) acc = mad(Tl[q * K + r], Win[r], acc);
            Sst[q] = acc;
        }
        T Sd[K];
#pragma unroll
        for (int q = 0; q < K; q++) Sd[q] = cvt<T, A>(Sst[q]);
        T yv[X];
        if constexpr (SEED) {
            // a6: y_u = t_u + sum_r b-r y_{u-r}, seeded with Sd = (y_{-1}, ..., y_{-K})
            const bool has_t = P > 0 || ragged;
#pragma unroll
            for (int u = 0; u < X; u++) {
                T acc = has_t ? at(u) : tb.alpha[0] * at(u);
#pragma unroll
                for (int r = K; r >= 1; r--) acc = mad(tb.cT[r - 1], Sd[r - 1], acc);
#pragma unroll
                for (int r = K - 1; r >= 1; r--) Sd[r] = Sd[r - 1];
                Sd[0] = acc;
                yv[u] = acc;
            }
        } else {
#pragma unroll
            for (int u = 0; u < X; u++) {
                T acc = at(u);
#pragma unroll
                for (int r = 0; r < K; r++) acc = mad(tb.H[u][r], Sd[r], acc);
                yv[u] = acc;
            }
        }
        if (!ragged) {
            if (STORE) {
#pragma unroll
                for (int u = 0; u < X; u++) at(u) = yv[u];
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
        fence_proxy_async();
        mbar_arrive(&done_bar[s]);
    };

    // software pipeline: phase A runs D tiles ahead of phase B.  Phase B
    // reads its tile id from tile_of[], stable until the tile's done barrier.
    int na = 0, nb = 0;                             // phases A / B done
    for (; na < D; na++)
        if (phaseA(na) >= ntiles) break;
    for (bool stop = na < D; !stop;) {
        const long long j = phaseA(na);
        phaseB(nb, tile_of[nb % S]);
        nb++;
        if (j >= ntiles) stop = true; else na++;
    }
    for (; nb < na; nb++) phaseB(nb, tile_of[nb % S]);   // drain
}

}  // namespace dev
}  // namespace plr
