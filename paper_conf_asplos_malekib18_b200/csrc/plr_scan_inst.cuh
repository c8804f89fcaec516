// plr_scan_inst.cuh -- host-side launch of the scan kernel for one
// (data type T, accumulation type A, pipeline config); included by the
// per-type .cu files so the instantiations compile in parallel.
#pragma once
#include "plr_kernels.cuh"
#include "plr_kernels_tmem.cuh"
#include "plr_kernels_rr.cuh"
#include "plr_kernels_dect.cuh"
#include "plr_launch.h"
#include <atomic>
#include <type_traits>

namespace plr {
namespace inst {

// Pipeline configs (measured on B200):
//   DECAY, fp32 and fp64 accumulation: the forward pass runs the
//   TMEM-parked kernel (plr_scan_dect_kernel); a kernel that allocates TMEM
//   runs one CTA per SM (profiles/r03g_tmem_occupancy.txt), so one wide CTA:
//   X = 31, W = 16 (tile 15872), 2 load stages + 1 store stage (measured
//   r03k: LP3 1.01, HP3 0.995 of a copy, against 0.83 / 0.81 for the
//   in-place kernel at 3 CTAs/SM with X = 31, W = 4; the fp32 rows 1.04
//   against 0.97-1.01 in place; profiles/r03h_*, r03i_*, r03k_*).  The
//   in-place kernel (S = 3 stages at this geometry) serves the anticausal
//   pass of fp32 plans; fp64 plans run that on the small-n kernel.
//   generic (multi-tile look-back, GEN_KIND 0, not shipped): S = 3, D = 1.
#ifndef PLR_DEC_S
#define PLR_DEC_S 3
#define PLR_DEC_D 1
#define PLR_DEC_NL 1
#define PLR_DEC_X 31
#define PLR_DEC_W 16
#define PLR_DEC_MINB 1
#endif
#ifndef PLR_DEC64_S
#define PLR_DEC64_S 3
#define PLR_DEC64_D 1
#define PLR_DEC64_NL 1
#define PLR_DEC64_X 31
#define PLR_DEC64_W 16
#define PLR_DEC64_MINB 1
#endif
#ifndef PLR_GEN_S
#define PLR_GEN_S 3
#define PLR_GEN_D 1
#define PLR_GEN_NL 2
#define PLR_GEN_X 31
#define PLR_GEN_W 16
#define PLR_GEN_MINB 1
#endif
// Kernel of the generic (non-decaying) classes, PLR_GEN_KIND:
//   2 (default) re-read kernel (plr_kernels_rr.cuh): phase B re-reads x from
//     L2 and recomputes from the true carry-in; lag NS-1 tiles
//   1 TMEM-parking kernel (plr_kernels_tmem.cuh): chunk values of up to 8
//     tiles parked in TMEM, phase B corrects them
//   0 shared-memory pipeline kernel (plr_scan_kernel, S-stage ring)
#ifndef PLR_GEN_KIND
#define PLR_GEN_KIND 2
#endif
// first-order signatures (k = 1) use their own kernel kind: the TMEM kernel
// reaches memcpy speed there (measured), the re-read kernel for k >= 2
#ifndef PLR_K1_KIND
#define PLR_K1_KIND 1
#endif
#define PLR_GEN_TMEM (PLR_GEN_KIND != 0)
// re-read kernel (measured r01r-r01u): X = 31, W = 8 (tile 7936), 3 look-back
// warps, 2 HBM load stages, 5 L2 re-read / store stages, phase-B lag 8 tiles,
// look-back units of 6 tiles with NS = 10 slots (r03d, profiles/r03d_rr_unit_cmp.txt:
// tuple3 0.910 -> 0.923, order2 0.936 -> 0.944 against G = 4 / NS = 9; the
// configuration hung before the chained agg waits of DESIGN.md §10)
#ifndef PLR_RR_X
#define PLR_RR_X 31
#endif
#ifndef PLR_RR_W
#define PLR_RR_W 8
#endif
#ifndef PLR_RR_NL
#define PLR_RR_NL 3
#endif
#ifndef PLR_RR_SA
#define PLR_RR_SA 2         // phase-A (HBM) load stages
#endif
#ifndef PLR_RR_SB
#define PLR_RR_SB 5         // phase-B (L2 re-read + y store) stages
#endif
#ifndef PLR_RR_NS
#define PLR_RR_NS 10        // slots: phase B lags phase A by NS-1 tiles (L2 reuse distance)
#endif
#ifndef PLR_RR_G
#define PLR_RR_G 6          // tiles per look-back unit (one ticket, one look-back)
#endif
#ifndef PLR_TM_X
#define PLR_TM_X 15
#endif
#ifndef PLR_TM_W
#define PLR_TM_W 16
#endif
#ifndef PLR_TM_NL
#define PLR_TM_NL 2
#endif
#ifndef PLR_TM_SL
#define PLR_TM_SL 3
#endif
#ifndef PLR_TM_ST
#define PLR_TM_ST 3
#endif
#ifndef PLR_TM_G
#define PLR_TM_G 3          // tiles per look-back unit (one ticket, one look-back)
#endif

// kernel kind of a non-decaying signature of order k (see PLR_GEN_KIND)
constexpr int gen_kind(int k) { return k == 1 ? PLR_K1_KIND : PLR_GEN_KIND; }

// S-stage ring, phase-A lead D, NL look-back warps, X elements per thread,
// W compute warps (tile m = 32 W X)
// W compute warps (tile m = 32 W X); MINB: CTAs per SM the registers must allow
// U1_: look-back units of one tile (the small-n launches, plr_api.cu), else
// PLR_RR_G / PLR_TM_G tiles per unit
// SEED_: phase B runs the seeded serial recurrence (plr_scan_kernel SEED)
// DT_: the forward DECAY pass runs plr_scan_dect_kernel (map outputs parked
// in TMEM, split load / store rings: PLR_DT_SL / PLR_DT_ST stages, lag PLR_DT_D)
template <int S_, int D_, int NL_, int X_, int W_, int MINB_, bool DEC_, bool U1_ = false, bool SEED_ = false,
          bool DT_ = false>
struct Cfg {
    static constexpr int S = S_, D = D_, NL = NL_, X = X_, W = W_, MINB = MINB_;
    static constexpr bool DEC = DEC_, U1 = U1_, SEED = SEED_, DT = DT_;
};
#ifndef PLR_DT_SL
#define PLR_DT_SL 2
#endif
#ifndef PLR_DT_ST
#define PLR_DT_ST 1
#endif
#ifndef PLR_DT_D
#define PLR_DT_D 1
#endif
#ifndef PLR_DEC_DT
#define PLR_DEC_DT 1
#endif
#ifndef PLR_DEC64_DT
#define PLR_DEC64_DT 1
#endif
// DECAY phase B (measured r03b at 2^30, fraction of copy): fp32 plans keep
// the correction y = l + sum_r S_r h^(r)_u (independent FMAs; seeded: LP1
// 0.99 -> 0.95, HP2 0.98 -> 0.95, the serial chain is exposed); fp64-
// accumulation plans run the fp32 recurrence seeded with the fp64 carry
// (no per-element fp64 -> fp32 conversion of l, no factor table: HP3 0.79 ->
// 0.81)
#ifndef PLR_DEC_SEED
#define PLR_DEC_SEED 0
#endif
#ifndef PLR_DEC64_SEED
#define PLR_DEC64_SEED 1
#endif
using CfgDec = Cfg<PLR_DEC_S, PLR_DEC_D, PLR_DEC_NL, PLR_DEC_X, PLR_DEC_W, PLR_DEC_MINB, true, false, PLR_DEC_SEED,
                   PLR_DEC_DT != 0>;
using CfgDec64 = Cfg<PLR_DEC64_S, PLR_DEC64_D, PLR_DEC64_NL, PLR_DEC64_X, PLR_DEC64_W, PLR_DEC64_MINB, true, false,
                     PLR_DEC64_SEED, PLR_DEC64_DT != 0>;
using CfgGen = Cfg<PLR_GEN_S, PLR_GEN_D, PLR_GEN_NL, PLR_GEN_X, PLR_GEN_W, PLR_GEN_MINB, false>;
using CfgGen1 = Cfg<PLR_GEN_S, PLR_GEN_D, PLR_GEN_NL, PLR_GEN_X, PLR_GEN_W, PLR_GEN_MINB, false, true>;

template <typename T, typename A, int K, bool U1>
struct TmCfg {
    static constexpr int X = PLR_TM_X, W = PLR_TM_W, NL = PLR_TM_NL, SL = PLR_TM_SL, ST = PLR_TM_ST;
    static constexpr int G = U1 ? 1 : PLR_TM_G;
    static constexpr int CW = dev::TmemCols<A, K, X>::CW;
#ifndef PLR_TM_NTMAX
#define PLR_TM_NTMAX 8
#endif
    static constexpr int NT0 = 512 / ((W / 4) * CW);
    static constexpr int NT = NT0 > PLR_TM_NTMAX ? PLR_TM_NTMAX : NT0;
};

template <typename T, typename A, class C, int K, int P, bool STORE, int SIG = 0>
cudaError_t launch_kps(const Tables<T, A>& tab, const LaunchArgs& la) {
    constexpr int kind = C::DEC ? 0 : gen_kind(K);
    constexpr bool tmem = kind != 0;
    size_t smem;
    int threads;
    void (*kern)(const ScanParams<T, A>);
    if constexpr (kind == 2) {
        kern = &dev::plr_scan_rr_kernel<T, A, K, P, PLR_RR_X, PLR_RR_W, PLR_RR_SA, PLR_RR_SB, PLR_RR_NS, PLR_RR_NL,
                                         C::U1 ? 1 : PLR_RR_G, STORE, SIG>;
        if constexpr (STORE) {                           // the anticausal pass
            if (la.reverse)
                kern = &dev::plr_scan_rr_kernel<T, A, K, P, PLR_RR_X, PLR_RR_W, PLR_RR_SA, PLR_RR_SB, PLR_RR_NS,
                                                 PLR_RR_NL, C::U1 ? 1 : PLR_RR_G, STORE, SIG, true>;
        }
        smem = dev::LayoutR<T, A, K, PLR_RR_X, PLR_RR_W, PLR_RR_SA, PLR_RR_SB, PLR_RR_NS>::bytes;
        threads = (PLR_RR_W + 1 + PLR_RR_NL) * 32;
    } else if constexpr (tmem) {
        using TC = TmCfg<T, A, K, C::U1>;
        kern = &dev::plr_scan_tmem_kernel<T, A, K, P, TC::X, TC::W, TC::SL, TC::ST, TC::NT, TC::NL, TC::G, STORE, SIG>;
        if constexpr (STORE) {                           // the anticausal pass
            if (la.reverse)
                kern = &dev::plr_scan_tmem_kernel<T, A, K, P, TC::X, TC::W, TC::SL, TC::ST, TC::NT, TC::NL, TC::G,
                                                   STORE, SIG, true>;
        }
        smem = dev::LayoutT<T, A, K, TC::X, TC::W, TC::SL, TC::ST, TC::NT>::bytes;
        threads = (TC::W + 1 + TC::NL) * 32;
    } else {
        kern = &dev::plr_scan_kernel<T, A, K, P, C::X, C::W, C::S, C::D, C::NL, C::DEC, STORE, C::MINB, C::SEED>;
        smem = dev::Layout<T, A, K, C::X, C::W, C::S, C::D>::bytes;
        threads = (C::W + 1 + C::NL) * 32;
        if constexpr (C::DEC && STORE) {                 // the anticausal pass (DECAY plans)
            if (la.reverse)
                kern = &dev::plr_scan_kernel<T, A, K, P, C::X, C::W, C::S, C::D, C::NL, C::DEC, STORE, C::MINB, C::SEED,
                                             true>;
        }
        if constexpr (C::DEC && STORE && C::DT) {         // DECAY passes with TMEM-parked map outputs
            kern = la.reverse
                ? &dev::plr_scan_dect_kernel<T, A, K, P, C::X, C::W, PLR_DT_SL, PLR_DT_ST, PLR_DT_D, C::MINB, true>
                : &dev::plr_scan_dect_kernel<T, A, K, P, C::X, C::W, PLR_DT_SL, PLR_DT_ST, PLR_DT_D, C::MINB, false>;
            smem = dev::LayoutDT<T, A, K, C::X, C::W, PLR_DT_SL, PLR_DT_ST, PLR_DT_D + 1>::bytes;
            threads = (C::W + 2) * 32;
        }
    }
    // the > 48 KB dynamic shared memory opt-in is a per-device (context)
    // attribute: one bit per device and kernel, set once (racing sets are
    // idempotent); bit 63 - dev: the reverse kernel
    static std::atomic<unsigned long long> configured{0};
    int dev = 0;
    if (cudaError_t e = cudaGetDevice(&dev); e != cudaSuccess) return e;
    const unsigned long long bit = 1ull << (la.reverse ? 63 - (dev & 31) : (dev & 31));
    if (!(configured.load(std::memory_order_acquire) & bit)) {
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        configured.fetch_or(bit, std::memory_order_acq_rel);
    }
    if (la.occupancy_out != nullptr) {  // occupancy query: report CTAs/SM, do not launch
        cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(la.occupancy_out, kern, threads, smem);
        if (tmem && *la.occupancy_out > 1) *la.occupancy_out = 1;   // 512 TMEM columns per CTA
        return e;
    }
    const ScanParams<T, A> prm = make_params(tab, la);
    kern<<<la.grid, threads, smem, la.stream>>>(prm);
    return cudaGetLastError();
}

// compile-time signature kernels (int32 ring, p = 0, TMEM kernel only)
template <typename T, typename A, class C, int K, int SIG>
cudaError_t launch_sig(const Tables<T, A>& tab, const LaunchArgs& la) {
    return la.store ? launch_kps<T, A, C, K, 0, true, SIG>(tab, la) : launch_kps<T, A, C, K, 0, false, SIG>(tab, la);
}

template <typename T, typename A, class C, int K>
cudaError_t launch_k(const Tables<T, A>& tab, const LaunchArgs& la, int p) {
    if constexpr (std::is_same<T, uint32_t>::value && std::is_same<A, uint32_t>::value && gen_kind(K) != 0 && !C::DEC) {
        if (la.sig != 0 && p == 0) {
            if constexpr (K == 1) { if (la.sig == kSigPrefix) return launch_sig<T, A, C, 1, kSigPrefix>(tab, la); }
            if constexpr (K == 2) {
                if (la.sig == kSigTuple2) return launch_sig<T, A, C, 2, kSigTuple2>(tab, la);
                if (la.sig == kSigOrder2) return launch_sig<T, A, C, 2, kSigOrder2>(tab, la);
            }
            if constexpr (K == 3) {
                if (la.sig == kSigTuple3) return launch_sig<T, A, C, 3, kSigTuple3>(tab, la);
                if (la.sig == kSigOrder3) return launch_sig<T, A, C, 3, kSigOrder3>(tab, la);
            }
            return cudaErrorInvalidValue;
        }
    }
    switch (p) {
        case 0: return la.store ? launch_kps<T, A, C, K, 0, true>(tab, la) : launch_kps<T, A, C, K, 0, false>(tab, la);
        case 1: return la.store ? launch_kps<T, A, C, K, 1, true>(tab, la) : launch_kps<T, A, C, K, 1, false>(tab, la);
        case 2: return la.store ? launch_kps<T, A, C, K, 2, true>(tab, la) : launch_kps<T, A, C, K, 2, false>(tab, la);
        case 3: return la.store ? launch_kps<T, A, C, K, 3, true>(tab, la) : launch_kps<T, A, C, K, 3, false>(tab, la);
    }
    return cudaErrorInvalidValue;
}

template <typename T, typename A, class C>
cudaError_t launch(const Tables<T, A>& tab, const LaunchArgs& la, int k, int p) {
    switch (k) {
        case 1: return launch_k<T, A, C, 1>(tab, la, p);
        case 2: return launch_k<T, A, C, 2>(tab, la, p);
        case 3: return launch_k<T, A, C, 3>(tab, la, p);
        case 4: return launch_k<T, A, C, 4>(tab, la, p);
    }
    return cudaErrorInvalidValue;
}

}  // namespace inst
}  // namespace plr
