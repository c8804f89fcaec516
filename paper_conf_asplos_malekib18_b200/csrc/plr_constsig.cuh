// plr_constsig.cuh -- compile-time signature specialisation of the scan
// kernels (the paper's generator bakes the signature into the emitted code and
// specialises constant, 0/1 and repeating factors).
//
// For the integer signatures of Table 1 the planner selects a
// kernel instance whose coefficient and transfer-matrix tables are constexpr:
// the compiler folds multiplications by 0 / 1 / -1 / small constants and the
// permutation-shaped T(L) of the tuple sums into adds and register moves.
// Every other signature runs the same kernel with the tables read from the
// kernel parameters (SIG = 0).  The tables are the ones the host planner
// builds (plr_planner.cpp): T(L) = M^L in Z/2^32 for the companion matrix M
// of (1: c), h^(r)_u = T(u+1)[0][r-1].
#pragma once
#include <cstdint>

#include "plr_internal.h"

#ifdef __CUDACC__
#define PLR_HD __host__ __device__
#else
#define PLR_HD
#endif

namespace plr {

// signature ids: 0 = runtime tables; the rest are (1: c) with a0 = 1, p = 0
enum ConstSig : int {
    kSigRuntime = 0,
    kSigPrefix = 1,      // (1: 1)
    kSigTuple2 = 2,      // (1: 0, 1)
    kSigTuple3 = 3,      // (1: 0, 0, 1)
    kSigOrder2 = 4,      // (1: 2, -1)
    kSigOrder3 = 5,      // (1: 3, -3, 1)
};

PLR_HD constexpr int const_sig_k(int sig) {
    return sig == kSigPrefix ? 1 : (sig == kSigTuple2 || sig == kSigOrder2) ? 2 : (sig == 0 ? 0 : 3);
}

PLR_HD constexpr uint32_t const_sig_c(int sig, int r) {
    // b-1, ..., b-k in Z/2^32
    return sig == kSigPrefix ? (r == 0 ? 1u : 0u)
         : sig == kSigTuple2 ? (r == 1 ? 1u : 0u)
         : sig == kSigTuple3 ? (r == 2 ? 1u : 0u)
         : sig == kSigOrder2 ? (r == 0 ? 2u : r == 1 ? 0xFFFFFFFFu : 0u)
         : sig == kSigOrder3 ? (r == 0 ? 3u : r == 1 ? 0xFFFFFFFDu : r == 2 ? 1u : 0u)
         : 0u;
}

struct CMat {
    uint32_t v[kMaxK * kMaxK];
};

PLR_HD constexpr CMat cmat_mul(const CMat& a, const CMat& b) {
    CMat c{};
    for (int q = 0; q < kMaxK; q++)
        for (int r = 0; r < kMaxK; r++) {
            uint32_t acc = 0;
            for (int t = 0; t < kMaxK; t++) acc += a.v[q * kMaxK + t] * b.v[t * kMaxK + r];
            c.v[q * kMaxK + r] = acc;
        }
    return c;
}

PLR_HD constexpr CMat cmat_pow(const CMat& m, unsigned long long L) {
    CMat r{};
    for (int i = 0; i < kMaxK; i++) r.v[i * kMaxK + i] = 1u;
    CMat b = m;
    while (L) {
        if (L & 1) r = cmat_mul(r, b);
        L >>= 1;
        if (L) b = cmat_mul(b, b);
    }
    return r;
}

// companion matrix of (1: c), restricted to the signature's k (zero-padded)
PLR_HD constexpr CMat const_sig_companion(int sig) {
    CMat m{};
    const int k = const_sig_k(sig);
    for (int r = 0; r < k; r++) m.v[r] = const_sig_c(sig, r);
    for (int q = 1; q < k; q++) m.v[q * kMaxK + q - 1] = 1u;
    return m;
}

// Tables<uint32_t, uint32_t> of signature `sig` for the tile geometry (X, W)
// and look-back unit of G tiles
template <typename T, typename A>
PLR_HD constexpr Tables<T, A> const_tables(int sig, int X, int W, int G) {
    Tables<T, A> t{};
    if constexpr (sizeof(T) == 4 && sizeof(A) == 4 && T(-1) > T(0)) {   // uint32 ring only
        if (sig == 0) return t;
        const int k = const_sig_k(sig);
        const CMat M = const_sig_companion(sig);
        const unsigned long long m = 32ull * W * X;
        t.alpha[0] = 1u;
        for (int r = 0; r < k; r++) t.c[r] = t.cT[r] = const_sig_c(sig, r);
        CMat Tu = M;                                   // T(u+1)
        for (int u = 0; u < kMaxX; u++) {
            for (int r = 0; r < kMaxK; r++) t.H[u][r] = (u < X) ? Tu.v[r] : 0u;
            Tu = cmat_mul(Tu, M);
        }
        CMat P = cmat_pow(M, (unsigned long long)X);
        for (int s = 0; s < 5; s++) {
            for (int e = 0; e < kMaxK * kMaxK; e++) t.Twarp[s][e] = P.v[e];
            P = cmat_mul(P, P);
        }
        const CMat T32 = cmat_pow(M, 32ull * X);
        P = T32;
        for (int s = 0; s < 4; s++) {
            for (int e = 0; e < kMaxK * kMaxK; e++) t.Tblk[s][e] = P.v[e];
            P = cmat_mul(P, P);
        }
        CMat Wn{};
        for (int i = 0; i < kMaxK; i++) Wn.v[i * kMaxK + i] = 1u;
        for (int w = 0; w < kMaxW; w++) {
            for (int e = 0; e < kMaxK * kMaxK; e++) t.Twin[w][e] = Wn.v[e];
            Wn = cmat_mul(Wn, T32);
        }
        P = cmat_pow(M, m);
        for (int e = 0; e < kMaxK * kMaxK; e++) t.Tm[e] = P.v[e];
        CMat Gn{};
        for (int i = 0; i < kMaxK; i++) Gn.v[i * kMaxK + i] = 1u;
        for (int g = 0; g < kMaxG; g++) {
            for (int e = 0; e < kMaxK * kMaxK; e++) t.Tsub[g][e] = Gn.v[e];
            Gn = cmat_mul(Gn, P);
        }
        P = cmat_pow(M, m * (unsigned long long)G);          // look-back unit U = G m
        for (int s = 0; s < 9; s++) {
            for (int e = 0; e < kMaxK * kMaxK; e++) t.Tpow[s][e] = P.v[e];
            P = cmat_mul(P, P);
        }
    }
    return t;
}

}  // namespace plr
