// plr_planner.cpp -- host-side planner of the PLR hot path (row a0 of
// SURVEY.md §8(a)).
//
// The paper's generator checks the signature, computes the
// correction factors as n-nacci numbers and emits them as k
// constant arrays of m factors, with specialised code for
// constant, 0/1, repeating and decaying factors.  Here the
// planner computes, once per plan:
//   * the companion matrix M of (1: c) and every transfer matrix
//     T(L) = M^L the kernels need (repeated squaring; exact in Z/2^32, fp64
//     then rounded to fp32 with denormals flushed for floats, SURVEY §7
//     "Factor-table numerics");
//   * the per-element factors h^(r)_u = T(u+1)[0][r-1] for u < x;
//   * the class (ONES / PERM / POLY / DECAY / FLOAT) and, for DECAY, the
//     last index at which the fp32 impulse response is nonzero (L_dec) and
//     the free-response table used by the sharded fixup.
#include <cmath>
#include <cfloat>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "plr_constsig.cuh"
#include "plr_internal.h"

namespace plr {
namespace {

// ---- small dense matrices over a ring --------------------------------------
template <typename R>
struct Mat {
    int k;
    R v[kMaxK * kMaxK];
    explicit Mat(int k_ = 1) : k(k_) { for (auto& e : v) e = R(0); }
    R& at(int q, int r) { return v[q * kMaxK + r]; }
    R at(int q, int r) const { return v[q * kMaxK + r]; }
    static Mat eye(int k) { Mat m(k); for (int i = 0; i < k; i++) m.at(i, i) = R(1); return m; }
};

template <typename R>
Mat<R> mul(const Mat<R>& A, const Mat<R>& B) {
    Mat<R> C(A.k);
    for (int q = 0; q < A.k; q++)
        for (int r = 0; r < A.k; r++) {
            R acc = R(0);
            for (int t = 0; t < A.k; t++) acc += A.at(q, t) * B.at(t, r);
            C.at(q, r) = acc;
        }
    return C;
}

// companion matrix of the recurrence (1: c): S' = M S with
// S = (y_{s-1}, ..., y_{s-k}) and zero input.
template <typename R>
Mat<R> companion(const R* c, int k) {
    Mat<R> M(k);
    for (int r = 0; r < k; r++) M.at(0, r) = c[r];
    for (int q = 1; q < k; q++) M.at(q, q - 1) = R(1);
    return M;
}

template <typename R>
Mat<R> mpow(const Mat<R>& M, uint64_t L) {
    Mat<R> result = Mat<R>::eye(M.k), base = M;
    while (L) {
        if (L & 1) result = mul(result, base);
        L >>= 1;
        if (L) base = mul(base, base);
    }
    return result;
}

inline float ftz(double v) {
    float f = (float)v;
    if (std::fabs(f) < FLT_MIN) f = 0.0f;       // flush denormals
    return f;
}

template <typename R, typename T, typename Cvt>
void store_mat(const Mat<R>& m, T* dst, Cvt cvt) {
    for (int q = 0; q < kMaxK; q++)
        for (int r = 0; r < kMaxK; r++)
            dst[q * kMaxK + r] = (q < m.k && r < m.k) ? cvt(m.at(q, r)) : T(0);
}

// Fill every transfer-matrix table of Tables<T, A>; cvtA converts the ring
// value to the accumulation type, cvtT to the data type (per-element H).
template <typename R, typename T, typename A, typename CvtT, typename CvtA>
void fill_tables(const Mat<R>& M, int k, Geometry geo, Tables<T, A>* tb, A* lane, CvtT cvtT, CvtA cvtA) {
    const uint64_t X = geo.X, m = (uint64_t)geo.tile();
    for (int u = 0; u < kMaxX; u++) {
        Mat<R> Tu = mpow(M, (uint64_t)u + 1);
        for (int r = 0; r < kMaxK; r++) tb->H[u][r] = (u < geo.X && r < k) ? cvtT(Tu.at(0, r)) : T(0);
    }
    for (int s = 0; s < 5; s++) store_mat(mpow(M, X << s), tb->Twarp[s], cvtA);
    for (int s = 0; s < 4; s++) store_mat(mpow(M, (32 * X) << s), tb->Tblk[s], cvtA);
    for (int w = 0; w < kMaxW; w++) store_mat(mpow(M, 32 * X * (uint64_t)w), tb->Twin[w], cvtA);
    store_mat(mpow(M, m), tb->Tm, cvtA);
    const uint64_t U = m * (uint64_t)geo.G;                  // look-back unit
    for (int s = 0; s < 9; s++) store_mat(mpow(M, U << s), tb->Tpow[s], cvtA);
    for (int g = 0; g < kMaxG; g++) store_mat(mpow(M, m * (uint64_t)g), tb->Tsub[g], cvtA);
    for (int l = 0; l < 32; l++) {
        Mat<R> Tl = mpow(M, X * (uint64_t)l);
        for (int q = 0; q < k; q++)
            for (int r = 0; r < k; r++) lane[(q * k + r) * 32 + l] = cvtA(Tl.at(q, r));
    }
}

// DECAY tables whose entries are all below kCut are treated as exactly zero
// (reading R17): a carry of magnitude <= 2^10 then moves an output
// by <= 2^-50, nine decades under the 1e-4 tolerance.  The fp32 tables of
// the warp-aggregate level (L >= 32X = 480 > L_dec) are already exactly zero.
constexpr double kCut = 0x1p-60;

template <typename A>
bool negligible(const A* t) {
    for (int e = 0; e < kMaxK * kMaxK; e++)
        if (std::fabs((double)t[e]) > kCut) return false;
    return true;
}

// ScanParams::dec_mask of a DECAY plan's tables; negligible tables are zeroed
// so the kernels that still read them see the same values they skip.
template <typename T, typename A>
uint32_t decay_mask(Tables<T, A>* tb, A* lane, int k, Geometry geo) {
    uint32_t mask = 0;
    for (int s = 0; s < 5; s++) {
        if (!negligible(tb->Twarp[s])) mask |= 1u << s;
        else for (auto& e : tb->Twarp[s]) e = A(0);
    }
    bool blk = false;
    for (int s = 0; s < 4; s++) blk = blk || !negligible(tb->Tblk[s]);
    for (int w = 1; w < geo.W; w++) blk = blk || !negligible(tb->Twin[w]);
    if (blk) {
        mask |= 1u << 5;
    } else {
        for (int s = 0; s < 4; s++) for (auto& e : tb->Tblk[s]) e = A(0);
        for (int w = 1; w < kMaxW; w++) for (auto& e : tb->Twin[w]) e = A(0);
    }
    for (int l = 0; l < 32; l++) {
        double mx = 0.0;
        for (int e = 0; e < k * k; e++) mx = std::fmax(mx, std::fabs((double)lane[e * 32 + l]));
        if (mx <= kCut) for (int e = 0; e < k * k; e++) lane[e * 32 + l] = A(0);
    }
    return mask;
}

}  // namespace

plr_status plan_tables(const double* a, int p, const double* b, int k, plr_dtype dtype,
                       Geometry geo, PlanTables* out, const char** why) {
    *why = "";
    if (a == nullptr || b == nullptr || out == nullptr) { *why = "null argument"; return PLR_ERR_INVALID_ARG; }
    if (dtype != PLR_INT32 && dtype != PLR_FLOAT32) { *why = "dtype must be PLR_INT32 or PLR_FLOAT32"; return PLR_ERR_DTYPE; }
    if (k < 1) { *why = "order k must be >= 1 (P:89-93)"; return PLR_ERR_SIGNATURE; }
    if (p < 0) { *why = "p must be >= 0"; return PLR_ERR_SIGNATURE; }
    if (k > kMaxK || p > kMaxP) { *why = "k > PLR_MAX_K or p > PLR_MAX_P"; return PLR_ERR_SIZE; }
    for (int j = 0; j <= p; j++) if (!std::isfinite(a[j])) { *why = "non-finite coefficient"; return PLR_ERR_SIGNATURE; }
    for (int j = 0; j < k; j++) if (!std::isfinite(b[j])) { *why = "non-finite coefficient"; return PLR_ERR_SIGNATURE; }
    if (a[p] == 0.0) { *why = "last non-recursive coefficient must not be zero (P:635-637)"; return PLR_ERR_SIGNATURE; }
    if (b[k - 1] == 0.0) { *why = "last recursive coefficient must not be zero (P:635-637)"; return PLR_ERR_SIGNATURE; }
    if (dtype == PLR_INT32) {
        for (int j = 0; j <= p + k; j++) {
            double v = j <= p ? a[j] : b[j - p - 1];
            if (v != std::floor(v) || v < -2147483648.0 || v >= 4294967296.0) {
                *why = "PLR_INT32 needs integer coefficients in [-2^31, 2^32)";
                return PLR_ERR_SIGNATURE;
            }
        }
    } else {
        for (int j = 0; j <= p + k; j++) {
            double v = j <= p ? a[j] : b[j - p - 1];
            if (std::fabs(v) > FLT_MAX) { *why = "coefficient overflows fp32"; return PLR_ERR_SIGNATURE; }
        }
        if ((float)a[p] == 0.0f || (float)b[k - 1] == 0.0f) { *why = "last coefficient rounds to 0 in fp32"; return PLR_ERR_SIGNATURE; }
    }
    if (geo.X < k || geo.X > kMaxX || geo.W > kMaxW || (geo.W & (geo.W - 1)) || geo.G < 1 || geo.G > kMaxG) {
        *why = "bad geometry";
        return PLR_ERR_INVALID_ARG;
    }

    PlanTables& pt = *out;
    std::memset(&pt, 0, sizeof(pt));
    pt.p = p; pt.k = k; pt.dtype = dtype; pt.geo = geo;
    pt.geo_s = Geometry{kSmallX, kSmallW, 1, 1};
    pt.dec_mask_s = 0x3fu;
    pt.decay_len = -1; pt.fixup_len = 0;
    pt.dec_mask = 0x3fu;
    pt.fix_table = nullptr;

    if (dtype == PLR_INT32) {
        uint32_t c[kMaxK] = {0};
        for (int j = 0; j <= p; j++) pt.a_u[j] = (uint32_t)(int64_t)(a[j] < 0 ? a[j] : std::fmod(a[j], 4294967296.0));
        for (int j = 0; j < k; j++) c[j] = pt.b_u[j] = (uint32_t)(int64_t)(b[j] < 0 ? b[j] : std::fmod(b[j], 4294967296.0));
        for (int j = 0; j <= kMaxP; j++) pt.ti.alpha[j] = j <= p ? pt.a_u[j] : 0u;
        for (int j = 0; j < kMaxK; j++) pt.ti.c[j] = pt.ti.cT[j] = j < k ? c[j] : 0u;
        Mat<uint32_t> M = companion<uint32_t>(c, k);
        auto id = [](uint32_t v) { return v; };
        fill_tables(M, k, geo, &pt.ti, pt.lane_i, id, id);
        {
            Geometry g1 = geo;
            g1.G = 1;
            uint32_t lane_tmp[kMaxK * kMaxK * 32];
            pt.ti1 = pt.ti;                    // coefficients (alpha, c); the matrices are refilled
            fill_tables(M, k, g1, &pt.ti1, lane_tmp, id, id);
        }
        pt.tis = pt.ti;                        // small-n kernel tables (own geometry, units of one tile)
        fill_tables(M, k, pt.geo_s, &pt.tis, pt.lane_is, id, id);
        {
            uint32_t lane_tmp[kMaxK * kMaxK * 32];
            pt.tr = pt.ti;                     // reduce-only kernel tables
            fill_tables(M, k, Geometry{kRedX, kRedW, kRedS, 1}, &pt.tr, lane_tmp, id, id);
        }
        // class: all factors 1 -> ONES; single unit feedback
        // coefficient -> PERM (0/1 repeating factors); otherwise POLY
        int nnz = 0, ones = 0;
        for (int j = 0; j < k; j++) { nnz += c[j] != 0; ones += c[j] == 1u; }
        if (k == 1 && c[0] == 1u) pt.cls = PLR_CLASS_ONES;
        else if (nnz == 1 && ones == 1) pt.cls = PLR_CLASS_PERM;
        else pt.cls = PLR_CLASS_POLY;
        pt.decay_flag = 0;
        // compile-time signature kernels for the integer rows of Table 1
        // (P:96-104), a0 = 1, p = 0 (plr_constsig.cuh)
        pt.sig_id = 0;
        if (p == 0 && pt.a_u[0] == 1u) {
            for (int sig = kSigPrefix; sig <= kSigOrder3; sig++) {
                if (const_sig_k(sig) != k) continue;
                bool eq = true;
                for (int j = 0; j < k; j++) eq = eq && c[j] == const_sig_c(sig, j);
                if (eq) pt.sig_id = sig;
            }
        }
    } else {
        double c[kMaxK] = {0}, al[kMaxP + 1] = {0};
        for (int j = 0; j <= p; j++) al[j] = pt.a_d[j] = (double)(float)a[j];
        for (int j = 0; j < k; j++) c[j] = pt.b_d[j] = (double)(float)b[j];
        for (int j = 0; j <= kMaxP; j++) pt.tf.alpha[j] = pt.td.alpha[j] = j <= p ? (float)al[j] : 0.0f;
        for (int j = 0; j < kMaxK; j++) pt.tf.c[j] = j < k ? (float)c[j] : 0.0f;
        for (int j = 0; j < kMaxK; j++) pt.td.c[j] = j < k ? c[j] : 0.0;
        for (int j = 0; j < kMaxK; j++) pt.tf.cT[j] = pt.td.cT[j] = j < k ? (float)c[j] : 0.0f;
        Mat<double> M = companion<double>(c, k);
        auto f32 = [](double v) { return ftz(v); };
        // fp64 accumulation keeps denormal-range values that fp32 would flush;
        // flush them too so both precisions see the same (exactly 0) tails
        auto f64 = [](double v) { return std::fabs(v) < (double)FLT_MIN ? 0.0 : v; };
        fill_tables(M, k, geo, &pt.tf, pt.lane_f, f32, f32);
        fill_tables(M, k, geo, &pt.td, pt.lane_d, f32, f64);
        {
            Geometry g1 = geo;
            g1.G = 1;
            double lane_tmp[kMaxK * kMaxK * 32];
            pt.td1 = pt.td;                    // coefficients (alpha, c); the matrices are refilled
            fill_tables(M, k, g1, &pt.td1, lane_tmp, f32, f64);
        }
        pt.tfs = pt.tf;                        // small-n kernel tables (own geometry, units of one tile)
        pt.tds = pt.td;
        fill_tables(M, k, pt.geo_s, &pt.tfs, pt.lane_fs, f32, f32);
        fill_tables(M, k, pt.geo_s, &pt.tds, pt.lane_ds, f32, f64);
        {
            double lane_tmp[kMaxK * kMaxK * 32];
            pt.trd = pt.td;                    // reduce-only kernel tables
            fill_tables(M, k, Geometry{kRedX, kRedW, kRedS, 1}, &pt.trd, lane_tmp, f32, f64);
        }
        // DECAY: the fp32 impulse response g of (1: c) becomes
        // exactly 0 and stays 0.  g_0 = 1, g_u = sum_j c_j g_{u-j}.
        const int64_t cap = 1 << 16;
        std::vector<double> g(cap, 0.0);
        int64_t last = -1;
        for (int64_t u = 0; u < cap; u++) {
            double v = (u == 0) ? 1.0 : 0.0;
            for (int j = 1; j <= k; j++) if (u - j >= 0) v += c[j - 1] * g[u - j];
            g[u] = v;
            if (ftz(v) != 0.0f) last = u;
        }
        const bool decays = last < cap / 2;
        bool tm_zero = true;
        for (int e = 0; e < kMaxK * kMaxK; e++) tm_zero = tm_zero && pt.tf.Tm[e] == 0.0f && pt.td.Tm[e] == 0.0;
        pt.decay_flag = (decays && tm_zero) ? 1 : 0;
        pt.cls = decays ? PLR_CLASS_DECAY : PLR_CLASS_FLOAT;
        // Accumulation precision (reading R16).  The zero-state
        // chunk values l_u and the carries reach ~sum|a| * sum|g| times the
        // input scale, and their rounding errors are amplified by the
        // transfer matrices again (~sum|g|): a-priori bound
        // eps32 * sum|a| * (sum|g|)^2 relative to the input scale.  The
        // tolerance is relative to the OUTPUT (1e-4 max(1,|y|)), so the bound
        // is divided by the gain the filter leaves an input at the Nyquist
        // frequency -- the worked example's (-1)^i (i+3) pattern, the
        // input a low-pass filter attenuates most: |H(-1)| = |A(-1)| / |B(-1)|
        // (capped at 1).  Above 1e-3 (10x the tolerance) the chunk recurrence
        // and every carry accumulate in fp64 (B200 fp64 runs at half the fp32
        // rate); data, the map and phase B stay fp32.
        double sa = 0.0, sg = 0.0;
        for (int j = 0; j <= p; j++) sa += std::fabs(al[j]);
        for (int64_t u = 0; u < cap; u++) sg += std::fabs(g[u]);
        double an = 0.0, bn = 1.0;                       // A(-1), B(-1) = 1 - sum_j c_j (-1)^j
        for (int j = 0; j <= p; j++) an += (j & 1) ? -al[j] : al[j];
        for (int j = 1; j <= k; j++) bn -= (j & 1) ? -c[j - 1] : c[j - 1];
        const double nyq = bn != 0.0 ? std::fabs(an / bn) : 1.0;
        pt.cond_bound = std::ldexp(1.0, -24) * sa * sg * sg / std::fmin(1.0, nyq);
        // R20: the floor every fp32-data evaluation (the serial one too) has
        // relative to the output: the map's fp32 rounding of the input scale,
        // amplified once by the recurrence, over the Nyquist gain
        pt.map_floor = std::ldexp(1.0, -24) * sa * sg / std::fmin(1.0, nyq);
        pt.nyquist_gain = nyq;
        pt.acc64 = (!decays || !(pt.cond_bound <= 1e-3)) ? 1 : 0;
        if (!pt.decay_flag) pt.acc64 = 1;      // multi-tile look-back kernels exist in fp64 accumulation only
        pt.dec_mask = 0x3fu;
        if (pt.decay_flag)                     // DECAY hierarchy: skip the negligible transfer matrices
            pt.dec_mask = pt.acc64 ? decay_mask(&pt.td, pt.lane_d, k, geo) : decay_mask(&pt.tf, pt.lane_f, k, geo);
        bool tms_zero = true;
        for (int e = 0; e < kMaxK * kMaxK; e++) tms_zero = tms_zero && pt.tfs.Tm[e] == 0.0f && pt.tds.Tm[e] == 0.0;
        pt.decay_s = (decays && tms_zero) ? 1 : 0;
        pt.dec_mask_s = 0x3fu;
        if (pt.decay_s)
            pt.dec_mask_s = pt.acc64 ? decay_mask(&pt.tds, pt.lane_ds, k, pt.geo_s)
                                     : decay_mask(&pt.tfs, pt.lane_fs, k, pt.geo_s);
        if (decays) {
            pt.decay_len = last;
            // free response of the augmented state (x_{-4..-1}, y_{-4..-1})
            std::vector<double> F((size_t)cap * kAug, 0.0);
            int64_t lastf = -1;
            for (int slot = 0; slot < kAug; slot++) {
                std::vector<double> xs(4, 0.0), ys(4, 0.0);
                if (slot < 4) xs[slot] = 1.0; else ys[slot - 4] = 1.0;
                std::vector<double> y(cap, 0.0);
                for (int64_t i = 0; i < cap; i++) {
                    double v = 0.0;
                    for (int j = 1; j <= p; j++) v += al[j] * (i - j >= 0 ? 0.0 : xs[4 + (i - j)]);
                    for (int j = 1; j <= k; j++) v += c[j - 1] * (i - j >= 0 ? y[i - j] : ys[4 + (i - j)]);
                    y[i] = v;
                    F[(size_t)i * kAug + slot] = v;
                    if (ftz(v) != 0.0f && i > lastf) lastf = i;
                }
            }
            pt.fixup_len = lastf + 1;
            pt.fix_table = (float*)std::malloc(sizeof(float) * (size_t)(pt.fixup_len > 0 ? pt.fixup_len : 1) * kAug);
            for (int64_t i = 0; i < pt.fixup_len; i++)
                for (int s = 0; s < kAug; s++) pt.fix_table[i * kAug + s] = ftz(F[(size_t)i * kAug + s]);
        }
    }
    return PLR_OK;
}

void plan_tables_free(PlanTables* pt) {
    if (pt && pt->fix_table) { std::free(pt->fix_table); pt->fix_table = nullptr; }
}

// k rows of (k + m): seed in memory order w_{m-k}..w_{m-1} (a one at the
// carry's position), then h^(r)_u = T(u+1)[0][r-1], u < m, from
// the same matrix powers the kernel tables come from.
void factor_lists(const PlanTables& pt, int64_t m, void* out) {
    const int k = pt.k;
    const int64_t len = k + m;
    if (pt.dtype == PLR_INT32) {
        uint32_t* o = (uint32_t*)out;
        Mat<uint32_t> M = companion<uint32_t>(pt.ti.c, k);
        for (int r = 1; r <= k; r++)
            for (int q = 0; q < k; q++) o[(r - 1) * len + q] = (q == k - r) ? 1u : 0u;
        Mat<uint32_t> Tu = Mat<uint32_t>::eye(k);
        for (int64_t u = 0; u < m; u++) {
            Tu = mpow(M, (uint64_t)u + 1);
            for (int r = 1; r <= k; r++) o[(r - 1) * len + k + u] = Tu.at(0, r - 1);
        }
    } else {
        float* o = (float*)out;
        Mat<double> M = companion<double>(pt.b_d, k);
        for (int r = 1; r <= k; r++)
            for (int q = 0; q < k; q++) o[(r - 1) * len + q] = (q == k - r) ? 1.0f : 0.0f;
        for (int64_t u = 0; u < m; u++) {
            Mat<double> Tu = mpow(M, (uint64_t)u + 1);
            for (int r = 1; r <= k; r++) o[(r - 1) * len + k + u] = ftz(Tu.at(0, r - 1));
        }
    }
}

}  // namespace plr
