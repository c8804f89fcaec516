// plr_internal.h -- shared between the host planner, the kernels and the ABI.
// Product code only; nothing here is shared with oracle/.
#pragma once
#include <cstddef>
#include <cstdint>

#include "../../include/plr.h"

namespace plr {

// ---- kernel geometry -------------------------------------------------------
// X contiguous elements per thread (odd: conflict-free strided shared-memory
// access), W compute warps, S-stage shared-memory ring, plus one producer warp
// (tickets, TMA bulk loads/stores) and one look-back warp.
constexpr int kMaxK = PLR_MAX_K;
constexpr int kMaxP = PLR_MAX_P;
constexpr int kHalo = 4;            // words in front of each stage: x_{-4}..x_{-1}
constexpr int kMaxX = 31;
constexpr int kMaxW = 16;
constexpr int kStatusWords = 4;     // u64 status words per tile (>= kMaxK)
constexpr int kStatusMaxBytes = 128; // bytes per status slot the plan allocates (max record stride)
constexpr int kAug = 8;             // augmented state slots: x_{-4..-1}, y_{-4..-1}
constexpr int kTPL = 8;             // look-back: tiles per lane in a wide window (2^3)

constexpr int kMaxG = 8;            // tiles per look-back unit (ticket)

// G consecutive tiles form one look-back unit: one ticket, one status record
// and one look-back per unit (the generic TMEM kernel; G = 1 elsewhere).
struct Geometry {
    int X, W, S, G;
    int tile() const { return 32 * W * X; }
};

// Tables the scan kernel reads from its parameter space.  T is the data type
// (uint32_t ring or float), A the accumulation type of the local recurrence
// and of every carry (uint32_t, float or double; see plan_tables()).
//   T(L)[q][r] = coefficient of S_r in S(s+L)_q, S(s) = (y_{s-1}, ..., y_{s-k}),
// i.e. T(L) = M^L for the companion matrix M, and T(L)[q][r] = h^(r+1)_{L-1-q}
// (the seed-extended correction factors of Sec. 2.1).
template <typename T, typename A>
struct Tables {
    T alpha[kMaxP + 1];                  // a0, a-1, ..., a-p       (FIR, data type)
    A c[kMaxK];                          // b-1, ..., b-k           (recurrence)
    T cT[kMaxK];                         // b-1, ..., b-k in the data type (seeded phase B of the DECAY kernel)
    T H[kMaxX][kMaxK];                   // H[u][r] = h^(r+1)_u = T(u+1)[0][r], u < X
    A Twarp[5][kMaxK * kMaxK];           // T(X * 2^s)          lane scan
    A Tblk[4][kMaxK * kMaxK];            // T(32 X * 2^s)       warp-aggregate scan
    A Twin[kMaxW][kMaxK * kMaxK];        // T(32 X * w)         warp carry-in
    A Tm[kMaxK * kMaxK];                 // T(m)                inclusive = agg + T(m) G
    A Tpow[9][kMaxK * kMaxK];            // T(U * 2^s), s <= 8  look-back folds and skips (unit U = G m)
    A Tsub[kMaxG][kMaxK * kMaxK];        // T(g m), g < G       tile carries inside a unit
};

template <typename T, typename A>
struct ScanParams {
    const T* x;
    T* y;
    uint64_t n;
    uint64_t ntiles;
    unsigned long long* ticket;          // [0] counter, [1] launch base, [2] epoch (launch_state_advance)
    unsigned long long* status;          // 2^c scattered records of {tag:32 | value:32} words
    uint32_t status_mask;                // 2^c - 1, 2^c >= ntiles
    int decay;                           // T(m) == 0 exactly: inclusive == aggregate
    uint32_t dec_mask;                   // DECAY kernels: bit s < 5 = lane-scan step s has a non-negligible
                                         // T(X 2^s); bit 5 = warp-aggregate level (T(32X d), d >= 1) non-negligible
    const T* x_hist;                     // p values x_{-p}..x_{-1} or null
    const T* y_hist;                     // k values y_{-k}..y_{-1} or null
    T* y_tail;                           // k slots y_{n-k}..y_{n-1} or null
    const A* lane_T;                     // [k*k][32]: T(X*l) per lane
    unsigned long long* stats;           // debug counters (PLR_STATS=1) or null
    Tables<T, A> tab;
    int lag;                             // re-read kernel, PLR_RR_RUNTIME_LAG builds: phase-B lag in tiles (0: NS-1)
};

// Host-side planner result.
struct PlanTables {
    int p, k;
    plr_dtype dtype;
    plr_class cls;
    Geometry geo;
    int64_t decay_len;
    int64_t fixup_len;
    int decay_flag;
    int acc64;                           // float: accumulate recurrence + carries in fp64
    uint32_t dec_mask;                   // ScanParams::dec_mask of the tables the plan launches with
    double cond_bound;                   // eps32 * sum|a| * (sum|g|)^2 / min(1, |H(-1)|) (float, R16)
    double map_floor;                    // eps32 * sum|a| * sum|g| / min(1, |H(-1)|) (float, R20)
    double nyquist_gain;                 // |H(-1)| = |A(-1)| / |B(-1)| (float)
    int sig_id;                          // compile-time signature kernel (plr_constsig.cuh), 0 = none
    Tables<uint32_t, uint32_t> ti;       // int32 ring
    Tables<float, float> tf;             // fp32, fp32 accumulation
    Tables<float, double> td;            // fp32, fp64 accumulation
    Tables<uint32_t, uint32_t> ti1;      // ti / td with look-back units of one tile (Tpow = T(m 2^s))
    Tables<float, double> td1;
    // small-n kernel (plr_kernels_small.cuh): its own tile geometry geo_s
    Geometry geo_s;
    Tables<uint32_t, uint32_t> tis;
    Tables<float, float> tfs;
    Tables<float, double> tds;
    uint32_t lane_is[kMaxK * kMaxK * 32];
    float lane_fs[kMaxK * kMaxK * 32];
    double lane_ds[kMaxK * kMaxK * 32];
    uint32_t dec_mask_s;                 // ScanParams::dec_mask of the small-n tables
    Tables<uint32_t, uint32_t> tr;       // reduce-only kernel tables (its own tile geometry)
    Tables<float, double> trd;
    int decay_s;                         // T(m_s) == 0 exactly (one-hop look-back)
    uint32_t lane_i[kMaxK * kMaxK * 32];
    float lane_f[kMaxK * kMaxK * 32];
    double lane_d[kMaxK * kMaxK * 32];
    // coefficients as the combine / fixup use them
    double a_d[kMaxP + 1], b_d[kMaxK];
    uint32_t a_u[kMaxP + 1], b_u[kMaxK];
    // DECAY fixup: F[i][slot] = response of y_i to a unit in augmented slot
    // (x_{-4..-1}, y_{-4..-1}) with zero input, i < fixup_len (fp32)
    float* fix_table;                    // host, fixup_len * kAug (owned)
};

// small-n kernel geometry: X = 15 elements per thread, W = 8 warps, m = 3840
#ifndef PLR_SMALL_X
#define PLR_SMALL_X 15
#endif
#ifndef PLR_SMALL_W
#define PLR_SMALL_W 8
#endif
constexpr int kSmallX = PLR_SMALL_X;
constexpr int kSmallW = PLR_SMALL_W;
// small-n cluster launches (non-decaying, forward, every tile resident):
// clusters of kSmallC tiles exchange aggregates over DSMEM, the look-back
// runs over cluster records (plr_kernels_small.cuh)
#ifndef PLR_SMALL_C
#define PLR_SMALL_C 4
#endif
constexpr int kSmallC = PLR_SMALL_C;
// reduce-only kernel geometry (plr_kernels_reduce.cuh): X = 31, W = 8
// (tile 7936), 3-stage TMA ring, 2 CTAs per SM
constexpr int kRedX = 31;
constexpr int kRedW = 8;
constexpr int kRedS = 3;
constexpr int kRedMaxGrid = 1024;   // reduce-only grid cap (the last CTA copies every CTA record to smem)

// planner (host, plr_planner.cpp)
plr_status plan_tables(const double* a, int p, const double* b, int k, plr_dtype dtype,
                       Geometry geo, PlanTables* out, const char** why);
void plan_tables_free(PlanTables* pt);
void factor_lists(const PlanTables& pt, int64_t m, void* out);

// 8x8 augmented companion matrix of Eq. (1) for the free evolution
// (zero input) of the state (x_{-4..-1}, y_{-4..-1}); used by the combine.
template <typename R>
void aug_companion(const R* alpha, int p, const R* c, int k, R* M8) {
    for (int i = 0; i < kAug * kAug; i++) M8[i] = R(0);
    for (int i = 0; i < 3; i++) M8[i * kAug + (i + 1)] = R(1);        // x shift, x_{-1}' = 0
    for (int i = 4; i < 7; i++) M8[i * kAug + (i + 1)] = R(1);        // y shift
    for (int j = 1; j <= p; j++) M8[7 * kAug + (4 - j)] = alpha[j];   // y_new += a_{-j} x_{-j}
    for (int j = 1; j <= k; j++) M8[7 * kAug + (8 - j)] = c[j - 1];   // y_new += b_{-j} y_{-j}
}

}  // namespace plr
