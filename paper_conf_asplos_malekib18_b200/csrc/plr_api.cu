// plr_api.cu -- the C ABI (include/plr.h): plans, launches, the sharded path
// (one NCCL allgather), the host-memory pipeline, and small helper kernels.
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>
#include <cmath>

#include "plr_internal.h"
#include "plr_launch.h"

using namespace plr;

// ============================================================ errors ======
static thread_local std::string g_last_error;

static plr_status fail(plr_status s, const std::string& msg) {
    g_last_error = msg;
    return s;
}
static plr_status cuda_fail(cudaError_t e, const char* what) {
    return fail(e == cudaErrorMemoryAllocation ? PLR_ERR_OOM : PLR_ERR_CUDA,
                std::string(what) + ": " + cudaGetErrorString(e));
}
#define CUDA_TRY(expr, what)                        \
    do {                                            \
        cudaError_t e_ = (expr);                    \
        if (e_ != cudaSuccess) return cuda_fail(e_, what); \
    } while (0)

// ============================================================ the plan ====
struct plr_plan {
    PlanTables pt;
    int device = 0;
    int num_sms = 0;
    int ctas_per_sm = 0;
    size_t n_max = 0;
    uint64_t max_tiles = 0;
    uint64_t status_slots = 0;              // power of two >= max_tiles (persistent kernels' tiles)
    uint64_t status_slots_s = 0;            // the small-n kernel's own status array (its tiles)
    unsigned long long* d_status_s = nullptr;
    unsigned long long* d_ticket = nullptr;
    unsigned long long* d_status = nullptr;
    uint32_t epoch = 0;                 // host count of launches since the last reset (overflow guard)
    void* d_lane = nullptr;
    void* d_lane_s = nullptr;           // lane table T(X_s l) of the small-n kernel
    size_t small_max = 0;               // n <= small_max: the small-n kernel (plr_kernels_small.cuh)
    int small_ctas = 0;                 // its CTAs per SM (all tiles resident: tile = blockIdx.x)
    int small_clusters = 0;             // co-resident clusters of kSmallC small-n CTAs (0: no cluster launches)
    bool cluster_ok = true;             // PLR_SMALL_CLUSTER != 0 at plan creation
    int rr_lag = 0;                     // PLR_RR_LAG at plan creation (0: the re-read kernel's NS-1)
    int reduce_ctas = 0;                // CTAs per SM of the reduce-only kernel (0: not available)
    unsigned long long* d_rd = nullptr; // its per-CTA records (kStatusMaxBytes each)
    void* d_scan_tmp = nullptr;         // CUB temp storage of the Scan comparator
    size_t scan_tmp_bytes = 0;
    float* d_fix = nullptr;
    bool dirty = false;
    bool sig_kernel = false;            // launch the compile-time signature kernel (pt.sig_id)
    unsigned long long* d_stats = nullptr;   // look-back counters when PLR_STATS=1
    // sharded path scratch
    unsigned char* d_send = nullptr;
    unsigned char* d_recv = nullptr;
    int recv_world = 0;
    uint32_t* d_hist = nullptr;
    // host pipeline scratch
    void* h_dx[3] = {nullptr, nullptr, nullptr};
    void* h_dy[3] = {nullptr, nullptr, nullptr};
    size_t h_chunk = 0;
    cudaStream_t s_in = nullptr, s_out = nullptr;
    cudaEvent_t ev_in[3] = {}, ev_comp[3] = {}, ev_out[3] = {};
};

static size_t elem_size(const plr_plan*) { return 4; }

// ticket counter, launch base, epoch: the launch state lives on the device
// (launch_state_advance), so plr_execute can be captured in a CUDA graph
static constexpr size_t kTicketBytes = 3 * sizeof(unsigned long long);

static bool aligned16(const void* p) { return ((uintptr_t)p & 15u) == 0; }

// Small-n launches use look-back units of one tile while the big-unit grid
// would give each CTA fewer than one unit (tail imbalance);
// PLR_UNIT1_WAVES overrides it (0: never) for size sweeps.
static uint64_t unit1_waves() {
    const char* e = std::getenv("PLR_UNIT1_WAVES");
    return e != nullptr ? (uint64_t)std::strtoull(e, nullptr, 10) : (uint64_t)1;
}

// Sizes up to this many elements run the small-n kernel (one CTA per tile,
// no pipeline).  Measured crossover against the
// persistent kernels (profiles/r03e_sweep_auto.md vs r03c_sweep_big.md):
// 2^21 for DECAY and first-order plans (single-hop / scalar look-back), 2^17
// for k >= 2 non-decaying plans with the per-tile look-back (its reads of
// every predecessor cost more than the persistent kernels' units beyond
// that); with cluster launches (§6) the k >= 2 crossover is 2^20 or the
// largest all-resident cluster launch if smaller (r03s: order3 at 2^20 15.3
// us against 18.3 us on the re-read kernel, tuple2 14.8 / 15.1).
// PLR_SMALL_MAX overrides it at plan creation (0: never).
static size_t small_max_default(const PlanTables& pt, int small_clusters) {
    const char* e = std::getenv("PLR_SMALL_MAX");
    if (e != nullptr) return (size_t)std::strtoull(e, nullptr, 10);
    if (pt.decay_flag || pt.k == 1) return (size_t)1 << 21;
    const size_t cl = (size_t)small_clusters * kSmallC * (size_t)pt.geo_s.tile();
    return small_clusters > 0 ? std::max(std::min(cl, (size_t)1 << 20), (size_t)1 << 17) : ((size_t)1 << 17);
}

// ============================================================ helpers =====
namespace {

// payload: u64 n | u32 x_tail[4] | u32 y_tail[4] | pad
__global__ void payload_kernel(const uint32_t* x, const uint32_t* y, unsigned long long n,
                               unsigned char* payload, int write_y) {
    const int t = threadIdx.x;
    uint32_t* w = reinterpret_cast<uint32_t*>(payload + 8);
    if (t == 0) *reinterpret_cast<unsigned long long*>(payload) = n;
    if (t < 4) {
        const long long i = (long long)n - 4 + t;
        w[t] = (i >= 0) ? x[i] : 0u;
        if (write_y) w[4 + t] = (i >= 0) ? y[i] : 0u;
    }
}

// Ring arithmetic for the combine: Z/2^32 (uint32) or fp64.
template <typename R> __host__ __device__ inline R from_word(uint32_t w);
template <> __host__ __device__ inline uint32_t from_word<uint32_t>(uint32_t w) { return w; }
template <> __host__ __device__ inline double from_word<double>(uint32_t w) {
    float f;
    memcpy(&f, &w, 4);
    return (double)f;
}
template <typename R> __host__ __device__ inline uint32_t to_word(R v);
template <> __host__ __device__ inline uint32_t to_word<uint32_t>(uint32_t v) { return v; }
template <> __host__ __device__ inline uint32_t to_word<double>(double v) {
    float f = (float)v;
    uint32_t w;
    memcpy(&w, &f, 4);
    return w;
}

template <typename R>
struct AugMat { R v[kAug * kAug]; };

// z_{r+1} = M^{n_r} z_r + payload_r, z_0 = 0; hist = z_rank (host version).
template <typename R>
void combine_host_impl(const AugMat<R>& M, const unsigned char* payloads, int rank, uint32_t* hist) {
    AugMat<R> P2[64];
    P2[0] = M;
    int maxbit = 0;
    for (int r = 0; r < rank; r++) {
        unsigned long long nr;
        memcpy(&nr, payloads + (size_t)r * PLR_PAYLOAD_BYTES, 8);
        while (maxbit < 63 && (nr >> (maxbit + 1))) maxbit++;
    }
    for (int i = 1; i <= maxbit; i++)
        for (int a = 0; a < kAug; a++)
            for (int b = 0; b < kAug; b++) {
                R acc = R(0);
                for (int t = 0; t < kAug; t++) acc += P2[i - 1].v[a * kAug + t] * P2[i - 1].v[t * kAug + b];
                P2[i].v[a * kAug + b] = acc;
            }
    R z[kAug];
    for (int a = 0; a < kAug; a++) z[a] = R(0);
    for (int r = 0; r < rank; r++) {
        const unsigned char* pl = payloads + (size_t)r * PLR_PAYLOAD_BYTES;
        unsigned long long nr;
        memcpy(&nr, pl, 8);
        for (int i = 0; i < 64; i++)
            if ((nr >> i) & 1ull) {
                R t[kAug];
                for (int a = 0; a < kAug; a++) {
                    R acc = R(0);
                    for (int b = 0; b < kAug; b++) acc += P2[i].v[a * kAug + b] * z[b];
                    t[a] = acc;
                }
                for (int a = 0; a < kAug; a++) z[a] = t[a];
            }
        uint32_t w[kAug];
        memcpy(w, pl + 8, sizeof(w));
        for (int a = 0; a < kAug; a++) z[a] += from_word<R>(w[a]);
    }
    for (int a = 0; a < kAug; a++) hist[a] = to_word<R>(z[a]);
}

// Device version: one warp; lanes square the 8x8 matrix in parallel.
template <typename R>
__global__ void combine_kernel(AugMat<R> M, const unsigned char* payloads, int rank, uint32_t* hist) {
    __shared__ R P2[64][kAug * kAug];
    __shared__ R z[kAug];
    const int lane = threadIdx.x;
    for (int e = lane; e < kAug * kAug; e += 32) P2[0][e] = M.v[e];
    int maxbit = 0;
    for (int r = 0; r < rank; r++) {
        const unsigned long long nr = *reinterpret_cast<const unsigned long long*>(payloads + (size_t)r * PLR_PAYLOAD_BYTES);
        while (maxbit < 63 && (nr >> (maxbit + 1))) maxbit++;
    }
    __syncwarp();
    for (int i = 1; i <= maxbit; i++) {
        for (int e = lane; e < kAug * kAug; e += 32) {
            const int a = e / kAug, b = e % kAug;
            R acc = R(0);
            for (int t = 0; t < kAug; t++) acc += P2[i - 1][a * kAug + t] * P2[i - 1][t * kAug + b];
            P2[i][e] = acc;
        }
        __syncwarp();
    }
    if (lane < kAug) z[lane] = R(0);
    __syncwarp();
    for (int r = 0; r < rank; r++) {
        const unsigned char* pl = payloads + (size_t)r * PLR_PAYLOAD_BYTES;
        const unsigned long long nr = *reinterpret_cast<const unsigned long long*>(pl);
        for (int i = 0; i < 64; i++) {
            if (!((nr >> i) & 1ull)) continue;
            R acc = R(0);
            if (lane < kAug)
                for (int b = 0; b < kAug; b++) acc += P2[i][lane * kAug + b] * z[b];
            __syncwarp();
            if (lane < kAug) z[lane] = acc;
            __syncwarp();
        }
        if (lane < kAug) z[lane] += from_word<R>(reinterpret_cast<const uint32_t*>(pl + 8)[lane]);
        __syncwarp();
    }
    if (lane < kAug) hist[lane] = to_word<R>(z[lane]);
}

// DECAY fixup: y_i += sum_s F[i][s] * hist[s], i < len.
__global__ void fixup_kernel(float* y, unsigned long long len, const float* F, const uint32_t* hist) {
    const unsigned long long i = blockIdx.x * (unsigned long long)blockDim.x + threadIdx.x;
    if (i >= len) return;
    float acc = y[i];
#pragma unroll
    for (int s = 0; s < kAug; s++) acc = __fmaf_rn(F[i * kAug + s], __uint_as_float(hist[s]), acc);
    y[i] = acc;
}

template <typename R>
AugMat<R> aug_matrix(const PlanTables& pt) {
    AugMat<R> M;
    R al[kMaxP + 1] = {}, c[kMaxK] = {};
    for (int j = 0; j <= pt.p; j++) al[j] = std::is_same<R, double>::value ? (R)pt.a_d[j] : (R)pt.a_u[j];
    for (int j = 0; j < pt.k; j++) c[j] = std::is_same<R, double>::value ? (R)pt.b_d[j] : (R)pt.b_u[j];
    aug_companion<R>(al, pt.p, c, pt.k, M.v);
    return M;
}

}  // namespace

// ============================================================ launches ====
static plr_status launch(plr_plan* plan, const void* x, void* y, size_t n, const void* x_hist,
                         const void* y_hist, void* y_tail, bool store, cudaStream_t stream, bool reverse = false) {
    if (n == 0) return PLR_OK;
    if (n > plan->n_max) return fail(PLR_ERR_SIZE, "n exceeds the plan's n_max");
    if (plan->dirty || plan->epoch >= 0x7ffffff0u) {
        CUDA_TRY(cudaMemsetAsync(plan->d_status, 0, plan->status_slots * kStatusMaxBytes, stream), "status reset");
        CUDA_TRY(cudaMemsetAsync(plan->d_status_s, 0, plan->status_slots_s * kStatusMaxBytes, stream), "status reset");
        CUDA_TRY(cudaMemsetAsync(plan->d_ticket, 0, kTicketBytes, stream), "ticket reset");
        plan->epoch = 0;
        plan->dirty = false;
    }
    // small n: one CTA per tile, no pipeline (the anticausal pass too; beyond
    // small_max it runs the REV instantiation of the plan's persistent kernel)
    if (n <= plan->small_max) {
        const uint64_t ms = (uint64_t)plan->pt.geo_s.tile();
        plan->epoch++;
        LaunchArgs la;
        la.x = x; la.y = store ? y : nullptr; la.n = n; la.ntiles = (n + ms - 1) / ms;
        la.ticket = plan->d_ticket;
        la.status = plan->d_status_s;
        la.status_mask = plan->status_slots_s - 1;
        la.decay = plan->pt.decay_s;
        la.dec_mask = plan->pt.dec_mask_s;
        // every tile resident at once (one wave): tile index = blockIdx.x, no
        // ticket before the load (PLR_SMALL_RESIDENT=0 turns it off)
        static const bool resident_ok = [] {
            const char* e = std::getenv("PLR_SMALL_RESIDENT");
            return e == nullptr || e[0] != '0';
        }();
        if (resident_ok && la.ntiles <= (uint64_t)plan->num_sms * plan->small_ctas) la.dec_mask |= 0x100u;
        // non-decaying forward launches of several tiles whose clusters are
        // all co-resident: the cluster look-back (PLR_SMALL_CLUSTER=0 turns it off)
        if (plan->cluster_ok && resident_ok && !reverse && !plan->pt.decay_s && la.ntiles >= 2 &&
            (la.ntiles + kSmallC - 1) / kSmallC <= (uint64_t)plan->small_clusters) {
            la.cluster = true;
            la.dec_mask |= 0x100u;
        }
        la.x_hist = x_hist; la.y_hist = y_hist; la.y_tail = y_tail;
        la.lane_T = plan->d_lane_s;
        la.stats = plan->d_stats;
        la.grid = (int)la.ntiles;
        la.store = store;
        la.reverse = reverse;
        la.stream = stream;
        cudaError_t e = launch_small(plan->pt, la);
        if (e != cudaSuccess) {
            plan->dirty = true;
            return cuda_fail(e, "small-n kernel launch");
        }
        return PLR_OK;
    }
    const uint64_t m = (uint64_t)plan->pt.geo.tile();
    const uint64_t ntiles = (n + m - 1) / m;
    // tiles per ticket (look-back unit).  Small n: units of one tile, so the
    // tiles spread over every SM (a unit of G tiles runs on one CTA);
    // DECAY plans always have G = 1.
    const uint64_t grid_max = (uint64_t)plan->num_sms * plan->ctas_per_sm;
    const bool unit1 = plan->pt.geo.G > 1 && ntiles < unit1_waves() * grid_max * (uint64_t)plan->pt.geo.G;
    const uint64_t G = unit1 ? 1 : (uint64_t)plan->pt.geo.G;
    const uint64_t nunits = (ntiles + G - 1) / G;
    plan->epoch++;
    const uint64_t grid = std::min<uint64_t>(nunits, grid_max);
    LaunchArgs la;
    la.x = x; la.y = y; la.n = n; la.ntiles = ntiles;
    la.ticket = plan->d_ticket;
    la.status = plan->d_status;
    la.status_mask = plan->status_slots - 1;
    la.decay = plan->pt.decay_flag;
    la.dec_mask = plan->pt.dec_mask;
    la.x_hist = x_hist; la.y_hist = y_hist; la.y_tail = y_tail;
    la.lane_T = plan->d_lane;
    la.stats = plan->d_stats;
    la.grid = (int)grid;
    la.sig = plan->sig_kernel ? plan->pt.sig_id : 0;
    la.store = store;
    la.unit1 = unit1;
    la.reverse = reverse;
    la.lag = plan->rr_lag;
    la.stream = stream;
    cudaError_t e = launch_scan(plan->pt, la);
    if (e != cudaSuccess) {
        plan->dirty = true;
        return cuda_fail(e, "scan kernel launch");
    }
    return PLR_OK;
}

static plr_status check_xy(const plr_plan* plan, const void* x, const void* y, size_t n, bool need_y) {
    if (plan == nullptr) return fail(PLR_ERR_INVALID_ARG, "null plan");
    if (n == 0) return PLR_OK;
    if (x == nullptr || (need_y && y == nullptr)) return fail(PLR_ERR_INVALID_ARG, "null data pointer");
    if (!aligned16(x) || (need_y && !aligned16(y))) return fail(PLR_ERR_MISALIGNED, "x and y must be 16-byte aligned");
    if (need_y) {
        const uintptr_t xa = (uintptr_t)x, ya = (uintptr_t)y, nb = n * elem_size(plan);
        const bool overlap = xa < ya + nb && ya < xa + nb;
        if (overlap && !(xa == ya && plan->pt.p == 0))
            return fail(PLR_ERR_ALIAS, "x and y overlap (allowed only x == y with p == 0)");
    }
    return PLR_OK;
}

// ============================================================ ABI =========
extern "C" {

int plr_abi_version(void) { return PLR_ABI_VERSION; }

const char* plr_last_error(void) { return g_last_error.c_str(); }

const char* plr_status_string(plr_status s) {
    switch (s) {
        case PLR_OK: return "PLR_OK";
        case PLR_ERR_INVALID_ARG: return "PLR_ERR_INVALID_ARG";
        case PLR_ERR_SIGNATURE: return "PLR_ERR_SIGNATURE";
        case PLR_ERR_DTYPE: return "PLR_ERR_DTYPE";
        case PLR_ERR_SIZE: return "PLR_ERR_SIZE";
        case PLR_ERR_ALIAS: return "PLR_ERR_ALIAS";
        case PLR_ERR_MISALIGNED: return "PLR_ERR_MISALIGNED";
        case PLR_ERR_CUDA: return "PLR_ERR_CUDA";
        case PLR_ERR_NCCL: return "PLR_ERR_NCCL";
        case PLR_ERR_OOM: return "PLR_ERR_OOM";
    }
    return "PLR_ERR_UNKNOWN";
}

plr_status plr_plan_destroy(plr_plan* plan) {
    if (plan == nullptr) return PLR_OK;
    cudaFree(plan->d_ticket);
    cudaFree(plan->d_status);
    cudaFree(plan->d_status_s);
    cudaFree(plan->d_lane);
    cudaFree(plan->d_lane_s);
    cudaFree(plan->d_rd);
    cudaFree(plan->d_scan_tmp);
    cudaFree(plan->d_fix);
    cudaFree(plan->d_send);
    cudaFree(plan->d_recv);
    cudaFree(plan->d_hist);
    cudaFree(plan->d_stats);
    for (int i = 0; i < 3; i++) {
        cudaFree(plan->h_dx[i]);
        cudaFree(plan->h_dy[i]);
        if (plan->ev_in[i]) cudaEventDestroy(plan->ev_in[i]);
        if (plan->ev_comp[i]) cudaEventDestroy(plan->ev_comp[i]);
        if (plan->ev_out[i]) cudaEventDestroy(plan->ev_out[i]);
    }
    if (plan->s_in) cudaStreamDestroy(plan->s_in);
    if (plan->s_out) cudaStreamDestroy(plan->s_out);
    plan_tables_free(&plan->pt);
    delete plan;
    return PLR_OK;
}

plr_status plr_plan_create(plr_plan** out, const double* a, int p, const double* b, int k,
                           plr_dtype dtype, size_t n_max) {
    if (out == nullptr) return fail(PLR_ERR_INVALID_ARG, "null out");
    *out = nullptr;
    plr_plan* plan = new plr_plan();
    const char* why = "";
    // plan with the DECAY geometry; non-decaying plans are re-planned with
    // the generic kernel's geometry (the class is known after planning)
    plr_status st = plan_tables(a, p, b, k, dtype, class_geometry(true, k), &plan->pt, &why);
    // ablation (Fig. 10 analogue): PLR_FORCE_GENERIC=1 disables
    // the DECAY specialisation (single-hop look-back) for this plan
    const char* fg = std::getenv("PLR_FORCE_GENERIC");
    const bool force_generic = fg != nullptr && fg[0] == '1';
    if (st == PLR_OK && plan->pt.decay_flag && plan->pt.acc64 && !force_generic) {
        // fp64-accumulation DECAY plans use their own tile geometry
        plan_tables_free(&plan->pt);
        st = plan_tables(a, p, b, k, dtype, class_geometry(true, k, true), &plan->pt, &why);
    }
    if (st == PLR_OK && (!plan->pt.decay_flag || force_generic)) {
        plan_tables_free(&plan->pt);
        st = plan_tables(a, p, b, k, dtype, class_geometry(false, k), &plan->pt, &why);
        if (st == PLR_OK && force_generic) {
            plan->pt.decay_flag = 0;
            plan->pt.decay_s = 0;                              // the small-n kernel's one-hop look-back too
            plan->pt.acc64 = dtype == PLR_FLOAT32 ? 1 : 0;   // generic float kernels accumulate in fp64
        }
    }
    if (st != PLR_OK) {
        delete plan;
        return fail(st, why);
    }
    // compile-time signature kernels (plr_constsig.cuh) unless the ablation
    // switches are set: PLR_FORCE_GENERIC=1 (all specialisations off) or
    // PLR_NO_CONSTSIG=1 (tables from kernel parameters only)
    const char* ncs = std::getenv("PLR_NO_CONSTSIG");
    plan->sig_kernel = !force_generic && !(ncs != nullptr && ncs[0] == '1') && plan->pt.sig_id != 0;
    plan->n_max = n_max;
    if (n_max == 0) {                      // host-only plan: planner tables, no device state
        *out = plan;
        return PLR_OK;
    }
    auto bail = [&](cudaError_t e, const char* what) {
        plr_status s = cuda_fail(e, what);
        std::string keep = g_last_error;
        plr_plan_destroy(plan);
        g_last_error = keep;
        return s;
    };
    cudaError_t e;
    if ((e = cudaGetDevice(&plan->device)) != cudaSuccess) return bail(e, "cudaGetDevice");
    if ((e = cudaDeviceGetAttribute(&plan->num_sms, cudaDevAttrMultiProcessorCount, plan->device)) != cudaSuccess)
        return bail(e, "SM count");
    if ((e = scan_occupancy(plan->pt, &plan->ctas_per_sm)) != cudaSuccess) return bail(e, "occupancy");
    if (plan->ctas_per_sm < 1) { plr_plan_destroy(plan); return fail(PLR_ERR_CUDA, "kernel does not fit on an SM"); }
    int small_ctas = 0;
    if ((e = small_occupancy(plan->pt, &small_ctas)) != cudaSuccess) return bail(e, "occupancy (small-n)");
    if (plan->pt.dtype == PLR_INT32 || plan->pt.acc64) {     // non-DECAY capable: the reduce-only kernel
        if ((e = reduce_occupancy(plan->pt, &plan->reduce_ctas)) != cudaSuccess) return bail(e, "occupancy (reduce)");
        if (plan->reduce_ctas > 0) {
            const size_t rb = (size_t)plan->num_sms * plan->reduce_ctas * kStatusMaxBytes;
            if ((e = cudaMalloc(&plan->d_rd, rb)) != cudaSuccess) return bail(e, "alloc reduce records");
        }
    }
    plan->small_ctas = small_ctas;
    // experiment switches, read once per plan: PLR_SMALL_CLUSTER=0 (no
    // cluster launches), PLR_RR_LAG (the re-read kernel's phase-B lag)
    if (const char* ce = std::getenv("PLR_SMALL_CLUSTER")) plan->cluster_ok = ce[0] != '0';
    if (const char* lg = std::getenv("PLR_RR_LAG")) plan->rr_lag = std::atoi(lg);
    if (!plan->pt.decay_s && small_ctas >= 1) {
        if ((e = small_cluster_occupancy(plan->pt, &plan->small_clusters)) != cudaSuccess) {
            (void)cudaGetLastError();                          // no cluster launches on this device
            plan->small_clusters = 0;
            if (std::getenv("PLR_DEBUG") != nullptr)
                std::fprintf(stderr, "plr: cluster occupancy query failed: %s\n", cudaGetErrorString(e));
        }
    }
    plan->small_max = small_ctas >= 1 ? std::min(n_max, small_max_default(plan->pt, plan->cluster_ok ? plan->small_clusters : 0)) : 0;
    const uint64_t m = (uint64_t)plan->pt.geo.tile(), ms = (uint64_t)plan->pt.geo_s.tile();
    plan->max_tiles = std::max<uint64_t>(1, (n_max + m - 1) / m);
    // Two status arrays: the persistent kernels' (their tiles up to n_max)
    // and the small-n kernel's (its tiles up to small_max).
    // One shared array sized for the small tiles doubled the persistent
    // kernels' and cost their forward pass ~3 % at 2^30 (r03e/r03f A/B).
    const uint64_t small_tiles = std::max<uint64_t>(1, (plan->small_max + ms - 1) / ms);
    if (plan->max_tiles > (1ull << 31) || small_tiles > (1ull << 31)) {
        plr_plan_destroy(plan);
        return fail(PLR_ERR_SIZE, "n_max too large");
    }
    plan->status_slots = 1;
    while (plan->status_slots < plan->max_tiles) plan->status_slots <<= 1;
    plan->status_slots_s = 1;
    while (plan->status_slots_s < small_tiles) plan->status_slots_s <<= 1;
    if ((e = cudaMalloc(&plan->d_ticket, kTicketBytes)) != cudaSuccess) return bail(e, "alloc ticket");
    if ((e = cudaMalloc(&plan->d_status, plan->status_slots * kStatusMaxBytes)) != cudaSuccess) return bail(e, "alloc status");
    if ((e = cudaMalloc(&plan->d_status_s, plan->status_slots_s * kStatusMaxBytes)) != cudaSuccess) return bail(e, "alloc status");
    if ((e = cudaMemset(plan->d_ticket, 0, kTicketBytes)) != cudaSuccess) return bail(e, "memset");
    if ((e = cudaMemset(plan->d_status, 0, plan->status_slots * kStatusMaxBytes)) != cudaSuccess) return bail(e, "memset");
    if ((e = cudaMemset(plan->d_status_s, 0, plan->status_slots_s * kStatusMaxBytes)) != cudaSuccess) return bail(e, "memset");
    const bool acc64 = dtype == PLR_FLOAT32 && plan->pt.acc64;
    const size_t lane_bytes = (size_t)k * k * 32 * (acc64 ? 8 : 4);
    if ((e = cudaMalloc(&plan->d_lane, lane_bytes)) != cudaSuccess) return bail(e, "alloc lane table");
    const void* lane_src = dtype == PLR_INT32 ? (const void*)plan->pt.lane_i
                         : acc64 ? (const void*)plan->pt.lane_d : (const void*)plan->pt.lane_f;
    if ((e = cudaMemcpy(plan->d_lane, lane_src, lane_bytes, cudaMemcpyHostToDevice)) != cudaSuccess) return bail(e, "copy lane table");
    if ((e = cudaMalloc(&plan->d_lane_s, lane_bytes)) != cudaSuccess) return bail(e, "alloc lane table");
    const void* lane_s = dtype == PLR_INT32 ? (const void*)plan->pt.lane_is
                       : acc64 ? (const void*)plan->pt.lane_ds : (const void*)plan->pt.lane_fs;
    if ((e = cudaMemcpy(plan->d_lane_s, lane_s, lane_bytes, cudaMemcpyHostToDevice)) != cudaSuccess) return bail(e, "copy lane table");
    if (plan->pt.cls == PLR_CLASS_DECAY && plan->pt.fixup_len > 0) {
        const size_t fb = (size_t)plan->pt.fixup_len * kAug * 4;
        if ((e = cudaMalloc(&plan->d_fix, fb)) != cudaSuccess) return bail(e, "alloc fixup table");
        if ((e = cudaMemcpy(plan->d_fix, plan->pt.fix_table, fb, cudaMemcpyHostToDevice)) != cudaSuccess) return bail(e, "copy fixup table");
    }
    if ((e = cudaMalloc(&plan->d_hist, 64)) != cudaSuccess) return bail(e, "alloc hist");
    const char* st_env = std::getenv("PLR_STATS");
    if (st_env != nullptr && st_env[0] == '1') {
        if ((e = cudaMalloc(&plan->d_stats, 128)) != cudaSuccess) return bail(e, "alloc stats");
        if ((e = cudaMemset(plan->d_stats, 0, 128)) != cudaSuccess) return bail(e, "memset stats");
    }
    if ((e = cudaMemset(plan->d_hist, 0, 64)) != cudaSuccess) return bail(e, "memset hist");
    *out = plan;
    return PLR_OK;
}

plr_status plr_plan_create_cascade(plr_plan** out, int nstages, const double* a, const int* p, const double* b,
                                   const int* k, plr_dtype dtype, size_t n_max) {
    if (out == nullptr) return fail(PLR_ERR_INVALID_ARG, "null out");
    *out = nullptr;
    if (nstages < 1 || a == nullptr || p == nullptr || k == nullptr) return fail(PLR_ERR_INVALID_ARG, "bad stage list");
    if (dtype != PLR_INT32 && dtype != PLR_FLOAT32) return fail(PLR_ERR_DTYPE, "dtype must be PLR_INT32 or PLR_FLOAT32");
    // numerator N(z) and denominator D(z) = 1 - sum_j b_j z^-j, multiplied
    // stage by stage: Z/2^32 (uint64 wrapped) or fp64
    constexpr int kCap = 64;
    std::vector<uint64_t> Nu(1, 1), Du(1, 1);
    std::vector<double> Nd(1, 1.0), Dd(1, 1.0);
    const double* ap = a;
    const double* bp = b;
    for (int s = 0; s < nstages; s++) {
        const int ps = p[s], ks = k[s];
        if (ps < 0 || ks < 0 || ps >= kCap || ks >= kCap) return fail(PLR_ERR_SIGNATURE, "bad stage order");
        if (ks > 0 && bp == nullptr) return fail(PLR_ERR_INVALID_ARG, "null b");
        for (int j = 0; j <= ps; j++)
            if (!std::isfinite(ap[j])) return fail(PLR_ERR_SIGNATURE, "non-finite coefficient");
        for (int j = 0; j < ks; j++)
            if (!std::isfinite(bp[j])) return fail(PLR_ERR_SIGNATURE, "non-finite coefficient");
        if (ap[ps] == 0.0 || (ks > 0 && bp[ks - 1] == 0.0))
            return fail(PLR_ERR_SIGNATURE, "a stage's last coefficient must not be zero (P:635-637)");
        std::vector<uint64_t> nu(Nu.size() + ps, 0), du(Du.size() + ks, 0);
        std::vector<double> nd(Nd.size() + ps, 0.0), dd(Dd.size() + ks, 0.0);
        for (int j = 0; j <= ps; j++) {
            const double v = ap[j];
            if (dtype == PLR_INT32 && (v != std::floor(v) || std::fabs(v) >= 9.0e15))
                return fail(PLR_ERR_SIGNATURE, "PLR_INT32 needs integer coefficients");
            const uint64_t vu = (uint64_t)(int64_t)v;
            const double vd = (double)(float)v;
            for (size_t i = 0; i < Nu.size(); i++) { nu[i + j] += Nu[i] * vu; nd[i + j] += Nd[i] * vd; }
        }
        for (int j = 0; j <= ks; j++) {
            const double v = j == 0 ? 1.0 : -bp[j - 1];
            if (dtype == PLR_INT32 && (v != std::floor(v) || std::fabs(v) >= 9.0e15))
                return fail(PLR_ERR_SIGNATURE, "PLR_INT32 needs integer coefficients");
            const uint64_t vu = (uint64_t)(int64_t)v;
            const double vd = j == 0 ? 1.0 : -(double)(float)bp[j - 1];
            for (size_t i = 0; i < Du.size(); i++) { du[i + j] += Du[i] * vu; dd[i + j] += Dd[i] * vd; }
        }
        for (auto& e : nu) e &= 0xffffffffull;
        for (auto& e : du) e &= 0xffffffffull;
        Nu.swap(nu); Du.swap(du); Nd.swap(nd); Dd.swap(dd);
        ap += ps + 1;
        bp += ks;
    }
    const int P = (int)Nu.size() - 1, K = (int)Du.size() - 1;
    if (K < 1) return fail(PLR_ERR_SIGNATURE, "the cascade has no feedback stage (k = 0, P:89-93)");
    if (K > kMaxK || P > kMaxP) return fail(PLR_ERR_SIZE, "combined order exceeds PLR_MAX_K / PLR_MAX_P");
    double ac[kMaxP + 1], bc[kMaxK];
    for (int j = 0; j <= P; j++) ac[j] = dtype == PLR_INT32 ? (double)Nu[j] : Nd[j];
    for (int j = 1; j <= K; j++)                       // b_j = -D_j
        bc[j - 1] = dtype == PLR_INT32 ? (double)((0x100000000ull - Du[j]) & 0xffffffffull) : -Dd[j];
    return plr_plan_create(out, ac, P, bc, K, dtype, n_max);
}

plr_status plr_plan_get_signature(const plr_plan* plan, double* a, double* b) {
    if (plan == nullptr || a == nullptr || b == nullptr) return fail(PLR_ERR_INVALID_ARG, "null argument");
    for (int j = 0; j <= plan->pt.p; j++) a[j] = plan->pt.dtype == PLR_INT32 ? (double)plan->pt.a_u[j] : plan->pt.a_d[j];
    for (int j = 0; j < plan->pt.k; j++) b[j] = plan->pt.dtype == PLR_INT32 ? (double)plan->pt.b_u[j] : plan->pt.b_d[j];
    return PLR_OK;
}

plr_status plr_plan_get_info(const plr_plan* plan, plr_plan_info* info) {
    if (plan == nullptr || info == nullptr) return fail(PLR_ERR_INVALID_ARG, "null argument");
    info->p = plan->pt.p;
    info->k = plan->pt.k;
    info->dtype = plan->pt.dtype;
    info->cls = plan->pt.cls;
    info->elems_per_thread = plan->pt.geo.X;
    info->threads_per_cta = plan->pt.geo.W * 32;
    info->tile_elems = plan->pt.geo.tile();
    info->stages = scan_stages(plan->pt);
    info->decay_len = plan->pt.decay_len;
    info->fixup_len = plan->pt.fixup_len;
    info->n_max = plan->n_max;
    info->scratch_bytes = 8 + (plan->status_slots + plan->status_slots_s) * kStatusMaxBytes + (size_t)plan->pt.k * plan->pt.k * 128 +
                          (size_t)plan->pt.fixup_len * kAug * 4 + 64;
    info->ctas_per_sm = plan->ctas_per_sm;
    info->num_sms = plan->num_sms;
    info->const_sig = plan->sig_kernel ? plan->pt.sig_id : 0;
    info->tiles_per_unit = plan->pt.geo.G;
    info->kernel_kind = kernel_kind(plan->pt);
    info->acc_bits = (plan->pt.dtype == PLR_FLOAT32 && plan->pt.acc64) ? 64 : 32;
    info->cond_bound = plan->pt.dtype == PLR_FLOAT32 ? plan->pt.cond_bound : 0.0;
    info->map_floor = plan->pt.dtype == PLR_FLOAT32 ? plan->pt.map_floor : 0.0;
    info->nyquist_gain = plan->pt.dtype == PLR_FLOAT32 ? plan->pt.nyquist_gain : 0.0;
    info->small_clusters = plan->small_clusters;
    info->small_cluster_ctas = kSmallC;
    info->small_ctas_per_sm = plan->small_ctas;
    info->small_max = plan->small_max;
    return PLR_OK;
}

plr_status plr_plan_debug_stats(plr_plan* plan, uint64_t* out, int reset) {
    if (plan == nullptr || out == nullptr) return fail(PLR_ERR_INVALID_ARG, "null argument");
    if (plan->d_stats == nullptr) {
        memset(out, 0, 16 * sizeof(uint64_t));
        return PLR_OK;
    }
    CUDA_TRY(cudaMemcpy(out, plan->d_stats, 128, cudaMemcpyDeviceToHost), "stats copy");
    if (reset) CUDA_TRY(cudaMemset(plan->d_stats, 0, 128), "stats reset");
    return PLR_OK;
}

plr_status plr_plan_factor_lists(const plr_plan* plan, int64_t m, void* out) {
    if (plan == nullptr || out == nullptr || m < 0) return fail(PLR_ERR_INVALID_ARG, "bad argument");
    factor_lists(plan->pt, m, out);
    return PLR_OK;
}

plr_status plr_execute(plr_plan* plan, const void* x, void* y, size_t n, void* stream) {
    plr_status st = check_xy(plan, x, y, n, true);
    if (st != PLR_OK || n == 0) return st;
    return launch(plan, x, y, n, nullptr, nullptr, nullptr, true, (cudaStream_t)stream);
}

plr_status plr_execute_reverse(plr_plan* plan, const void* x, void* y, size_t n, void* stream) {
    plr_status st = check_xy(plan, x, y, n, true);
    if (st != PLR_OK || n == 0) return st;
    return launch(plan, x, y, n, nullptr, nullptr, nullptr, true, (cudaStream_t)stream, true);
}

plr_status plr_execute_bidirectional(plr_plan* plan, const void* x, void* y, size_t n, void* tmp, void* stream) {
    plr_status st = check_xy(plan, x, y, n, true);
    if (st != PLR_OK || n == 0) return st;
    if (tmp == nullptr && plan->pt.p > 0)
        return fail(PLR_ERR_INVALID_ARG, "p > 0: the forward pass needs a tmp buffer (the reverse pass cannot run in place)");
    void* mid = tmp != nullptr ? tmp : y;
    if (tmp != nullptr) {
        if ((st = check_xy(plan, x, tmp, n, true)) != PLR_OK) return st;
        if ((st = check_xy(plan, tmp, y, n, true)) != PLR_OK) return st;
    }
    cudaStream_t s = (cudaStream_t)stream;
    st = launch(plan, x, mid, n, nullptr, nullptr, nullptr, true, s, false);        // causal pass
    if (st != PLR_OK) return st;
    return launch(plan, mid, y, n, nullptr, nullptr, nullptr, true, s, true);        // anticausal pass
}

plr_status plr_scan_comparator(plr_plan* plan, const void* x, void* y, size_t n, void* stream) {
    plr_status st = check_xy(plan, x, y, n, true);
    if (st != PLR_OK || n == 0) return st;
    if (n > plan->n_max) return fail(PLR_ERR_SIZE, "n exceeds the plan's n_max");
    cudaStream_t s = (cudaStream_t)stream;
    const PlanTables& pt = plan->pt;
    float cf[kMaxK], af[kMaxP + 1];
    for (int r = 0; r < pt.k; r++) cf[r] = (float)pt.b_d[r];
    for (int j = 0; j <= pt.p; j++) af[j] = (float)pt.a_d[j];
    auto run = [&](void* tmp, size_t& bytes) -> cudaError_t {
        if (pt.dtype == PLR_INT32)
            return blelloch_i32((const uint32_t*)x, (uint32_t*)y, (long long)n, pt.b_u, pt.k, pt.a_u, pt.p, tmp, bytes, s);
        return blelloch_f32((const float*)x, (float*)y, (long long)n, cf, pt.k, af, pt.p, tmp, bytes, s);
    };
    size_t need = 0;
    CUDA_TRY(run(nullptr, need), "Scan comparator size query");
    if (need > plan->scan_tmp_bytes) {
        cudaFree(plan->d_scan_tmp);
        plan->d_scan_tmp = nullptr;
        plan->scan_tmp_bytes = 0;
        CUDA_TRY(cudaMalloc(&plan->d_scan_tmp, need), "alloc Scan comparator storage");
        plan->scan_tmp_bytes = need;
    }
    size_t have = plan->scan_tmp_bytes;
    CUDA_TRY(run(plan->d_scan_tmp, have), "Scan comparator");
    return PLR_OK;
}

plr_status plr_execute_continue(plr_plan* plan, const void* x, void* y, size_t n, const void* x_hist,
                                const void* y_hist, void* stream) {
    plr_status st = check_xy(plan, x, y, n, true);
    if (st != PLR_OK || n == 0) return st;
    if (plan->pt.p == 0) x_hist = nullptr;
    return launch(plan, x, y, n, x_hist, y_hist, nullptr, true, (cudaStream_t)stream);
}

plr_status plr_reduce(plr_plan* plan, const void* x, size_t n, void* payload, void* stream) {
    plr_status st = check_xy(plan, x, nullptr, n, false);
    if (st != PLR_OK) return st;
    if (payload == nullptr) return fail(PLR_ERR_INVALID_ARG, "null payload");
    cudaStream_t s = (cudaStream_t)stream;
    CUDA_TRY(cudaMemsetAsync(payload, 0, PLR_PAYLOAD_BYTES, s), "payload memset");
    if (n > 0) {
        uint32_t* y_tail = reinterpret_cast<uint32_t*>((unsigned char*)payload + 24) + (4 - plan->pt.k);
        if (n > plan->n_max) return fail(PLR_ERR_SIZE, "n exceeds the plan's n_max");
        if (n > plan->small_max && plan->d_rd != nullptr && std::getenv("PLR_NO_REDUCE_KERNEL") == nullptr) {
            // contiguous-range streaming fold, no look-back (plr_kernels_reduce.cuh)
            if (plan->dirty || plan->epoch >= 0x7ffffff0u) {
                CUDA_TRY(cudaMemsetAsync(plan->d_status, 0, plan->status_slots * kStatusMaxBytes, s), "status reset");
                CUDA_TRY(cudaMemsetAsync(plan->d_status_s, 0, plan->status_slots_s * kStatusMaxBytes, s), "status reset");
                CUDA_TRY(cudaMemsetAsync(plan->d_ticket, 0, kTicketBytes, s), "ticket reset");
                plan->epoch = 0;
                plan->dirty = false;
            }
            plan->epoch++;
            const uint64_t m = (uint64_t)kRedX * kRedW * 32;
            LaunchArgs la;
            la.x = x; la.y = nullptr; la.n = n; la.ntiles = (n + m - 1) / m;
            la.ticket = plan->d_ticket;
            la.status = plan->d_rd;
            la.status_mask = 0;
            la.decay = 0;
            la.x_hist = nullptr; la.y_hist = nullptr; la.y_tail = y_tail;
            la.lane_T = nullptr;
            la.grid = (int)std::min<uint64_t>(std::min<uint64_t>(la.ntiles, (uint64_t)plan->num_sms * plan->reduce_ctas),
                                                 (uint64_t)kRedMaxGrid);
            la.store = false;
            la.stream = s;
            cudaError_t e = launch_reduce(plan->pt, la);
            if (e != cudaSuccess) {
                plan->dirty = true;
                return cuda_fail(e, "reduce kernel launch");
            }
        } else {
            st = launch(plan, x, nullptr, n, nullptr, nullptr, y_tail, false, s);
            if (st != PLR_OK) return st;
        }
    }
    payload_kernel<<<1, 32, 0, s>>>((const uint32_t*)x, nullptr, n, (unsigned char*)payload, 0);
    CUDA_TRY(cudaGetLastError(), "payload kernel");
    return PLR_OK;
}

plr_status plr_payload_from_output(plr_plan* plan, const void* x, const void* y, size_t n, void* payload,
                                   void* stream) {
    if (plan == nullptr || payload == nullptr) return fail(PLR_ERR_INVALID_ARG, "null argument");
    cudaStream_t s = (cudaStream_t)stream;
    CUDA_TRY(cudaMemsetAsync(payload, 0, PLR_PAYLOAD_BYTES, s), "payload memset");
    payload_kernel<<<1, 32, 0, s>>>((const uint32_t*)x, (const uint32_t*)y, n, (unsigned char*)payload, 1);
    CUDA_TRY(cudaGetLastError(), "payload kernel");
    return PLR_OK;
}

plr_status plr_combine(plr_plan* plan, const void* payloads, int rank, int world, void* hist, void* stream) {
    if (plan == nullptr || payloads == nullptr || hist == nullptr || world < 1 || rank < 0 || rank >= world)
        return fail(PLR_ERR_INVALID_ARG, "bad combine arguments");
    cudaStream_t s = (cudaStream_t)stream;
    if (plan->pt.dtype == PLR_INT32)
        combine_kernel<uint32_t><<<1, 32, 0, s>>>(aug_matrix<uint32_t>(plan->pt), (const unsigned char*)payloads, rank,
                                                  (uint32_t*)hist);
    else
        combine_kernel<double><<<1, 32, 0, s>>>(aug_matrix<double>(plan->pt), (const unsigned char*)payloads, rank,
                                                (uint32_t*)hist);
    CUDA_TRY(cudaGetLastError(), "combine kernel");
    return PLR_OK;
}

plr_status plr_combine_host(const plr_plan* plan, const void* payloads, int rank, int world, void* hist) {
    if (plan == nullptr || payloads == nullptr || hist == nullptr || world < 1 || rank < 0 || rank >= world)
        return fail(PLR_ERR_INVALID_ARG, "bad combine arguments");
    if (plan->pt.dtype == PLR_INT32)
        combine_host_impl<uint32_t>(aug_matrix<uint32_t>(plan->pt), (const unsigned char*)payloads, rank, (uint32_t*)hist);
    else
        combine_host_impl<double>(aug_matrix<double>(plan->pt), (const unsigned char*)payloads, rank, (uint32_t*)hist);
    return PLR_OK;
}

plr_status plr_fixup(plr_plan* plan, void* y, size_t n, const void* hist, void* stream) {
    if (plan == nullptr || hist == nullptr) return fail(PLR_ERR_INVALID_ARG, "null argument");
    if (plan->pt.cls != PLR_CLASS_DECAY) return fail(PLR_ERR_INVALID_ARG, "fixup needs a DECAY-class plan");
    const unsigned long long len = std::min<unsigned long long>(n, (unsigned long long)plan->pt.fixup_len);
    if (len == 0) return PLR_OK;
    fixup_kernel<<<(unsigned)((len + 255) / 256), 256, 0, (cudaStream_t)stream>>>((float*)y, len, plan->d_fix,
                                                                                  (const uint32_t*)hist);
    CUDA_TRY(cudaGetLastError(), "fixup kernel");
    return PLR_OK;
}

// ------------------------------------------------------------- NCCL -------
typedef int (*nccl_get_id_t)(void*);
struct NcclId { char internal[128]; };   // ncclUniqueId (NCCL_UNIQUE_ID_BYTES = 128), passed by value
typedef int (*nccl_init_t)(void**, int, NcclId, int);
typedef int (*nccl_allgather_t)(const void*, void*, size_t, int, void*, cudaStream_t);
typedef int (*nccl_destroy_t)(void*);
typedef const char* (*nccl_errstr_t)(int);

static struct {
    bool tried = false;
    void* h = nullptr;
    nccl_get_id_t get_id = nullptr;
    nccl_init_t init = nullptr;
    nccl_allgather_t allgather = nullptr;
    nccl_destroy_t destroy = nullptr;
    nccl_errstr_t errstr = nullptr;
} g_nccl;

static plr_status nccl_load() {
    if (!g_nccl.tried) {
        g_nccl.tried = true;
        g_nccl.h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (g_nccl.h) {
            g_nccl.get_id = (nccl_get_id_t)dlsym(g_nccl.h, "ncclGetUniqueId");
            g_nccl.init = (nccl_init_t)dlsym(g_nccl.h, "ncclCommInitRank");
            g_nccl.allgather = (nccl_allgather_t)dlsym(g_nccl.h, "ncclAllGather");
            g_nccl.destroy = (nccl_destroy_t)dlsym(g_nccl.h, "ncclCommDestroy");
            g_nccl.errstr = (nccl_errstr_t)dlsym(g_nccl.h, "ncclGetErrorString");
        }
    }
    if (!g_nccl.h || !g_nccl.get_id || !g_nccl.init || !g_nccl.allgather || !g_nccl.destroy)
        return fail(PLR_ERR_NCCL, "libnccl.so.2 not loadable");
    return PLR_OK;
}

static plr_status nccl_fail(int r, const char* what) {
    return fail(PLR_ERR_NCCL, std::string(what) + ": " + (g_nccl.errstr ? g_nccl.errstr(r) : "nccl error"));
}

plr_status plr_nccl_unique_id(void* id_out, size_t id_bytes) {
    if (id_out == nullptr || id_bytes < 128) return fail(PLR_ERR_INVALID_ARG, "id buffer must hold 128 bytes");
    plr_status st = nccl_load();
    if (st != PLR_OK) return st;
    int r = g_nccl.get_id(id_out);
    return r == 0 ? PLR_OK : nccl_fail(r, "ncclGetUniqueId");
}

plr_status plr_nccl_comm_init(void** comm_out, const void* id, int rank, int world) {
    if (comm_out == nullptr || id == nullptr) return fail(PLR_ERR_INVALID_ARG, "null argument");
    plr_status st = nccl_load();
    if (st != PLR_OK) return st;
    NcclId nid;
    memcpy(nid.internal, id, 128);
    int r = g_nccl.init(comm_out, world, nid, rank);
    return r == 0 ? PLR_OK : nccl_fail(r, "ncclCommInitRank");
}

plr_status plr_nccl_comm_destroy(void* comm) {
    if (comm == nullptr) return PLR_OK;
    plr_status st = nccl_load();
    if (st != PLR_OK) return st;
    int r = g_nccl.destroy(comm);
    return r == 0 ? PLR_OK : nccl_fail(r, "ncclCommDestroy");
}

plr_status plr_execute_sharded(plr_plan* plan, const void* x, void* y, size_t n, int rank, int world, void* comm,
                               void* stream) {
    plr_status st = check_xy(plan, x, y, n, true);
    if (st != PLR_OK) return st;
    if (world < 1 || rank < 0 || rank >= world) return fail(PLR_ERR_INVALID_ARG, "bad rank/world");
    if (world > 1 && comm == nullptr) return fail(PLR_ERR_INVALID_ARG, "null comm");
    cudaStream_t s = (cudaStream_t)stream;
    if (plan->d_send == nullptr) CUDA_TRY(cudaMalloc(&plan->d_send, PLR_PAYLOAD_BYTES), "alloc payload");
    if (plan->recv_world < world) {
        cudaFree(plan->d_recv);
        plan->d_recv = nullptr;
        CUDA_TRY(cudaMalloc(&plan->d_recv, (size_t)world * PLR_PAYLOAD_BYTES), "alloc payloads");
        plan->recv_world = world;
    }
    const bool decay = plan->pt.cls == PLR_CLASS_DECAY;
    if (decay) {
        st = launch(plan, x, y, n, nullptr, nullptr, nullptr, true, s);            // zero boundary, 2n
        if (st != PLR_OK) return st;
        st = plr_payload_from_output(plan, x, y, n, plan->d_send, stream);
    } else {
        st = plr_reduce(plan, x, n, plan->d_send, stream);                          // reads n
    }
    if (st != PLR_OK) return st;
    if (comm != nullptr) {                      // the collective, also for a 1-rank communicator
        st = nccl_load();
        if (st != PLR_OK) return st;
        int r = g_nccl.allgather(plan->d_send, plan->d_recv, PLR_PAYLOAD_BYTES, /*ncclUint8*/ 1, comm, s);
        if (r != 0) return nccl_fail(r, "ncclAllGather");
    } else {                                    // world == 1 without a communicator: loopback
        CUDA_TRY(cudaMemcpyAsync(plan->d_recv, plan->d_send, PLR_PAYLOAD_BYTES, cudaMemcpyDeviceToDevice, s), "copy");
    }
    st = plr_combine(plan, plan->d_recv, rank, world, plan->d_hist, stream);
    if (st != PLR_OK) return st;
    if (decay) return plr_fixup(plan, y, n, plan->d_hist, stream);                // sparse, <= fixup_len
    const uint32_t* xh = plan->d_hist + (4 - plan->pt.p);
    const uint32_t* yh = plan->d_hist + 4 + (4 - plan->pt.k);
    return launch(plan, x, y, n, plan->pt.p ? xh : nullptr, yh, nullptr, true, s);  // seeded single pass, 2n
}

// ------------------------------------------------------------- host e2e ---
plr_status plr_execute_host(plr_plan* plan, const void* x_host, void* y_host, size_t n, void* stream) {
    if (plan == nullptr) return fail(PLR_ERR_INVALID_ARG, "null plan");
    if (n == 0) return PLR_OK;
    if (x_host == nullptr || y_host == nullptr) return fail(PLR_ERR_INVALID_ARG, "null host pointer");
    cudaStream_t s = (cudaStream_t)stream;
    const size_t C = std::min<size_t>(plan->n_max, (size_t)1 << 25) & ~(size_t)3;
    if (C < 16) return fail(PLR_ERR_SIZE, "n_max too small for the host pipeline");
    if (plan->h_chunk != C) {
        for (int i = 0; i < 3; i++) {
            cudaFree(plan->h_dx[i]); cudaFree(plan->h_dy[i]);
            plan->h_dx[i] = plan->h_dy[i] = nullptr;
            CUDA_TRY(cudaMalloc(&plan->h_dx[i], C * 4), "alloc pipeline buffer");
            CUDA_TRY(cudaMalloc(&plan->h_dy[i], C * 4), "alloc pipeline buffer");
            if (!plan->ev_in[i]) {
                CUDA_TRY(cudaEventCreateWithFlags(&plan->ev_in[i], cudaEventDisableTiming), "event");
                CUDA_TRY(cudaEventCreateWithFlags(&plan->ev_comp[i], cudaEventDisableTiming), "event");
                CUDA_TRY(cudaEventCreateWithFlags(&plan->ev_out[i], cudaEventDisableTiming), "event");
            }
        }
        if (!plan->s_in) CUDA_TRY(cudaStreamCreateWithFlags(&plan->s_in, cudaStreamNonBlocking), "stream");
        if (!plan->s_out) CUDA_TRY(cudaStreamCreateWithFlags(&plan->s_out, cudaStreamNonBlocking), "stream");
        plan->h_chunk = C;
    }
    // order the pipeline after work already queued on the caller's stream
    CUDA_TRY(cudaEventRecord(plan->ev_comp[2], s), "record");
    CUDA_TRY(cudaStreamWaitEvent(plan->s_in, plan->ev_comp[2], 0), "wait");
    CUDA_TRY(cudaStreamWaitEvent(plan->s_out, plan->ev_comp[2], 0), "wait");
    const size_t nch = (n + C - 1) / C;
    const int p = plan->pt.p, k = plan->pt.k;
    for (size_t i = 0; i < nch; i++) {
        const int slot = (int)(i % 3), prev = (int)((i + 2) % 3);
        const size_t off = i * C, len = std::min(C, n - off);
        if (i >= 2) CUDA_TRY(cudaStreamWaitEvent(plan->s_in, plan->ev_comp[(i - 2) % 3], 0), "wait");
        CUDA_TRY(cudaMemcpyAsync(plan->h_dx[slot], (const char*)x_host + off * 4, len * 4, cudaMemcpyHostToDevice,
                                 plan->s_in), "H2D");
        CUDA_TRY(cudaEventRecord(plan->ev_in[slot], plan->s_in), "record");
        CUDA_TRY(cudaStreamWaitEvent(s, plan->ev_in[slot], 0), "wait");
        if (i >= 3) CUDA_TRY(cudaStreamWaitEvent(s, plan->ev_out[slot], 0), "wait");
        const void* xh = nullptr;
        const void* yh = nullptr;
        if (i > 0) {
            xh = p ? (const char*)plan->h_dx[prev] + (C - p) * 4 : nullptr;
            yh = (const char*)plan->h_dy[prev] + (C - k) * 4;
        }
        plr_status st = launch(plan, plan->h_dx[slot], plan->h_dy[slot], len, xh, yh, nullptr, true, s);
        if (st != PLR_OK) return st;
        CUDA_TRY(cudaEventRecord(plan->ev_comp[slot], s), "record");
        CUDA_TRY(cudaStreamWaitEvent(plan->s_out, plan->ev_comp[slot], 0), "wait");
        CUDA_TRY(cudaMemcpyAsync((char*)y_host + off * 4, plan->h_dy[slot], len * 4, cudaMemcpyDeviceToHost,
                                 plan->s_out), "D2H");
        CUDA_TRY(cudaEventRecord(plan->ev_out[slot], plan->s_out), "record");
    }
    CUDA_TRY(cudaStreamSynchronize(plan->s_out), "sync");
    CUDA_TRY(cudaStreamSynchronize(s), "sync");
    return PLR_OK;
}

}  // extern "C"
