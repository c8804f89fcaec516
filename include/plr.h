/*
 * plr.h -- C ABI of the B200-native PLR hot path.
 *
 * Evaluates an order-k constant-coefficient linear recurrence given in the
 * paper's signature notation (a0, a-1, ..., a-p : b-1, ..., b-k):
 *
 *     y_i = a0 x_i + a-1 x_{i-1} + ... + a-p x_{i-p}
 *               + b-1 y_{i-1} + ... + b-k y_{i-k},      x_j = y_j = 0 for j < 0
 *
 * (Eq. (1)), in one pass over the data on an sm_100a GPU: fused
 * feed-forward map (Eq. (2)), per-thread sequential chunks, warp- and
 * block-level carry propagation with precomputed correction factors
 * (Sec. 2.1), grid-level decoupled look-back of the k carries
 * (Sec. 2.2-2.3) and the correction y_i += sum_r carry_r*f_r[i]
 * (P:254-274).  "P:n" is line n of the paper text
 * (Maleki & Burtscher, ASPLOS'18).
 *
 * Conventions shared by every entry point
 *  - Status codes only; nothing throws across this ABI.  plr_last_error()
 *    returns a thread-local description of the last failure.
 *  - Sizes are element counts (size_t, 64-bit); n = 0 is a no-op (PLR_OK).
 *  - Device pointers must be 16-byte aligned (PLR_ERR_MISALIGNED).  x and y
 *    must not overlap unless x == y and p == 0 (PLR_ERR_ALIAS): with p > 0
 *    the feed-forward halo would read already overwritten inputs.
 *  - Data types: PLR_INT32 computes in the ring
 *    Z/2^32 (two's-complement wraparound everywhere, reading R1;
 *    coefficients must be integers in [-2^31, 2^32)); PLR_FLOAT32 computes in
 *    fp32 with the coefficients rounded to fp32 (reading R3).
 *  - `stream` is a cudaStream_t (NULL = legacy default stream).  Every
 *    device-side call is asynchronous and stream-ordered; it performs no host
 *    synchronisation and no allocation (except plr_execute_host, which is
 *    synchronous, and plr_execute_sharded's first call, which allocates its
 *    payload buffer).
 *  - A plan is like a cuFFT plan: it owns its scratch (tile-status words,
 *    ticket counter, tables, payload buffers) and must be used on one
 *    stream at a time.
 *  - plr_execute, plr_execute_continue and plr_reduce may be captured in a
 *    CUDA graph (stream capture) after one eager call on the plan: the
 *    per-launch state (ticket base, status epoch) lives in device memory and
 *    each launch advances it for the next, so replays and eager launches of
 *    the same plan can be interleaved in stream order.
 */
#ifndef PLR_H
#define PLR_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define PLR_ABI_VERSION 4
#define PLR_MAX_K 4            /* maximum order k supported by the kernels      */
#define PLR_MAX_P 3            /* maximum feed-forward order p                  */
#define PLR_PAYLOAD_BYTES 64   /* one rank's end-state record, see plr_reduce   */

typedef enum { PLR_INT32 = 0, PLR_FLOAT32 = 1 } plr_dtype;

typedef enum {
    PLR_OK = 0,
    PLR_ERR_INVALID_ARG = 1,
    PLR_ERR_SIGNATURE = 2,     /* k < 1, a[p] == 0, b[k-1] == 0, non-finite, non-integer for INT32 */
    PLR_ERR_DTYPE = 3,
    PLR_ERR_SIZE = 4,          /* n > n_max, or k/p beyond PLR_MAX_K/PLR_MAX_P */
    PLR_ERR_ALIAS = 5,
    PLR_ERR_MISALIGNED = 6,
    PLR_ERR_CUDA = 7,
    PLR_ERR_NCCL = 8,
    PLR_ERR_OOM = 9
} plr_status;

/* Signature classes (SURVEY.md notation; "Optimizations"). */
typedef enum {
    PLR_CLASS_ONES = 0,        /* (1: 1): every correction factor is 1              */
    PLR_CLASS_PERM = 1,        /* s-tuple prefix sums: 0/1 periodic factors         */
    PLR_CLASS_POLY = 2,        /* other integer signatures (dense factors, mod 2^32) */
    PLR_CLASS_DECAY = 3,       /* fp32 factors underflow to exactly 0    */
    PLR_CLASS_FLOAT = 4        /* fp32 signature whose factors do not decay          */
} plr_class;

typedef struct plr_plan plr_plan;   /* opaque */

typedef struct {
    int p, k;
    plr_dtype dtype;
    plr_class cls;
    int elems_per_thread;      /* x: contiguous elements per thread              */
    int threads_per_cta;       /* compute threads (the CTA adds one producer warp) */
    int tile_elems;            /* m = 32 * warps * x                              */
    int stages;                /* shared-memory ring depth                        */
    int64_t decay_len;         /* DECAY: last index u with fp32 g_u != 0, else -1 */
    int64_t fixup_len;         /* DECAY: outputs a boundary state can still change */
    size_t n_max;
    size_t scratch_bytes;      /* device bytes the plan owns                      */
    int ctas_per_sm;
    int num_sms;
    int const_sig;             /* != 0: the scan kernel has this signature's tables as
                                  compile-time constants (the generator's per-signature
                                  code); 0: tables read from the
                                  kernel parameters                                   */
    int tiles_per_unit;        /* G: consecutive tiles per ticket / status record / look-back */
    int kernel_kind;           /* scan kernel: 0 DECAY single-hop pipeline, 1 TMEM-parking,
                                  2 L2 re-read (generic classes), 3 generic smem pipeline,
                                  4 DECAY single-hop with TMEM-parked map outputs        */
    int acc_bits;              /* accumulation of the chunk recurrence and carries: 32 (the
                                  data type) or 64 (fp64, reading R16)       */
    double cond_bound;         /* float: the planner's a-priori error bound of fp32
                                  accumulation relative to the output scale (R16); 0 int */
    double map_floor;          /* float: the error floor of ANY fp32-data evaluation (the map
                                  rounds the input) relative to a Nyquist-frequency output
                                  (reading R20); 0 int                        */
    double nyquist_gain;       /* float: |H(-1)|, the gain at the Nyquist frequency; 0 int */
    int small_clusters;        /* co-resident thread-block clusters of small-n CTAs (the
                                  cluster look-back of non-decaying small launches); 0: none */
    int small_cluster_ctas;    /* CTAs (tiles) per such cluster                        */
    int small_ctas_per_sm;     /* CTAs per SM of the small-n kernel                    */
    size_t small_max;          /* n <= small_max runs the small-n kernel               */
} plr_plan_info;

/* Create a plan.  a[0..p] = (a0, a-1, ..., a-p) (p = feed-forward order, so
 * p+1 entries, reading R5); b[0..k-1] = (b-1, ..., b-k).  Checks
 * of P:87-93 and P:634-637: k >= 1, b[k-1] != 0 and a[p] != 0 ("the last
 * non-recursive and the last recursive coefficients must not be zero");
 * trailing zeros are rejected, not trimmed.  The host planner precomputes
 * the correction factors (impulse responses) and every transfer
 * matrix the kernels use.  Allocates device scratch for up to n_max
 * elements per call on the current device.  n_max = 0 creates a host-only
 * plan (planner tables only, no CUDA calls): usable for plr_plan_get_info,
 * plr_plan_factor_lists and plr_combine_host without a GPU.  On failure
 * *out is NULL. */
plr_status plr_plan_create(plr_plan** out, const double* a, int p, const double* b, int k,
                           plr_dtype dtype, size_t n_max);
plr_status plr_plan_destroy(plr_plan* plan);
plr_status plr_plan_get_info(const plr_plan* plan, plr_plan_info* info);

/* A cascade of `nstages` signatures evaluated in ONE pass ("inputs that
 * consist of multiple signatures"; a higher-order filter as
 * several lower-order ones).  Stage s is (a_s : b_s) with p[s]+1
 * feed-forward and k[s] feedback coefficients (k[s] = 0: a pure map stage),
 * packed stage after stage in a[] and b[].  The planner combines the stages
 * by multiplying their z-transforms (numerators A_s(z) and denominators
 * 1 - sum_j b_{s,j} z^-j) -- the combination the paper leaves to the user,
 * offline -- and plans the resulting single signature: one read
 * and one write of the data instead of one per stage.  PLR_INT32 combines in
 * Z/2^32 (bit-exact: a ring homomorphism); PLR_FLOAT32 combines in fp64 the
 * fp32-rounded stage coefficients.  Each stage is checked like a signature
 * (last coefficients nonzero); the combination must have k >= 1,
 * k <= PLR_MAX_K and p <= PLR_MAX_P (PLR_ERR_SIZE). */
plr_status plr_plan_create_cascade(plr_plan** out, int nstages, const double* a, const int* p,
                                   const double* b, const int* k, plr_dtype dtype, size_t n_max);

/* The signature a plan evaluates (for a cascade: the combined one), as the
 * kernels use it: a[0..p] (a0, a-1, ..., a-p) and b[0..k-1] (b-1, ..., b-k);
 * int32 coefficients as their residues in [0, 2^32), float32 ones rounded to
 * fp32.  Host memory (PLR_MAX_P+1 and PLR_MAX_K doubles suffice). */
plr_status plr_plan_get_signature(const plr_plan* plan, double* a, double* b);

/* Planner introspection (tests): the correction-factor lists of Sec. 2.1 as
 * the kernels use them.  out receives k rows of (k + m) values (the seed in
 * memory order w_{m-k}..w_{m-1}, then m factors), int32 for PLR_INT32, float
 * for PLR_FLOAT32 (rounded from fp64, denormals flushed).  Host memory. */
plr_status plr_plan_factor_lists(const plr_plan* plan, int64_t m, void* out);

/* Debug counters of the generic look-back, enabled by PLR_STATS=1 in the
 * environment at plan creation (otherwise all zero): out[0] look-backs,
 * out[1] window polls, out[2] polls that folded nothing, out[3] summed
 * depth in tiles, out[4] SM cycles waiting for the tile's own aggregate,
 * out[5] cycles looking back, out[6] of which sleeping, out[7] loading and
 * classifying windows, out[8] folding.  Synchronous;
 * reset != 0 clears them.  Host memory. */
plr_status plr_plan_debug_stats(plr_plan* plan, uint64_t* out /* 16 */, int reset);

/* y[0..n) = recurrence over x[0..n) with zero initial conditions.
 * x, y: device pointers of the plan's dtype. */
plr_status plr_execute(plr_plan* plan, const void* x, void* y, size_t n, void* stream);

/* The anticausal recurrence over x[0..n):
 *     y_i = a0 x_i + a-1 x_{i+1} + ... + a-p x_{i+p} + b-1 y_{i+1} + ... + b-k y_{i+k},
 * with x_j = y_j = 0 for j >= n -- Eq. (1) run from the end of the data to its
 * start, the backward half of the causal/anticausal filter pairs of P:809-811
 * and P:866-868.  Same layout, alignment and aliasing rules as plr_execute
 * (x == y allowed when p == 0).  One pass: tiles are processed from the end
 * with the same hierarchy and look-back. */
plr_status plr_execute_reverse(plr_plan* plan, const void* x, void* y, size_t n, void* stream);

/* The paper's "Scan" comparator: Blelloch's
 * (k x k matrix, k-vector) prefix-scan formulation of the same recurrence,
 * through CUB DeviceScan, fp32 / Z/2^32 arithmetic, zero initial state.  A
 * comparison baseline for benchmarks, NOT the PLR
 * path.  Same arguments and rules as plr_execute; the first call (and any
 * larger n) allocates CUB's temporary storage in the plan (synchronously). */
plr_status plr_scan_comparator(plr_plan* plan, const void* x, void* y, size_t n, void* stream);

/* Forward-backward (zero-phase) filtering: y = reverse(forward(x)), i.e. the
 * causal recurrence then the anticausal one (plr_execute_reverse) on its
 * output, two passes.  tmp (device, n elements of the dtype) holds the
 * intermediate; it may be NULL when p == 0 (the backward pass then runs in
 * place in y).  The intermediate is rounded to the dtype. */
plr_status plr_execute_bidirectional(plr_plan* plan, const void* x, void* y, size_t n, void* tmp,
                                     void* stream);

/* Same, continuing a sequence: x_hist points at the p inputs before x[0]
 * (x_{-p}..x_{-1}, index order) and y_hist at the k outputs before y[0]
 * (y_{-k}..y_{-1}).  Either may be NULL (zeros).  For a long array split in
 * chunks, x_hist = x - p and y_hist = y - k.  Device pointers (4-byte
 * aligned suffices for the histories). */
plr_status plr_execute_continue(plr_plan* plan, const void* x, void* y, size_t n,
                                const void* x_hist, const void* y_hist, void* stream);

/* Reduce-only pass: the end state of x[0..n) with zero history, without
 * writing y (reads n elements).  payload (device, PLR_PAYLOAD_BYTES) gets
 *   uint64 n | uint32 x_tail[4] (x_{n-4}..x_{n-1}) | uint32 y_tail[4] (y_{n-4}..y_{n-1})
 * (bit patterns of the dtype; indices < 0 are 0; plr_reduce fills only the
 * last k y slots, the others stay 0 and are never read by the combine's
 * order-k recurrence row).  This is a segment's
 * contribution to the sharded combine. */
plr_status plr_reduce(plr_plan* plan, const void* x, size_t n, void* payload, void* stream);

/* Payload of an already evaluated segment (zero history): reads the tails of
 * x and y only. */
plr_status plr_payload_from_output(plr_plan* plan, const void* x, const void* y, size_t n,
                                   void* payload, void* stream);

/* Segment prefix over ranks: given `world` payloads (device, contiguous,
 * rank order), write rank `rank`'s history hist (device, 8 uint32 slots:
 * x_{-4}..x_{-1}, y_{-4}..y_{-1} relative to the start of its segment) using
 *   z_0 = 0,  z_{r+1} = M^{n_r} z_r + payload_r
 * with M the (p+k)-dimensional companion matrix of Eq. (1) (repeated
 * squaring; Z/2^32 or fp64).  One device thread. */
plr_status plr_combine(plr_plan* plan, const void* payloads, int rank, int world, void* hist,
                       void* stream);
/* The same combine evaluated on the host (host pointers); no GPU needed. */
plr_status plr_combine_host(const plr_plan* plan, const void* payloads, int rank, int world,
                            void* hist);

/* DECAY class: add the free response of the boundary state `hist` (layout as
 * plr_combine) to y[0..min(n, fixup_len)); beyond fixup_len the fp32
 * correction factors are exactly 0. */
plr_status plr_fixup(plr_plan* plan, void* y, size_t n, const void* hist, void* stream);

/* One segment of a sequence sharded over `world` ranks (rank r holds the
 * r-th contiguous segment; n_local may differ per rank).  `comm` is an
 * ncclComm_t from plr_nccl_comm_init (a 1-rank communicator is valid and
 * takes the same NCCL path; comm may be NULL only when world == 1, which
 * copies the payload instead of gathering it).  One ncclAllGather of
 * PLR_PAYLOAD_BYTES per rank over NVLink/NVSwitch; no other collective.
 * DECAY: local pass, allgather, sparse fixup (2n traffic).  Others:
 * reduce-only pass, allgather, seeded single pass (3n traffic). */
plr_status plr_execute_sharded(plr_plan* plan, const void* x_local, void* y_local, size_t n_local,
                               int rank, int world, void* comm, void* stream);

/* End-to-end from host memory: x_host/y_host are host pointers (pinned for
 * full copy-engine speed).  Streams chunks H2D -> recurrence -> D2H through
 * plan-owned device buffers with copies overlapped with compute; each chunk
 * continues from the previous one (plr_execute_continue).  Synchronous. */
plr_status plr_execute_host(plr_plan* plan, const void* x_host, void* y_host, size_t n, void* stream);

/* NCCL bootstrap: rank 0 creates the id, the caller broadcasts its bytes
 * (e.g. through torch.distributed), every rank calls plr_nccl_comm_init.
 * NCCL is loaded with dlopen("libnccl.so.2") (the process's NCCL). */
plr_status plr_nccl_unique_id(void* id_out, size_t id_bytes /* >= 128 */);
plr_status plr_nccl_comm_init(void** comm_out, const void* id, int rank, int world);
plr_status plr_nccl_comm_destroy(void* comm);

const char* plr_status_string(plr_status s);
const char* plr_last_error(void);
int plr_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* PLR_H */
