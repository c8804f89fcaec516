/*
 * plr_oracle.c -- CPU ORACLE for the PLR hot path.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference legs may load this library.  The product path
 * (paper_conf_asplos_malekib18_b200/) never links, imports or executes it,
 * and this file shares no code, header, table or constant generator with it.
 *
 * Citations: "P:n" = line n of the paper text (Maleki & Burtscher,
 * "Automatic Hierarchical Parallelization of Linear Recurrences", ASPLOS'18).
 *
 * What is here, each written as the paper states it (no blocking, fusion or
 * reordering beyond the stated definition / algorithm):
 *
 *  oracle_eq1_i32   Eq. (1), evaluated sequentially in index order
 *                   (serial code, applied to the split form
 *                   Eq. (2)+(3)) in the ring Z/2^32: every operand
 *                   is taken mod 2^32 in uint64_t and y is wrapped after every
 *                   element (reading R1: two's-complement wrap).
 *  oracle_eq1_f64   Eq. (1) in IEEE fp64, same order: feed-forward terms
 *                   j = 0..p, then feedback terms j = 1..k; no FTZ.
 *                   Both accept an optional history (x_{-p..-1}, y_{-k..-1});
 *                   NULL means the paper's zero initial conditions.
 *                   A history lets a long sequence be evaluated segment by
 *                   segment with the state carried across, which is the same
 *                   computation as one call over the concatenation.
 *  oracle_factor_lists_*  the correction-factor lists of Sec. 2.1:
 *                   for carry r, k seed elements that are all zero except a
 *                   one at the carry's position in the previous chunk, then
 *                   the recurrence (0: c) applied m more times.
 *  oracle_phase1_i32  Phase 1: chunks of size one are
 *                   merged pairwise, the i-th element of the second chunk of
 *                   each pair being corrected by sum_r carry_r * factor_r[i];
 *                   carries outside the first chunk are missing and count as
 *                   zero.  Records the array after each iteration
 *                   (the rows printed at P:592-596).
 *  oracle_phase2_i32  Phase 2: chunks of size m are
 *                   corrected in order with the last k values of the
 *                   previous (final) chunk.
 *  oracle_carry_precompute_i32  the look-back carry precomputation of
 *                   global carries of chunk j from the global
 *                   carries of chunk j-1 and the local carries of chunk j.
 *
 * Parity is pinned in tests/test_oracle.py (worked example P:578-602,
 * n-nacci identities P:350-361, closed forms, scipy lfilter, brute-force
 * lower-triangular solve, ...).  No function here is "parity unpinned".
 */
#include <stdint.h>
#include <stddef.h>
#include <string.h>

/* ---------------------------------------------------------------------- */
/* Eq. (1) in Z/2^32                                                        */
/* ---------------------------------------------------------------------- */

/* x[0..n), y[0..n): int32 sequences.  a[0..p]: (a0, a-1, ..., a-p) as int64;
 * b[0..k-1]: (b-1, ..., b-k) as int64.  x_hist: x_{-p}..x_{-1} (p values, in
 * index order) or NULL; y_hist: y_{-k}..y_{-1} (k values) or NULL. */
void oracle_eq1_i32(const int32_t* x, int32_t* y, int64_t n,
                    const int64_t* a, int p, const int64_t* b, int k,
                    const int32_t* x_hist, const int32_t* y_hist)
{
    for (int64_t i = 0; i < n; i++) {
        uint64_t acc = 0;
        /* feed-forward (map) terms, Eq. (2): t_i = sum_j a_{-j} x_{i-j} */
        for (int j = 0; j <= p; j++) {
            int64_t idx = i - j;
            uint32_t xv;
            if (idx >= 0) xv = (uint32_t)x[idx];
            else if (x_hist != NULL && -idx <= p) xv = (uint32_t)x_hist[p + idx];
            else xv = 0u;                                   /* x_j = 0, j < 0 */
            acc += (uint64_t)(uint32_t)a[j] * (uint64_t)xv;
            acc &= 0xffffffffull;
        }
        /* feedback terms, Eq. (3): y_i = t_i + sum_j b_{-j} y_{i-j} */
        for (int j = 1; j <= k; j++) {
            int64_t idx = i - j;
            uint32_t yv;
            if (idx >= 0) yv = (uint32_t)y[idx];
            else if (y_hist != NULL && -idx <= k) yv = (uint32_t)y_hist[k + idx];
            else yv = 0u;                                   /* y_j = 0, j < 0 */
            acc += (uint64_t)(uint32_t)b[j - 1] * (uint64_t)yv;
            acc &= 0xffffffffull;
        }
        y[i] = (int32_t)(uint32_t)acc;
    }
}

/* ---------------------------------------------------------------------- */
/* Eq. (1) in fp64                                                          */
/* ---------------------------------------------------------------------- */

/* x: fp32 inputs (promoted exactly); y: fp64 outputs.  a, b: coefficients
 * exactly as passed (the Python wrapper passes (double)(float)c, DESIGN.md
 * reading R3).  x_hist: p floats or NULL; y_hist: k doubles or NULL. */
void oracle_eq1_f64(const float* x, double* y, int64_t n,
                    const double* a, int p, const double* b, int k,
                    const float* x_hist, const double* y_hist)
{
    for (int64_t i = 0; i < n; i++) {
        double acc = 0.0;
        for (int j = 0; j <= p; j++) {
            int64_t idx = i - j;
            double xv;
            if (idx >= 0) xv = (double)x[idx];
            else if (x_hist != NULL && -idx <= p) xv = (double)x_hist[p + idx];
            else xv = 0.0;
            acc += a[j] * xv;
        }
        for (int j = 1; j <= k; j++) {
            int64_t idx = i - j;
            double yv;
            if (idx >= 0) yv = y[idx];
            else if (y_hist != NULL && -idx <= k) yv = y_hist[k + idx];
            else yv = 0.0;
            acc += b[j - 1] * yv;
        }
        y[i] = acc;
    }
}

/* Eq. (1) in fp64 over an fp64 input: one stage of a cascade, whose input is
 * the previous stage's (unrounded) output.  A cascade of filters feeds the
 * output of one filter into the next (a higher-order filter
 * decomposed into several lower-order ones; "inputs that consist of multiple
 * signatures").  Same order of terms as oracle_eq1_f64, zero
 * initial conditions. */
void oracle_eq1_f64_dd(const double* x, double* y, int64_t n,
                       const double* a, int p, const double* b, int k)
{
    for (int64_t i = 0; i < n; i++) {
        double acc = 0.0;
        for (int j = 0; j <= p; j++)
            if (i - j >= 0) acc += a[j] * x[i - j];
        for (int j = 1; j <= k; j++)
            if (i - j >= 0) acc += b[j - 1] * y[i - j];
        y[i] = acc;
    }
}

/* The anticausal recurrence: Eq. (1) with the time direction reversed,
 *   y_i = sum_{j=0..p} a_{-j} x_{i+j} + sum_{j=1..k} b_{-j} y_{i+j},
 * x_j = y_j = 0 for j >= n, evaluated from i = n-1 down to 0 -- the backward
 * filter of the causal/anticausal pairs of P:809-811 and P:866-868.  Same
 * arithmetic as oracle_eq1_i32 (Z/2^32) and oracle_eq1_f64_dd (fp64). */
void oracle_rev_i32(const int32_t* x, int32_t* y, int64_t n, const int64_t* a, int p, const int64_t* b, int k)
{
    for (int64_t i = n - 1; i >= 0; i--) {
        uint64_t acc = 0;
        for (int j = 0; j <= p; j++)
            if (i + j < n) acc += (uint64_t)a[j] * (uint64_t)(uint32_t)x[i + j];
        for (int j = 1; j <= k; j++)
            if (i + j < n) acc += (uint64_t)b[j - 1] * (uint64_t)(uint32_t)y[i + j];
        y[i] = (int32_t)(uint32_t)(acc & 0xffffffffu);
    }
}

void oracle_rev_f64(const double* x, double* y, int64_t n, const double* a, int p, const double* b, int k)
{
    for (int64_t i = n - 1; i >= 0; i--) {
        double acc = 0.0;
        for (int j = 0; j <= p; j++)
            if (i + j < n) acc += a[j] * x[i + j];
        for (int j = 1; j <= k; j++)
            if (i + j < n) acc += b[j - 1] * y[i + j];
        y[i] = acc;
    }
}

/* ---------------------------------------------------------------------- */
/* Correction-factor lists (Sec. 2.1)                            */
/* ---------------------------------------------------------------------- */

/* out: k lists of length k+m, row-major out[(r-1)*(k+m) + pos].  Positions
 * 0..k-1 are the seed ("extend ... by two elements on the left"),
 * written in memory order w_{m-k}, ..., w_{m-1} of the previous chunk, so the
 * list for carry w_{m-r} has its one at position k-r: for k = 2 list 1
 * starts "0, 1" and list 2 starts "1, 0".  Positions k..k+m-1
 * are the m correction factors produced by the recurrence (0: c)
 * (P:346-347). */
void oracle_factor_lists_i32(const int64_t* b, int k, int64_t m, int32_t* out)
{
    int64_t len = k + m;
    for (int r = 1; r <= k; r++) {
        int32_t* L = out + (int64_t)(r - 1) * len;
        for (int q = 0; q < k; q++) L[q] = (q == k - r) ? 1 : 0;
        for (int64_t i = k; i < len; i++) {
            uint64_t acc = 0;                    /* non-recursive term is 0 */
            for (int j = 1; j <= k; j++) {
                acc += (uint64_t)(uint32_t)b[j - 1] * (uint64_t)(uint32_t)L[i - j];
                acc &= 0xffffffffull;
            }
            L[i] = (int32_t)(uint32_t)acc;
        }
    }
}

void oracle_factor_lists_f64(const double* b, int k, int64_t m, double* out)
{
    int64_t len = k + m;
    for (int r = 1; r <= k; r++) {
        double* L = out + (int64_t)(r - 1) * len;
        for (int q = 0; q < k; q++) L[q] = (q == k - r) ? 1.0 : 0.0;
        for (int64_t i = k; i < len; i++) {
            double acc = 0.0;
            for (int j = 1; j <= k; j++) acc += b[j - 1] * L[i - j];
            L[i] = acc;
        }
    }
}

/* ---------------------------------------------------------------------- */
/* Phase 1 (Sec. 2.1) and Phase 2 (Sec. 2.2/2.3) on int32, Z/2^32           */
/* ---------------------------------------------------------------------- */

/* In place on w[0..n): the input of recurrence (3), i.e. t.  lists: output of
 * oracle_factor_lists_i32 with the same k and a length >= m.  Merges chunk
 * pairs while the chunk size is < m (so the result consists of chunks of size
 * m).  rows (may be NULL): receives a copy of w after each
 * iteration, rows[it*n + i].  Returns the number of iterations. */
int oracle_phase1_i32(int32_t* w, int64_t n, const int64_t* b, int k, int64_t m,
                      const int32_t* lists, int64_t list_len, int32_t* rows)
{
    (void)b;
    int it = 0;
    for (int64_t sz = 1; sz < m; sz *= 2) {
        /* each pair: first chunk [s, s+sz), second chunk [s+sz, s+2sz) */
        for (int64_t s = 0; s + sz < n; s += 2 * sz) {
            int64_t f_end = s + sz;                 /* one past first chunk */
            /* carries from the first chunk, read before any correction */
            uint32_t carry[16];
            for (int r = 1; r <= k; r++) {
                int64_t idx = f_end - r;            /* w_{m-r} */
                carry[r - 1] = (idx >= s) ? (uint32_t)w[idx] : 0u;
            }
            for (int64_t i = 0; i < sz && f_end + i < n; i++) {
                uint64_t acc = (uint32_t)w[f_end + i];
                for (int r = 1; r <= k; r++) {
                    uint32_t f = (uint32_t)lists[(int64_t)(r - 1) * list_len + k + i];
                    acc += (uint64_t)carry[r - 1] * (uint64_t)f;
                    acc &= 0xffffffffull;
                }
                w[f_end + i] = (int32_t)(uint32_t)acc;
            }
        }
        if (rows != NULL) memcpy(rows + (int64_t)it * n, w, (size_t)n * sizeof(int32_t));
        it++;
    }
    return it;
}

/* Phase 2 without pipelining: for chunks c = 1, 2, ... in order,
 * correct every element of chunk c with the last k values of chunk c-1
 * (already final).  w holds the Phase-1 result. */
void oracle_phase2_i32(int32_t* w, int64_t n, int k, int64_t m,
                       const int32_t* lists, int64_t list_len)
{
    for (int64_t s = m; s < n; s += m) {
        uint32_t carry[16];
        for (int r = 1; r <= k; r++) {
            int64_t idx = s - r;
            carry[r - 1] = (idx >= 0) ? (uint32_t)w[idx] : 0u;
        }
        for (int64_t i = 0; i < m && s + i < n; i++) {
            uint64_t acc = (uint32_t)w[s + i];
            for (int r = 1; r <= k; r++) {
                uint32_t f = (uint32_t)lists[(int64_t)(r - 1) * list_len + k + i];
                acc += (uint64_t)carry[r - 1] * (uint64_t)f;
                acc &= 0xffffffffull;
            }
            w[s + i] = (int32_t)(uint32_t)acc;
        }
    }
}

/* Carry precomputation: given the global carries of a chunk
 * (gc[r-1] = its w_{m-r}) and the local carries of the next chunk
 * (lc[r-1] = its local w_{m-r}), return that next chunk's global carries:
 * out[q-1] = lc[q-1] + sum_r gc[r-1] * factor_r[m-q]  (0-based position m-q
 * inside the m factors).  Example: 24 = 44 + 8*8 + (-7)*12. */
void oracle_carry_precompute_i32(const int32_t* gc, const int32_t* lc, int k,
                                 int64_t m, const int32_t* lists, int64_t list_len,
                                 int32_t* out)
{
    for (int q = 1; q <= k; q++) {
        uint64_t acc = (uint32_t)lc[q - 1];
        for (int r = 1; r <= k; r++) {
            uint32_t f = (uint32_t)lists[(int64_t)(r - 1) * list_len + k + (m - q)];
            acc += (uint64_t)(uint32_t)gc[r - 1] * (uint64_t)f;
            acc &= 0xffffffffull;
        }
        out[q - 1] = (int32_t)(uint32_t)acc;
    }
}
