"""Pins of the CPU oracle against what the paper and mathematics fix (no GPU).

Each test names the passage it follows.  The oracle is pinned here, before
and independently of any CUDA code: worked example, n-nacci
identities (OEIS), closed forms, scipy.signal.lfilter, exact
big-integer evaluation, a dense lower-triangular solve, DC gains, linearity,
shift invariance and the segment-split invariant.
"""
import math

import numpy as np
import pytest

import oracle
import workloads
from conftest import read_golden

M32 = 1 << 32


def wrap32(v):
    v %= M32
    return v - M32 if v >= (1 << 31) else v


# ---------------------------------------------------------------- P1 -------
def test_worked_example_output():
    g = read_golden("worked_example.txt")
    y = oracle.recurrence(np.array(g["input"]), (1,), (2, -1), "int32")
    assert y.tolist() == g["expected_output"]


def test_worked_example_factor_lists():
    g = read_golden("worked_example.txt")
    L = oracle.factor_lists((2, -1), 8, "int32")
    assert L[0].tolist() == g["list1"]
    assert L[1].tolist() == g["list2"]


def test_worked_example_phase1_rows_and_phase2():
    g = read_golden("worked_example.txt")
    w, rows = oracle.phase1(np.array(g["input"]), (2, -1), 8)
    assert rows.shape[0] == 3
    assert rows[0].tolist() == g["phase1_iter1"]
    assert rows[1].tolist() == g["phase1_iter2"]
    assert rows[2].tolist() == g["phase1_iter3"]
    fin = oracle.phase2(w, (2, -1), 8)
    assert fin[:8].tolist() == g["final_chunk0"]
    assert fin[8:16].tolist() == g["final_chunk1"]
    assert fin[16:].tolist() == g["final_chunk2"]
    assert fin.tolist() == g["expected_output"]


def test_worked_example_carry_precompute():
    g = read_golden("worked_example.txt")
    out = oracle.carry_precompute(g["chunk1_global_carries"], g["chunk2_local_carries"], (2, -1), 8)
    assert out.tolist() == g["chunk2_global_carries"]          # (16, 24)


# ---------------------------------------------------------------- P2 -------
def test_nnacci_fibonacci():
    o = read_golden("nnacci.txt")
    L = oracle.factor_lists((1, 1), 18, "int32")
    fib = o["A000045"]
    assert L[0].tolist() == fib[:20]                           # "0, 1" start
    assert L[1].tolist() == [1] + fib[:19]                     # "1, 0" start: shifted by one


def test_nnacci_tribonacci():
    o = read_golden("nnacci.txt")
    L = oracle.factor_lists((1, 1, 1), 17, "int32")
    assert L[0].tolist() == o["A000073"][:20]                  # "0, 0, 1"
    assert L[1].tolist() == o["A001590"][:20]                  # "0, 1, 0": the different one
    assert L[2].tolist() == [1] + o["A000073"][:19]            # "1, 0, 0": shifted by one


# ---------------------------------------------------------------- P3 -------
@pytest.mark.parametrize("b", [(2, -1), (3, -3, 1), (0, 1), (0, 0, 1), (1, 1), (1, 2)])
def test_first_last_list_shift_relation(b):
    """the first and last lists hold the same values shifted by one
    position; in detail list_k[i] = c_k * list_1[i-1] over the m factors."""
    k, m = len(b), 64
    L = oracle.factor_lists(b, m, "int32").astype(np.int64)
    for i in range(k, k + m):
        assert wrap32(int(L[k - 1][i])) == wrap32(b[-1] * int(L[0][i - 1]))


def test_first_order_factors_are_powers():
    """(1: d) -> factors d, d^2, ..., d^m with a leading 1."""
    L = oracle.factor_lists((0.8,), 30, "float64")
    assert L[0][0] == 1.0
    np.testing.assert_allclose(L[0][1:], 0.8 ** np.arange(1, 31), rtol=1e-14)


def test_second_order_factor_closed_forms():
    """(1: d, e): d, d^2+e, d^3+2de, d^4+3d^2e+e^2 and e, de, d^2e+e^2,
    d^3e+2de^2."""
    d, e = 0.7, -0.3
    L = oracle.factor_lists((d, e), 4, "float64")
    np.testing.assert_allclose(L[0][2:], [d, d * d + e, d ** 3 + 2 * d * e, d ** 4 + 3 * d * d * e + e * e], rtol=1e-14)
    np.testing.assert_allclose(L[1][2:], [e, d * e, d * d * e + e * e, d ** 3 * e + 2 * d * e * e], rtol=1e-14)


# ---------------------------------------------------------------- P4 -------
def test_closed_forms_on_ones():
    """Prefix sums of ones: i+1; 2nd order: C(i+2,2); 3rd order: C(i+3,3),
    all mod 2^32 (binomial signatures).  n large enough that
    C(i+3,3) wraps."""
    n = 1 << 20
    x = np.ones(n, dtype=np.int32)
    i = np.arange(n, dtype=np.uint64)
    exp1 = (i + 1)
    exp2 = ((i + 1) * (i + 2) // 2)
    exp3 = ((i + 1) * (i + 2) * (i + 3) // 6)                 # < 2^61, exact in uint64
    for b, e in (((1,), exp1), ((2, -1), exp2), ((3, -3, 1), exp3)):
        y = oracle.recurrence(x, (1,), b, "int32")
        assert np.array_equal(y.view(np.uint32), (e % M32).astype(np.uint32))


# ---------------------------------------------------------------- P5/P6 ----
@pytest.mark.parametrize("s", [2, 3])
def test_tuple_prefix_is_per_lane_cumsum(s):
    """Tuple prefix sums (b-s = 1, others 0) are independent scans of each
    lane."""
    x = workloads.host_input(10007, "int32", 1)
    b = tuple([0] * (s - 1) + [1])
    y = oracle.recurrence(x, (1,), b, "int32")
    for lane in range(s):
        assert np.array_equal(y[lane::s], np.cumsum(x[lane::s], dtype=np.int32))


@pytest.mark.parametrize("order,b", [(2, (2, -1)), (3, (3, -3, 1))])
def test_higher_order_is_repeated_cumsum(order, b):
    """Higher-order prefix sums are prefix sums of prefix sums."""
    x = workloads.host_input(4096, "int32", 2)
    ref = x.copy()
    for _ in range(order):
        ref = np.cumsum(ref, dtype=np.int32)
    assert np.array_equal(oracle.recurrence(x, (1,), b, "int32"), ref)


# ---------------------------------------------------------------- P7 -------
def test_impulse_response_lp1():
    """Impulse response of (0.2: 0.8) is 0.2 * 0.8^i (north_star pin)."""
    x = workloads.structured_input("impulse", 200, "float32")
    y = oracle.recurrence(x, (0.2,), (0.8,), "float32")
    c = oracle.f32c([0.2, 0.8])
    np.testing.assert_allclose(y, c[0] * c[1] ** np.arange(200), rtol=1e-12, atol=0)


def test_impulse_response_lp2_lp3_closed_forms():
    """Repeated real poles: (g/(1-rz^-1)^s) has impulse response
    g*C(i+s-1, s-1)*r^i.  With exact coefficients these are the 2- and 3-stage
    low-pass rows of Table 1."""
    n = 300
    x = np.zeros(n, dtype=np.float32)
    x[0] = 1
    i = np.arange(n)
    # decimal coefficients in fp64 (the fp32 rounding of a repeated pole
    # splits it, which is reading R3's business, not this pin's)
    y2 = oracle.recurrence(x, (0.04,), (1.6, -0.64), "float32", exact_coeffs=True)
    y3 = oracle.recurrence(x, (0.008,), (2.4, -1.92, 0.512), "float32", exact_coeffs=True)
    np.testing.assert_allclose(y2, 0.04 * (i + 1) * 0.8 ** i, rtol=1e-9, atol=0)
    np.testing.assert_allclose(y3, 0.008 * (i + 1) * (i + 2) / 2 * 0.8 ** i, rtol=1e-9, atol=0)


# ---------------------------------------------------------------- P8 -------
@pytest.mark.parametrize("sig", [s for s in workloads.TABLE1 if s.dtype == "float32"], ids=lambda s: s.name)
def test_float_matches_scipy_lfilter(sig):
    """scipy.signal.lfilter(a, [1, -b-1, ..., -b-k], x) evaluates Eq. (1)
    (note the sign convention of the denominator)."""
    from scipy.signal import lfilter
    x = workloads.host_input(50000, "float32", 3)
    a = oracle.f32c(sig.a)
    b = oracle.f32c(sig.b)
    ref = lfilter(a, np.concatenate([[1.0], -b]), x.astype(np.float64))
    y = oracle.recurrence(x, sig.a, sig.b, "float32")
    np.testing.assert_allclose(y, ref, rtol=0, atol=1e-12)


@pytest.mark.parametrize("sig", [s for s in workloads.TABLE1 if s.dtype == "int32"], ids=lambda s: s.name)
def test_int_small_values_match_lfilter(sig):
    """Without wraparound the int recurrence is the rational filter; small
    inputs and short n keep every value exact in fp64."""
    from scipy.signal import lfilter
    rng = np.random.default_rng(4)
    x = rng.integers(-3, 4, size=60).astype(np.int32)
    ref = lfilter(np.array(sig.a, float), np.concatenate([[1.0], -np.array(sig.b, float)]), x.astype(float))
    y = oracle.recurrence(x, sig.a, sig.b, "int32")
    assert np.all(np.abs(ref) < 2 ** 31)
    assert np.array_equal(y, np.round(ref).astype(np.int64))


# ---------------------------------------------------------------- P9 -------
@pytest.mark.parametrize("sig", workloads.TABLE1, ids=lambda s: s.name)
def test_brute_force_lower_triangular(sig):
    """y = B^-1 A x with banded lower-triangular Toeplitz A[i][i-j] = a_{-j}
    and B = I - sum_j b_{-j} S^j.  Float: dense fp64 solve.  Int: exact
    big-integer evaluation with no wraparound, reduced mod 2^32 only at the
    end (Z -> Z/2^32 is a ring homomorphism, reading R1)."""
    N = 160
    if sig.dtype == "float32":
        x = workloads.host_input(N, "float32", 5)
        a, b = oracle.f32c(sig.a), oracle.f32c(sig.b)
        A = np.zeros((N, N))
        B = np.eye(N)
        for j, aj in enumerate(a):
            A += aj * np.eye(N, k=-j)
        for j, bj in enumerate(b, start=1):
            B -= bj * np.eye(N, k=-j)
        ref = np.linalg.solve(B, A @ x.astype(np.float64))
        y = oracle.recurrence(x, sig.a, sig.b, "float32")
        np.testing.assert_allclose(y, ref, rtol=0, atol=1e-10)
    else:
        x = workloads.host_input(N, "int32", 5)
        a = [int(v) for v in sig.a]
        b = [int(v) for v in sig.b]
        yy = []
        for i in range(N):                      # exact integers, no wrap
            acc = sum(a[j] * int(x[i - j]) for j in range(len(a)) if i - j >= 0)
            acc += sum(b[j - 1] * yy[i - j] for j in range(1, len(b) + 1) if i - j >= 0)
            yy.append(acc)
        ref = [wrap32(v) for v in yy]
        assert max(abs(v) for v in yy) > 2 ** 40 or sig.name in ("prefix", "tuple2", "tuple3")
        assert oracle.recurrence(x, sig.a, sig.b, "int32").tolist() == ref


# ---------------------------------------------------------------- P10 ------
@pytest.mark.parametrize("sig", [s for s in workloads.TABLE1 if s.dtype == "float32"], ids=lambda s: s.name)
def test_dc_gain(sig):
    """Step response settles at A(1)/B(1): 1 for the low-pass rows, 0 for the
    high-pass rows (Smith's filter design)."""
    x = np.ones(6000, dtype=np.float32)
    y = oracle.recurrence(x, sig.a, sig.b, "float32")
    a, b = oracle.f32c(sig.a), oracle.f32c(sig.b)
    gain = a.sum() / (1.0 - b.sum())
    assert abs(y[-1] - gain) < 1e-9
    target = 1.0 if sig.name.startswith("lp") else 0.0
    assert abs(gain - target) < 1e-4      # fp32-rounded coefficients, R3


def test_printed_hp3_has_pole_at_one():
    """Reading R4: the printed (truncated) 3-stage high-pass feedback
    coefficients sum to one, so B(1) = 0 and the filter is not stable."""
    assert abs(1.0 - sum(workloads.HP3_PRINTED.b)) < 1e-12
    assert abs(1.0 - sum(workloads.BY_NAME["hp3"].b) - 0.008) < 1e-12


# ---------------------------------------------------------------- P11 ------
@pytest.mark.parametrize("sig", [s for s in workloads.TABLE1 if s.dtype == "int32"], ids=lambda s: s.name)
def test_linearity_mod_2_32(sig):
    x1 = workloads.host_input(3000, "int32", 6)
    x2 = workloads.host_input(3000, "int32", 7)
    s = (x1.astype(np.int64) * 3 + x2.astype(np.int64) * -5).astype(np.int32)   # wraps
    y = oracle.recurrence(s, sig.a, sig.b, "int32").astype(np.int64)
    y1 = oracle.recurrence(x1, sig.a, sig.b, "int32").astype(np.int64)
    y2 = oracle.recurrence(x2, sig.a, sig.b, "int32").astype(np.int64)
    assert np.array_equal(y.astype(np.int32), (3 * y1 - 5 * y2).astype(np.int32))


@pytest.mark.parametrize("sig", workloads.TABLE1, ids=lambda s: s.name)
def test_shift_invariance(sig):
    """Prepending zeros shifts the output (zero initial conditions)."""
    x = workloads.host_input(2000, sig.dtype, 8)
    z = np.concatenate([np.zeros(37, dtype=x.dtype), x])
    y = oracle.recurrence(x, sig.a, sig.b, sig.dtype)
    yz = oracle.recurrence(z, sig.a, sig.b, sig.dtype)
    assert np.all(yz[:37] == 0)
    assert np.array_equal(yz[37:], y)


# ---------------------------------------------------------------- P12 ------
@pytest.mark.parametrize("sig", workloads.TABLE1, ids=lambda s: s.name)
def test_history_split_invariant(sig):
    """Evaluating x_A || x_B in one call equals evaluating x_A, then x_B with
    the history (last p inputs, last k outputs) carried over (reading R12)."""
    x = workloads.host_input(5000, sig.dtype, 9)
    cut = 1777
    y = oracle.recurrence(x, sig.a, sig.b, sig.dtype)
    ya = oracle.recurrence(x[:cut], sig.a, sig.b, sig.dtype)
    xh = x[cut - sig.p:cut] if sig.p else None
    yb = oracle.recurrence(x[cut:], sig.a, sig.b, sig.dtype, x_hist=xh, y_hist=ya[cut - sig.k:cut])
    assert np.array_equal(np.concatenate([ya, yb]), y)


def test_zero_length_and_short():
    for sig in workloads.TABLE1:
        assert oracle.recurrence(np.zeros(0, np.float32 if sig.dtype == "float32" else np.int32),
                                 sig.a, sig.b, sig.dtype).shape == (0,)
    y = oracle.recurrence(np.array([5, 7], np.int32), (1,), (3, -3, 1), "int32")
    assert y.tolist() == [5, 7 + 15]


# ---------------------------------------------------------------- cascade --
def test_cascade_of_prefix_sums_is_binomial():
    """Three cascaded prefix sums (1: 1) on ones give C(i+3, 3) mod 2^32 --
    the 3rd-order prefix sum (binomial signatures) as a
    multi-signature input."""
    n = 3000
    i = np.arange(n, dtype=object)
    y = oracle.cascade(np.ones(n, np.int32), [((1,), (1,))] * 3, "int32")
    expect = [wrap32(int(v)) for v in (i + 1) * (i + 2) * (i + 3) // 6]
    assert y.tolist() == expect


def test_cascade_int_matches_composed_signature_bitwise():
    """Z/2^32 is a ring: a cascade equals the single signature with the
    multiplied polynomials, bit for bit (full-range inputs, wraparound)."""
    x = workloads.host_input(5000, "int32", 3)
    y = oracle.cascade(x, [((3, -1), (0, 1)), ((1,), (2, -1))], "int32")
    # (3 - z^-1) / ((1 - z^-2)(1 - 2 z^-1 + z^-2)) = (3, -1 : 2, 0, -2, 1)
    assert np.array_equal(y, oracle.recurrence(x, (3, -1), (2, 0, -2, 1), "int32"))


def test_cascade_lp1_twice_impulse_closed_form():
    """(0.2: 0.8) twice: impulse response 0.04 (i+1) 0.8^i (the LP2 row's
    closed form, with the fp32-rounded coefficients)."""
    n = 300
    x = np.zeros(n, np.float32)
    x[0] = 1
    y = oracle.cascade(x, [((0.2,), (0.8,))] * 2, "float32")
    a, c = float(np.float32(0.2)), float(np.float32(0.8))
    i = np.arange(n)
    np.testing.assert_allclose(y, a * a * (i + 1) * c ** i, rtol=1e-12, atol=0)


def test_cascade_float_matches_scipy_composed():
    """Stage by stage (oracle) vs scipy.signal.lfilter with the convolved
    numerator and denominator polynomials of the same fp32-rounded stages."""
    signal = pytest.importorskip("scipy.signal")
    stages = [((0.9, -0.9), (0.8,)), ((0.9, -0.9), (0.8,)), ((0.04,), (1.6, -0.64))]
    x = workloads.host_input(20000, "float32", 4)
    num, den = np.array([1.0]), np.array([1.0])
    for a, b in stages:
        num = np.convolve(num, oracle.f32c(a))
        den = np.convolve(den, np.concatenate([[1.0], -oracle.f32c(b)]))
    ref = signal.lfilter(num, den, x.astype(np.float64))
    y = oracle.cascade(x, stages, "float32")
    np.testing.assert_allclose(y, ref, rtol=1e-9, atol=1e-12)


# ------------------------------------------------------------ anticausal ---
def test_anticausal_closed_forms_on_ones():
    """Backward prefix sums of ones: (1: 1) -> n - i, (1: 2, -1) -> C(n-i+1, 2)
    (the binomial signatures of P:140-143, run from the end)."""
    n = 5000
    i = np.arange(n, dtype=np.int64)
    x = np.ones(n, np.int32)
    assert oracle.anticausal(x, (1,), (1,), "int32").tolist() == (n - i).tolist()
    assert oracle.anticausal(x, (1,), (2, -1), "int32").tolist() == ((n - i + 1) * (n - i) // 2).tolist()


def test_anticausal_is_time_reversal_of_causal():
    """Reversing time maps the anticausal recurrence onto Eq. (1): checked
    against the causal oracle on reversed full-range / float inputs."""
    for dtype, a, b in (("int32", (3, -1, 2), (2, -1)), ("float32", (0.729, -2.187, 2.187, -0.729), (2.4, -1.92, 0.512))):
        x = workloads.host_input(3000, dtype, 8)
        y = oracle.anticausal(x, a, b, dtype)
        r = oracle.recurrence(x[::-1].copy(), a, b, dtype)[::-1]
        if dtype == "int32":
            assert np.array_equal(y, r)
        else:
            np.testing.assert_allclose(y, r, rtol=1e-12, atol=1e-12)


def test_bidirectional_lp1_impulse_is_symmetric_closed_form():
    """Zero-phase LP1: an impulse far from both ends gives
    z_i = a^2 r^|i-c| / (1 - r^2) (the autocorrelation of a r^i), symmetric
    about the impulse; a, r the fp32-rounded 0.2 and 0.8."""
    n, c = 2000, 1000
    x = np.zeros(n, np.float32)
    x[c] = 1
    z = oracle.bidirectional(x, (0.2,), (0.8,), "float32")
    a, r = float(np.float32(0.2)), float(np.float32(0.8))
    i = np.arange(n)
    sel = np.abs(i - c) < 300
    np.testing.assert_allclose(z[sel], (a * a * r ** np.abs(i - c) / (1 - r * r))[sel], rtol=1e-9, atol=1e-15)


def test_bidirectional_prefix_closed_form():
    """Forward then backward prefix sum of ones: sum_{j>=i} (j+1) =
    (n(n+1) - i(i+1)) / 2, mod 2^32."""
    n = 100000
    i = np.arange(n, dtype=object)
    z = oracle.bidirectional(np.ones(n, np.int32), (1,), (1,), "int32")
    assert z.tolist() == [wrap32(int(v)) for v in (n * (n + 1) - i * (i + 1)) // 2]
