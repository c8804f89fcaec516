"""C-ABI checks that need no GPU: the library loads, exports every symbol of
include/plr.h, validates signatures, and its host-side
planner reproduces the paper's correction factors (worked example
P:584-586, n-nacci P:350-361) against the independent oracle."""
import ctypes
import re
import struct

import numpy as np
import pytest

import oracle
import workloads
from conftest import ROOT, read_golden

plr = pytest.importorskip("paper_conf_asplos_malekib18_b200")


def header_symbols():
    src = open(ROOT + "/include/plr.h").read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(plr_[a-z_0-9]+)\s*\(", src)))


def test_exports_every_declared_symbol():
    syms = header_symbols()
    assert len(syms) >= 18
    for s in syms:
        assert hasattr(plr.lib, s), s
    assert set(syms) == set(plr.binding.EXPORTED)
    assert plr.abi_version() == 4


@pytest.mark.parametrize("a,b,dtype,code", [
    ((1,), (), "int32", 2),                 # k = 0: a map, excluded
    ((0,), (1,), "int32", 2),               # last non-recursive coefficient 0
    ((1,), (1, 0), "int32", 2),             # trailing zero feedback coefficient
    ((1, 0), (1,), "int32", 2),             # trailing zero feed-forward coefficient
    ((1.5,), (1,), "int32", 2),             # non-integer for PLR_INT32
    ((1,), (1, 1, 1, 1, 1), "int32", 4),    # k > PLR_MAX_K
    ((1, 1, 1, 1, 1), (1,), "float32", 4),  # p > PLR_MAX_P
    ((float("nan"),), (0.5,), "float32", 2),
])
def test_signature_validation(a, b, dtype, code):
    with pytest.raises(plr.PLRError) as e:
        plr.Plan(a, b, dtype, n_max=0)
    assert e.value.status == code


def test_classes():
    cls = {s.name: plr.Plan(s.a, s.b, s.dtype, n_max=0).info["cls"] for s in workloads.TABLE1}
    assert cls["prefix"] == "ONES"
    assert cls["tuple2"] == cls["tuple3"] == "PERM"
    assert cls["order2"] == cls["order3"] == "POLY"
    for nm in ("lp1", "lp2", "lp3", "hp1", "hp2", "hp3"):
        assert cls[nm] == "DECAY"
    assert plr.Plan((1.0,), (1.0,), "float32", n_max=0).info["cls"] == "FLOAT"


def test_precision_rule_r16():
    """DESIGN.md reading R16: fp64 accumulation when the a-priori fp32 bound
    eps32 sum|a| (sum|g|)^2 / min(1, |H(-1)|) exceeds 1e-3.  Closed forms for
    (a0: c) with the pole 0.8 of multiplicity s (LP_s, Table 1):
    sum|g| = 0.2^-s and |H(-1)| = a0 / 1.8^s."""
    eps = 2.0 ** -24
    for name, s in (("lp1", 1), ("lp2", 2), ("lp3", 3)):
        sig = workloads.BY_NAME[name]
        info = plr.Plan(sig.a, sig.b, sig.dtype, n_max=0).info
        a0 = float(np.float32(sig.a[0]))
        bound = eps * a0 * (0.2 ** -s) ** 2 / min(1.0, a0 / 1.8 ** s)
        assert info["cond_bound"] == pytest.approx(bound, rel=1e-4), name
    acc = {s.name: plr.Plan(s.a, s.b, s.dtype, n_max=0).info["acc_bits"] for s in workloads.TABLE1}
    assert acc == {"prefix": 32, "tuple2": 32, "tuple3": 32, "order2": 32, "order3": 32,
                   "lp1": 32, "lp2": 32, "lp3": 64, "hp1": 32, "hp2": 32, "hp3": 64}


def test_decay_length_matches_ftz_threshold():
    """(1: 0.8): g_u = 0.8^u (fp32 coefficient) drops below FLT_MIN, where it
    is flushed, after u = floor(log(FLT_MIN)/log(c))."""
    c = float(np.float32(0.8))
    expect = int(np.floor(np.log(np.finfo(np.float32).tiny) / np.log(c)))
    assert plr.Plan((0.2,), (0.8,), "float32", n_max=0).info["decay_len"] == expect


def test_planner_factor_lists_worked_example():
    g = read_golden("worked_example.txt")
    L = plr.Plan((1,), (2, -1), "int32", n_max=0).factor_lists(8)
    assert L[0].tolist() == g["list1"] and L[1].tolist() == g["list2"]


def test_planner_factor_lists_nnacci():
    o = read_golden("nnacci.txt")
    L = plr.Plan((1,), (1, 1, 1), "int32", n_max=0).factor_lists(17)
    assert L[0].tolist() == o["A000073"][:20]
    assert L[1].tolist() == o["A001590"][:20]
    assert L[2].tolist() == [1] + o["A000073"][:19]


@pytest.mark.parametrize("sig", workloads.TABLE1, ids=lambda s: s.name)
def test_planner_factor_lists_vs_oracle(sig):
    """Planner (matrix powers) vs oracle (n-nacci iteration) over 600 factors."""
    m = 600
    L = plr.Plan(sig.a, sig.b, sig.dtype, n_max=0).factor_lists(m)
    ref = oracle.factor_lists(sig.b, m, sig.dtype)
    if sig.dtype == "int32":
        assert np.array_equal(L, ref)
    else:
        r32 = ref.astype(np.float32)
        r32[np.abs(r32) < np.finfo(np.float32).tiny] = 0           # FTZ
        np.testing.assert_allclose(L, r32, rtol=2e-6, atol=0)


def _payload(n, x_tail, y_tail, dtype):
    npdt = np.int32 if dtype == "int32" else np.float32
    xt = np.zeros(4, npdt)
    yt = np.zeros(4, npdt)
    if len(x_tail):
        xt[4 - len(x_tail):] = x_tail
    if len(y_tail):
        yt[4 - len(y_tail):] = y_tail
    return struct.pack("<Q", n) + xt.tobytes() + yt.tobytes() + bytes(24)


@pytest.mark.parametrize("sig", workloads.TABLE1, ids=lambda s: s.name)
def test_combine_host_matches_oracle(sig):
    """The segment prefix z_{r+1} = M^{n_r} z_r + payload_r reproduces the
    true boundary history (reading R12) for uneven segments, incl. n_r < k."""
    sizes = [5000, 3, 1777, 0, 4096, 1]
    x = workloads.host_input(sum(sizes), sig.dtype, 11)
    yfull = oracle.recurrence(x, sig.a, sig.b, sig.dtype)
    plan = plr.Plan(sig.a, sig.b, sig.dtype, n_max=0)
    pls = b""
    off = 0
    for nr in sizes:
        seg = x[off:off + nr]
        yz = oracle.recurrence(seg, sig.a, sig.b, sig.dtype)     # zero history
        if sig.dtype == "float32":
            yz = yz.astype(np.float32)
        pls += _payload(nr, seg[-4:] if nr else [], yz[-4:] if nr else [], sig.dtype)
        off += nr
    starts = np.cumsum([0] + sizes)
    for r in range(len(sizes)):
        hist = plan.combine_host(pls, r, len(sizes))
        npdt = np.int32 if sig.dtype == "int32" else np.float32
        h = np.frombuffer(hist, dtype=npdt)
        s = starts[r]
        ex_x = np.array([x[s - 4 + i] if s - 4 + i >= 0 else 0 for i in range(4)], dtype=npdt)
        ex_y = np.array([yfull[s - 4 + i] if s - 4 + i >= 0 else 0 for i in range(4)])
        assert np.array_equal(h[:4], ex_x)
        if sig.dtype == "int32":
            assert np.array_equal(h[4:], ex_y.astype(np.int32))
        else:
            np.testing.assert_allclose(h[4:], ex_y, rtol=1e-5, atol=1e-5)


# ------------------------------------------------------------ cascade ------
def test_cascade_combines_polynomials():
    """plr_plan_create_cascade multiplies the stages' z-transforms:
    three prefix sums -> (1: 3, -3, 1); a FIR stage with a tuple
    sum and a 2nd-order sum -> (3, -1 : 2, 0, -2, 1) in Z/2^32; three 1-stage
    high-pass filters -> the untruncated 3-stage high-pass row (reading R4)."""
    pl = plr.Plan.cascade([((1,), (1,))] * 3, "int32", n_max=0)
    assert (pl.p, pl.k) == (0, 3)
    assert pl.a == (1.0,) and pl.b == (3.0, float(2 ** 32 - 3), 1.0)
    pl = plr.Plan.cascade([((3, -1), (0, 1)), ((1,), (2, -1))], "int32", n_max=0)
    assert pl.a == (3.0, float(2 ** 32 - 1)) and pl.b == (2.0, 0.0, float(2 ** 32 - 2), 1.0)
    pl = plr.Plan.cascade([((0.9, -0.9), (0.8,))] * 3, "float32", n_max=0)
    hp3 = workloads.BY_NAME["hp3"]
    np.testing.assert_allclose(pl.a, hp3.a, rtol=1e-6)
    np.testing.assert_allclose(pl.b, hp3.b, rtol=1e-6)
    assert pl.info["cls"] == "DECAY"


@pytest.mark.parametrize("stages,code", [
    ([((1,), ())], 2),                                   # no feedback stage at all
    ([((1,), (1, 0))], 2),                               # a stage's trailing zero
    ([((1,), (1,))] * 5, 4),                             # combined k = 5 > PLR_MAX_K
    ([((1, 1), (1,))] * 4, 4),                           # combined p = 4 > PLR_MAX_P
])
def test_cascade_validation(stages, code):
    with pytest.raises(plr.PLRError) as e:
        plr.Plan.cascade(stages, "int32", n_max=0)
    assert e.value.status == code


def test_map_floor_reading_r20():
    """Reading R20: every Table-1 float row has an fp32-data floor
    eps32 sum|a| sum|g| / min(1, |H(-1)|) below the 1e-4 bar, so the
    worked example's (-1)^i (i+3) input is a fair parity input for all of
    them; a filter with a zero at the Nyquist frequency has no finite floor."""
    for s in workloads.TABLE1:
        if s.dtype == "float32":
            info = plr.Plan(s.a, s.b, s.dtype, n_max=0).info
            assert info["map_floor"] <= 1e-4, (s.name, info["map_floor"])
    lp3 = plr.Plan((0.008,), (2.4, -1.92, 0.512), "float32", n_max=0).info
    assert lp3["nyquist_gain"] == pytest.approx(0.008 / 5.832, rel=1e-5)
    assert plr.Plan((0.25, 0.5, 0.25), (0.8,), "float32", n_max=0).info["map_floor"] == float("inf")


def test_plan_info_layout_host_only():
    """plr_plan_info as the binding reads it (ctypes mirror of include/plr.h,
    ABI 4): the fields after the doubles land where the C struct puts them.
    A host-only plan reports the small-n cluster size (a compile-time
    constant), no device state (0 clusters, 0 CTAs/SM, small_max 0)."""
    info = plr.Plan((1,), (2, -1), "int32", n_max=0).info
    assert info["small_cluster_ctas"] == 4
    assert info["small_clusters"] == 0 and info["small_ctas_per_sm"] == 0 and info["small_max"] == 0
    assert info["k"] == 2 and info["p"] == 0 and info["cls"] == "POLY"
    assert info["nyquist_gain"] == 0.0 and info["map_floor"] == 0.0
