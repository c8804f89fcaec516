"""CPU oracle for the PLR hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and ``--impl reference``) may import this package.  The
product package ``paper_conf_asplos_malekib18_b200`` never imports it, and the
two share no code: this module wraps ``oracle/plr_oracle.c`` (plain C,
compiled with gcc into ``oracle/liboracle.so``) with ctypes.

Citations ("P:n" = line n of the paper text):

* :func:`recurrence` -- Eq. (1) with zero initial conditions, the
  serial loop of P:206-214 over the split form Eq. (2)/(3); int32
  in the ring Z/2^32 (reading R1), float32 data in fp64 with coefficients
  ``(double)(float)c`` (reading R3).
* :func:`factor_lists` -- correction-factor lists, Sec. 2.1.
* :func:`phase1`, :func:`phase2`, :func:`carry_precompute` -- the paper's own
  two-phase algorithm, Sec. 2.1-2.3, step by step, used to
  reproduce the worked example.

Pins: tests/test_oracle.py.  Nothing here is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "plr_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile plr_oracle.c with gcc (plain -O2, no vectorisation flags)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            lib = ctypes.CDLL(_LIB)
            P = ctypes.c_void_p
            I64 = ctypes.c_int64
            I = ctypes.c_int
            lib.oracle_eq1_i32.argtypes = [P, P, I64, P, I, P, I, P, P]
            lib.oracle_eq1_f64.argtypes = [P, P, I64, P, I, P, I, P, P]
            lib.oracle_eq1_f64_dd.argtypes = [P, P, I64, P, I, P, I]
            lib.oracle_rev_i32.argtypes = [P, P, I64, P, I, P, I]
            lib.oracle_rev_f64.argtypes = [P, P, I64, P, I, P, I]
            lib.oracle_factor_lists_i32.argtypes = [P, I, I64, P]
            lib.oracle_factor_lists_f64.argtypes = [P, I, I64, P]
            lib.oracle_phase1_i32.argtypes = [P, I64, P, I, I64, P, I64, P]
            lib.oracle_phase1_i32.restype = I
            lib.oracle_phase2_i32.argtypes = [P, I64, I, I64, P, I64]
            lib.oracle_carry_precompute_i32.argtypes = [P, P, I, I64, P, I64, P]
            _lib = lib
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def f32c(c) -> np.ndarray:
    """The coefficient the GPU multiplies by: round to fp32, promote to fp64."""
    return np.asarray(c, dtype=np.float64).astype(np.float32).astype(np.float64)


def _int_coeffs(c) -> np.ndarray:
    arr = np.asarray(c, dtype=np.float64)
    if not np.all(arr == np.round(arr)):
        raise ValueError("integer recurrences need integer coefficients")
    return np.round(arr).astype(np.int64)


def recurrence(x, a, b, dtype: str, x_hist=None, y_hist=None, exact_coeffs: bool = False) -> np.ndarray:
    """Evaluate Eq. (1) sequentially.

    dtype "int32": x int32 -> y int32 (Z/2^32).  dtype "float32": x float32 ->
    y float64 (fp64 evaluation with fp32-rounded coefficients).
    x_hist: the p inputs before x[0] (index order); y_hist: the k outputs
    before y[0] (index order).  None means zero.
    exact_coeffs (float only): use the decimal coefficients in fp64 instead of
    their fp32 roundings -- a diagnostic for reading R3, not the parity target.
    """
    lib = _load()
    p, k = len(a) - 1, len(b)
    if dtype == "int32":
        x = np.ascontiguousarray(x, dtype=np.int32)
        y = np.empty(x.shape[0], dtype=np.int32)
        ai, bi = _int_coeffs(a), _int_coeffs(b)
        xh = None if x_hist is None else np.ascontiguousarray(x_hist, dtype=np.int32)
        yh = None if y_hist is None else np.ascontiguousarray(y_hist, dtype=np.int32)
        assert xh is None or xh.shape[0] == p
        assert yh is None or yh.shape[0] == k
        lib.oracle_eq1_i32(_ptr(x), _ptr(y), x.shape[0], _ptr(ai), p, _ptr(bi), k, _ptr(xh), _ptr(yh))
        return y
    if dtype == "float32":
        x = np.ascontiguousarray(x, dtype=np.float32)
        y = np.empty(x.shape[0], dtype=np.float64)
        if exact_coeffs:
            af, bf = np.asarray(a, dtype=np.float64), np.asarray(b, dtype=np.float64)
        else:
            af, bf = f32c(a), f32c(b)
        xh = None if x_hist is None else np.ascontiguousarray(x_hist, dtype=np.float32)
        yh = None if y_hist is None else np.ascontiguousarray(y_hist, dtype=np.float64)
        assert xh is None or xh.shape[0] == p
        assert yh is None or yh.shape[0] == k
        lib.oracle_eq1_f64(_ptr(x), _ptr(y), x.shape[0], _ptr(af), p, _ptr(bf), k, _ptr(xh), _ptr(yh))
        return y
    raise ValueError(dtype)


def cascade(x, stages, dtype: str) -> np.ndarray:
    """A cascade of signatures ("inputs that consist of multiple signatures",
    P:1851-1852; filters applied one after the other): stage s
    evaluates Eq. (1) with its own (a_s : b_s) on the previous stage's
    output, zero initial conditions.  int32: every stage in Z/2^32; float32:
    every stage in fp64 with its fp32-rounded coefficients, stage outputs
    not rounded in between.  stages: sequence of (a, b) pairs (b may be
    empty: a feed-forward stage)."""
    lib = _load()
    if dtype == "int32":
        y = np.ascontiguousarray(x, dtype=np.int32)
        for a, b in stages:
            y = recurrence(y, a, b, "int32")
        return y
    if dtype == "float32":
        y = np.ascontiguousarray(x, dtype=np.float32).astype(np.float64)
        for a, b in stages:
            af, bf = f32c(a), f32c(b)
            out = np.empty_like(y)
            lib.oracle_eq1_f64_dd(_ptr(y), _ptr(out), y.shape[0], _ptr(af), len(a) - 1,
                                  _ptr(bf) if len(bf) else None, len(bf))
            y = out
        return y
    raise ValueError(dtype)


def anticausal(x, a, b, dtype: str) -> np.ndarray:
    """The anticausal recurrence (Eq. (1) run from the end, zero beyond it;
    P:809-811).  int32 in Z/2^32; float32 input (or the fp64
    output of a previous stage) evaluated in fp64 with fp32-rounded
    coefficients."""
    lib = _load()
    if dtype == "int32":
        x = np.ascontiguousarray(x, dtype=np.int32)
        y = np.empty_like(x)
        ai, bi = _int_coeffs(a), _int_coeffs(b)
        lib.oracle_rev_i32(_ptr(x), _ptr(y), x.shape[0], _ptr(ai), len(a) - 1, _ptr(bi) if len(bi) else None, len(bi))
        return y
    if dtype == "float32":
        xd = np.ascontiguousarray(x, dtype=np.float64)
        y = np.empty_like(xd)
        af, bf = f32c(a), f32c(b)
        lib.oracle_rev_f64(_ptr(xd), _ptr(y), xd.shape[0], _ptr(af), len(a) - 1, _ptr(bf) if len(bf) else None, len(bf))
        return y
    raise ValueError(dtype)


def bidirectional(x, a, b, dtype: str) -> np.ndarray:
    """Forward-backward (zero-phase) filtering: the anticausal recurrence of
    the causal one's output (intermediate unrounded for float32)."""
    return anticausal(recurrence(x, a, b, dtype), a, b, dtype)


def factor_lists(b, m: int, dtype: str) -> np.ndarray:
    """k seed-extended correction-factor lists of length k+m (Sec. 2.1).

    Row r-1 is the list for carry w_{m-r}; columns 0..k-1 are the seed in
    memory order, columns k.. the m factors.
    """
    lib = _load()
    k = len(b)
    if dtype == "int32":
        bi = _int_coeffs(b)
        out = np.empty((k, k + m), dtype=np.int32)
        lib.oracle_factor_lists_i32(_ptr(bi), k, m, _ptr(out))
        return out
    bf = np.asarray(b, dtype=np.float64) if dtype == "float64" else f32c(b)
    out = np.empty((k, k + m), dtype=np.float64)
    lib.oracle_factor_lists_f64(_ptr(bf), k, m, _ptr(out))
    return out


def phase1(t, b, m: int):
    """Phase 1 merging up to chunk size m (int32).  Returns (w, rows)."""
    lib = _load()
    w = np.array(t, dtype=np.int32)
    n, k = w.shape[0], len(b)
    lists = factor_lists(b, m, "int32")
    iters = max(0, int(np.ceil(np.log2(m)))) if m > 1 else 0
    rows = np.zeros((max(iters, 1), n), dtype=np.int32)
    bi = _int_coeffs(b)
    it = lib.oracle_phase1_i32(_ptr(w), n, _ptr(bi), k, m, _ptr(lists), lists.shape[1], _ptr(rows))
    return w, rows[:it]


def phase2(w, b, m: int) -> np.ndarray:
    """Phase 2 (unpipelined) over chunks of size m, in place on a copy."""
    lib = _load()
    w = np.array(w, dtype=np.int32)
    lists = factor_lists(b, m, "int32")
    lib.oracle_phase2_i32(_ptr(w), w.shape[0], len(b), m, _ptr(lists), lists.shape[1])
    return w


def carry_precompute(gc, lc, b, m: int) -> np.ndarray:
    lib = _load()
    k = len(b)
    lists = factor_lists(b, m, "int32")
    gc = np.ascontiguousarray(gc, dtype=np.int32)
    lc = np.ascontiguousarray(lc, dtype=np.int32)
    out = np.empty(k, dtype=np.int32)
    lib.oracle_carry_precompute_i32(_ptr(gc), _ptr(lc), k, m, _ptr(lists), lists.shape[1], _ptr(out))
    return out
