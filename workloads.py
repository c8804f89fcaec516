"""Seeded synthetic workloads shared by the tests, smoke() and bench.py.

This module holds INPUTS only: the Table-1 signatures as data and seeded
random-number recipes.  It contains none of the method's arithmetic, so both
the oracle side and the CUDA side may use it without sharing code.

Signatures are Table 1 of the paper, in the paper's signature
notation (a0, a-1, ..., a-p : b-1, ..., b-k).  The 3-stage high-pass
row is printed "truncated for improved readability"; the printed
values place a pole at z = 1 (2.4 - 1.9 + 0.5 = 1).  We use the untruncated
Smith values (0.729, -2.187, 2.187, -0.729 : 2.4, -1.92, 0.512), the triple
pole 0.8 that matches the untruncated 3-stage low-pass row
(reading R4).

Input recipe: the paper states values do not affect
performance; int32 inputs are uniform over the full 32-bit range
(exercising wraparound), float32 inputs are uniform in [-1, 1).  Seeds are
``SEED_BASE + 1000*cfg + rank``.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

SEED_BASE = 20180324


@dataclass(frozen=True)
class Signature:
    name: str
    a: tuple          # (a0, a-1, ..., a-p)
    b: tuple          # (b-1, ..., b-k)
    dtype: str        # "int32" | "float32"
    what: str
    cite: str

    @property
    def p(self) -> int:
        return len(self.a) - 1

    @property
    def k(self) -> int:
        return len(self.b)

    def text(self) -> str:
        f = (lambda v: "%d" % v) if self.dtype == "int32" else (lambda v: "%g" % v)
        return "(%s: %s)" % (", ".join(f(v) for v in self.a), ", ".join(f(v) for v in self.b))


TABLE1 = [
    Signature("prefix", (1,), (1,), "int32", "prefix sum", "P:97"),
    Signature("tuple2", (1,), (0, 1), "int32", "2-tuple prefix sum", "P:98"),
    Signature("tuple3", (1,), (0, 0, 1), "int32", "3-tuple prefix sum", "P:99"),
    Signature("order2", (1,), (2, -1), "int32", "2nd-order prefix sum", "P:100"),
    Signature("order3", (1,), (3, -3, 1), "int32", "3rd-order prefix sum", "P:101"),
    Signature("lp1", (0.2,), (0.8,), "float32", "1-stage low-pass filter", "P:102"),
    Signature("lp2", (0.04,), (1.6, -0.64), "float32", "2-stage low-pass filter", "P:103"),
    Signature("lp3", (0.008,), (2.4, -1.92, 0.512), "float32", "3-stage low-pass filter", "P:104"),
    Signature("hp1", (0.9, -0.9), (0.8,), "float32", "1-stage high-pass filter", "P:105"),
    Signature("hp2", (0.81, -1.62, 0.81), (1.6, -0.64), "float32", "2-stage high-pass filter", "P:106"),
    Signature("hp3", (0.729, -2.187, 2.187, -0.729), (2.4, -1.92, 0.512), "float32",
              "3-stage high-pass filter (untruncated, reading R4)", "P:107, P:109-111"),
]
BY_NAME = {s.name: s for s in TABLE1}

# Printed (truncated) 3-stage high-pass row of Table 1, kept only so a test can
# show why reading R4 is needed.
HP3_PRINTED = Signature("hp3_printed", (0.73, -2.19, 2.19, -0.73), (2.4, -1.9, 0.5), "float32",
                        "3-stage high-pass filter as printed (truncated)", "P:107")


def seed_for(cfg: int, rank: int = 0) -> int:
    return SEED_BASE + 1000 * cfg + rank


def host_input(n: int, dtype: str, seed: int) -> np.ndarray:
    """Seeded host input: int32 full range, or float32 U[-1, 1)."""
    rng = np.random.default_rng(seed)
    if dtype == "int32":
        return rng.integers(-(2 ** 31), 2 ** 31, size=n, dtype=np.int64).astype(np.int32)
    return (2.0 * rng.random(n, dtype=np.float32) - 1.0).astype(np.float32)


def device_input(n: int, dtype: str, seed: int, device="cuda"):
    """Seeded device input (torch generator on the device), same recipe."""
    import torch
    g = torch.Generator(device=device)
    g.manual_seed(seed)
    if dtype == "int32":   # uniform random bytes viewed as int32: full range
        return torch.randint(0, 256, (4 * n,), dtype=torch.uint8, device=device,
                             generator=g).view(torch.int32)
    x = torch.rand(n, dtype=torch.float32, device=device, generator=g)
    return x.mul_(2.0).sub_(1.0)


def structured_input(kind: str, n: int, dtype: str) -> np.ndarray:
    """Structured inputs used by parity tests (P4/P7/P10 pins)."""
    npdt = np.int32 if dtype == "int32" else np.float32
    if kind == "ones":
        return np.ones(n, dtype=npdt)
    if kind == "impulse":
        x = np.zeros(n, dtype=npdt)
        if n:
            x[0] = 1
        return x
    if kind == "alternating":          # the worked example's input pattern (-1)^i (i+3)
        i = np.arange(n, dtype=np.int64)
        v = np.where(i % 2 == 0, 1, -1) * (i + 3)
        return v.astype(npdt)
    if kind == "extremes":
        v = np.array([2 ** 31 - 1, -(2 ** 31), -1, 1], dtype=np.int64)
        return np.resize(v, n).astype(np.int32) if dtype == "int32" else \
            np.resize(np.array([1.0, -1.0, 0.999, -0.999], dtype=np.float32), n)
    raise ValueError(kind)
