"""GPU parity beyond Table 1 ("wider signatures"): order
k = 4 (4-tuple and 4th-order prefix sums, a 4-stage low-pass), a
non-decaying float signature (class FLOAT, fp64 accumulation), and both
look-back unit sizes of the multi-tile kernels (units of one tile at small
n, PLR_UNIT1_WAVES; units of G tiles otherwise).  Same bar as
test_gpu_parity: bit-exact int32, 1e-4 relative float."""
import os

import numpy as np
import pytest

import oracle
import workloads

pytestmark = pytest.mark.gpu

TOL = 1e-4
WIDER = [
    workloads.Signature("tuple4", (1,), (0, 0, 0, 1), "int32", "4-tuple prefix sum", "P:138-140"),
    workloads.Signature("order4", (1,), (4, -6, 4, -1), "int32", "4th-order prefix sum", "P:140-143"),
    workloads.Signature("fir_order2", (3, -1, 2, 5), (2, -1), "int32", "FIR map + 2nd-order sum", "Eq. (1)"),
    workloads.Signature("lp4", (0.0016,), (3.2, -3.84, 2.048, -0.4096), "float32", "4-stage low-pass", "P:102-104"),
    workloads.Signature("fsum", (1.0,), (1.0,), "float32", "float prefix sum (FLOAT class)", "P:97"),
    workloads.Signature("fosc", (0.5, 0.25), (1.0, -0.5), "float32", "damped-oscillator filter", "Eq. (1)"),
]


def check(y, ref, sig, what):
    if sig.dtype == "int32":
        bad = np.flatnonzero(y != ref)
        assert bad.size == 0, "%s: %d mismatches, first at %d" % (what, bad.size, bad[0])
    else:
        e = float(np.max(np.abs(y.astype(np.float64) - ref) / np.maximum(1.0, np.abs(ref))))
        assert e <= TOL, "%s: rel err %.3g" % (what, e)


@pytest.mark.parametrize("sig", WIDER, ids=lambda s: s.name)
@pytest.mark.parametrize("waves", ["4", "0", "small"])
def test_wider_signatures(cuda_plr, sig, waves, monkeypatch):
    """waves "4" / "0": the persistent kernels (PLR_SMALL_MAX=0) with look-back
    units of one tile / of G tiles; "small": the small-n kernel at every size."""
    import torch
    if waves == "small":
        monkeypatch.setenv("PLR_SMALL_MAX", str(1 << 22))
    else:
        monkeypatch.setenv("PLR_SMALL_MAX", "0")
        monkeypatch.setenv("PLR_UNIT1_WAVES", waves)
    m = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=1 << 10).info["tile_elems"]
    sizes = [1, 5, m - 1, m + 1, 7 * m + 3, 33 * m + 5, (1 << 20) + 12345]
    x_all = workloads.host_input(max(sizes), sig.dtype, workloads.seed_for(7))
    plan = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=max(sizes))
    for n in sizes:
        x = x_all[:n].copy()
        y = plan(torch.from_numpy(x).cuda()).cpu().numpy()
        check(y, oracle.recurrence(x, sig.a, sig.b, sig.dtype), sig, "%s n=%d waves=%s" % (sig.name, n, waves))
    plan.close()


@pytest.mark.parametrize("name", ["tuple3", "order3", "prefix"])
def test_unit_sizes_agree(cuda_plr, name):
    """The same input through both unit sizes gives the identical int32 result."""
    import torch
    sig = workloads.BY_NAME[name]
    n = (1 << 22) + 777
    x = torch.from_numpy(workloads.host_input(n, sig.dtype, workloads.seed_for(8))).cuda()
    plan = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
    outs = []
    for waves in ("1000000", "0"):
        os.environ["PLR_UNIT1_WAVES"] = waves
        outs.append(plan(x).cpu().numpy())
    os.environ.pop("PLR_UNIT1_WAVES", None)
    plan.close()
    assert np.array_equal(outs[0], outs[1])
    assert np.array_equal(outs[0], oracle.recurrence(x.cpu().numpy(), sig.a, sig.b, sig.dtype))
