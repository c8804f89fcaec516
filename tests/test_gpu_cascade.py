"""GPU parity of cascades (multi-signature inputs,
P:1851-1852; filters applied one after the other): one pass of
the combined signature (plr_plan_create_cascade) against the oracle applied
stage by stage (oracle.cascade), bit-exact for int32, 1e-4 relative for
float32 -- through both the small-n and the persistent kernels."""
import numpy as np
import pytest

import oracle
import workloads

pytestmark = pytest.mark.gpu

HP1 = ((0.9, -0.9), (0.8,))
LP1 = ((0.2,), (0.8,))
CASCADES = {
    "hp1x3": ([HP1] * 3, "float32"),                         # the 3-stage high-pass as three stages
    "lp1x3": ([LP1] * 3, "float32"),
    "lp2_lp2": ([((0.04,), (1.6, -0.64))] * 2, "float32"),    # k = 4
    "fir_lp1_hp1": ([((0.25, 0.5, 0.25), ()), LP1], "float32"),  # a pure map stage, then a filter
    "prefix_x3": ([((1,), (1,))] * 3, "int32"),              # = 3rd-order prefix sum
    "tuple2_order2": ([((3, -1), (0, 1)), ((1,), (2, -1))], "int32"),
}


def check(y, ref, dtype, what):
    if dtype == "int32":
        bad = np.flatnonzero(y != ref)
        assert bad.size == 0, "%s: %d mismatches, first at %d" % (what, bad.size, bad[0])
    else:
        e = float(np.max(np.abs(y.astype(np.float64) - ref) / np.maximum(1.0, np.abs(ref))))
        assert e <= 1e-4, "%s: rel err %.3g" % (what, e)


@pytest.mark.parametrize("name", sorted(CASCADES))
@pytest.mark.parametrize("small_max", ["0", str(1 << 22)])
def test_cascade_parity(cuda_plr, name, small_max, monkeypatch):
    import torch
    monkeypatch.setenv("PLR_SMALL_MAX", small_max)
    stages, dtype = CASCADES[name]
    sizes = [1, 7, 5000, 3 * 7936 + 5, (1 << 20) + 12345, (1 << 22) + 3]
    x_all = workloads.host_input(max(sizes), dtype, workloads.seed_for(12))
    plan = cuda_plr.Plan.cascade(stages, dtype, n_max=max(sizes))
    for n in sizes:
        x = x_all[:n].copy()
        y = plan(torch.from_numpy(x).cuda()).cpu().numpy()
        check(y, oracle.cascade(x, stages, dtype), dtype, "%s n=%d" % (name, n))
    # the worked example's (-1)^i (i+3) input wherever fp32 data can meet the
    # output-relative bar at the Nyquist frequency (reading R20: map_floor)
    if dtype == "int32" or plan.info["map_floor"] <= 1e-4:
        xa = workloads.structured_input("alternating", 7 * 3840 + 123, dtype)
        y = plan(torch.from_numpy(xa).cuda()).cpu().numpy()
        check(y, oracle.cascade(xa, stages, dtype), dtype, "%s alternating" % name)
    plan.close()


def test_cascade_prefix_equals_order3(cuda_plr):
    """Three cascaded prefix sums and the (1: 3, -3, 1) row give the same
    bits on the GPU (Z/2^32 ring)."""
    import torch
    n = (1 << 24) + 99
    x = workloads.device_input(n, "int32", 13)
    a = cuda_plr.Plan.cascade([((1,), (1,))] * 3, "int32", n_max=n)(x)
    o3 = workloads.BY_NAME["order3"]
    b = cuda_plr.Plan(o3.a, o3.b, "int32", n_max=n)(x)
    assert torch.equal(a, b)
