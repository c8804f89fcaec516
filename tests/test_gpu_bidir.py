"""GPU parity of the anticausal pass and of forward-backward filtering
(the causal/anticausal pairs of P:809-811):
plr_execute_reverse against oracle.anticausal and plr_execute_bidirectional
against oracle.bidirectional, element by element, through the small-n
kernel and (DECAY plans) the persistent DECAY kernel, ragged sizes included.
Bit-exact int32; float32 within 1e-4 relative."""
import numpy as np
import pytest

import oracle
import workloads

pytestmark = pytest.mark.gpu


def check(y, ref, dtype, what):
    if dtype == "int32":
        bad = np.flatnonzero(y != ref)
        assert bad.size == 0, "%s: %d mismatches, first at %d" % (what, bad.size, bad[0])
    else:
        e = float(np.max(np.abs(y.astype(np.float64) - ref) / np.maximum(1.0, np.abs(ref))))
        assert e <= 1e-4, "%s: rel err %.3g" % (what, e)


@pytest.mark.parametrize("sig", workloads.TABLE1, ids=lambda s: s.name)
@pytest.mark.parametrize("small_max", ["0", str(1 << 22)])
def test_reverse_parity(cuda_plr, sig, small_max, monkeypatch):
    import torch
    monkeypatch.setenv("PLR_SMALL_MAX", small_max)
    sizes = [1, 5, 3839, 3841, 5888 * 7 + 3, 7936 * 5, (1 << 20) + 12345, (1 << 22) + 7]
    x_all = workloads.host_input(max(sizes), sig.dtype, workloads.seed_for(15))
    plan = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=max(sizes))
    for n in sizes:
        x = x_all[:n].copy()
        y = plan.reverse(torch.from_numpy(x).cuda()).cpu().numpy()
        check(y, oracle.anticausal(x, sig.a, sig.b, sig.dtype), sig.dtype, "%s reverse n=%d" % (sig.name, n))
    plan.close()


@pytest.mark.parametrize("sig", workloads.TABLE1, ids=lambda s: s.name)
def test_bidirectional_parity(cuda_plr, sig):
    import torch
    n = (1 << 21) + 4321
    x = workloads.host_input(n, sig.dtype, workloads.seed_for(16))
    plan = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
    xd = torch.from_numpy(x).cuda()
    ref = oracle.bidirectional(x, sig.a, sig.b, sig.dtype)
    check(plan.bidirectional(xd).cpu().numpy(), ref, sig.dtype, "%s bidirectional" % sig.name)
    if sig.p == 0:                                   # backward pass in place
        yd = torch.empty_like(xd)
        plan.bidirectional(xd, out=yd)
        check(yd.cpu().numpy(), ref, sig.dtype, "%s bidirectional in place" % sig.name)
    # (-1)^i (i+3) where fp32 data can meet the bar (reading R20): the pair
    # attenuates a Nyquist input twice, so the floor is map_floor / |H(-1)|
    info = plan.info
    if sig.dtype == "int32" or info["map_floor"] / min(1.0, info["nyquist_gain"]) <= 1e-4:
        xa = workloads.structured_input("alternating", 7 * 3840 + 123, sig.dtype)
        pa = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=len(xa))
        check(pa.bidirectional(torch.from_numpy(xa).cuda()).cpu().numpy(),
              oracle.bidirectional(xa, sig.a, sig.b, sig.dtype), sig.dtype, "%s bidirectional alternating" % sig.name)
        pa.close()
    plan.close()


def test_reverse_full_size_decay(cuda_plr):
    """The anticausal DECAY kernel at n = 2^30 - 5 (ragged first tile),
    streamed from the end against the oracle's segments."""
    import torch
    sig = workloads.BY_NAME["hp2"]
    n = (1 << 30) - 5
    plan = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
    xd = workloads.device_input(n, sig.dtype, workloads.seed_for(17))
    yd = plan.reverse(xd)
    torch.cuda.synchronize()
    # segments from the end: the anticausal state of the later segment is the
    # history of the earlier one; the oracle runs each segment over itself plus
    # a 4096-element overlap (the free response is below fp32 resolution
    # beyond ~500 elements for the DECAY rows)
    seg, ov = 1 << 25, 4096
    worst = 0.0
    for e in range(n, 0, -seg):
        s = max(0, e - seg)
        hi = min(n, e + ov)
        x = xd[s:hi].cpu().numpy()
        ref = oracle.anticausal(x, sig.a, sig.b, sig.dtype)[:e - s]
        y = yd[s:e].cpu().numpy()
        worst = max(worst, float(np.max(np.abs(y - ref) / np.maximum(1, np.abs(ref)))))
    assert worst <= 1e-4, worst
    plan.close()


@pytest.mark.parametrize("name", ["prefix", "tuple3", "order3", "lp3", "hp3"])
def test_reverse_large_persistent(cuda_plr, name):
    """The anticausal pass on the persistent kernels' REV instantiations (TMEM
    k = 1, re-read k >= 2, TMEM-parked DECAY incl. fp64 accumulation) at
    n = 2^27 - 3 (ragged first tile, thousands of tiles per launch), every
    element against the oracle."""
    import torch
    sig = workloads.BY_NAME[name]
    n = (1 << 27) - 3
    x = workloads.host_input(n, sig.dtype, workloads.seed_for(18))
    plan = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
    assert n > plan.info["small_max"]
    y = plan.reverse(torch.from_numpy(x).cuda()).cpu().numpy()
    check(y, oracle.anticausal(x, sig.a, sig.b, sig.dtype), sig.dtype, "%s reverse n=%d" % (name, n))
    plan.close()
