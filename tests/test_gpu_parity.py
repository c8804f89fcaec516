"""GPU parity: the CUDA path through the C ABI vs the CPU oracle, element by
element, on seeded inputs.  Bar: bit-exact for int32
(ring Z/2^32); for float32 max_i |y_gpu - y_ref| / max(1, |y_ref|) <= 1e-4
against the fp64 oracle (BASELINE.json north_star; the paper used 1e-3
against serial fp32)."""
import numpy as np
import pytest

import oracle
import workloads

pytestmark = pytest.mark.gpu

TOL = 1e-4
M = 3840                 # nominal tile (DECAY kernels); sizes below span many tiles either way


def rel_err(y, ref):
    y = np.asarray(y, dtype=np.float64)
    return float(np.max(np.abs(y - ref) / np.maximum(1.0, np.abs(ref)))) if len(ref) else 0.0


def check(y, ref, dtype, what=""):
    if dtype == "int32":
        bad = np.flatnonzero(y != ref)
        assert bad.size == 0, "%s: %d mismatches, first at %d: %d vs %d" % (
            what, bad.size, bad[0], y[bad[0]], ref[bad[0]])
    else:
        e = rel_err(y, ref)
        assert e <= TOL, "%s: rel err %.3g" % (what, e)


def run(plr, torch, sig, x, n_max=None):
    plan = plr.Plan(sig.a, sig.b, sig.dtype, n_max=n_max or max(1, len(x)))
    xd = torch.from_numpy(x).cuda()
    y = plan(xd).cpu().numpy()
    plan.close()
    return y


def sizes_for(m):
    """Edge sizes around the plan's tile m (the generic and DECAY kernels use
    different tiles), several tiles with ragged tails, and larger sizes."""
    return [1, 2, 3, 4, 5, 14, 15, 16, 31, 32, 33, 480, 481, m - 1, m, m + 1, 3 * m + 7, 33 * m + 5,
            (1 << 16) + 3, (1 << 20) + 12345]


# "auto": the size-dependent kernel choice (the small-n kernel up to
# PLR_SMALL_MAX elements); "big": PLR_SMALL_MAX=0, the persistent kernels at
# every size
PATHS = {"auto": None, "big": "0"}


def use_path(monkeypatch, path):
    if PATHS[path] is None:
        monkeypatch.delenv("PLR_SMALL_MAX", raising=False)
    else:
        monkeypatch.setenv("PLR_SMALL_MAX", PATHS[path])


@pytest.mark.parametrize("sig", workloads.TABLE1, ids=lambda s: s.name)
@pytest.mark.parametrize("path", sorted(PATHS))
def test_parity_sizes(cuda_plr, sig, path, monkeypatch):
    import torch
    use_path(monkeypatch, path)
    m = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=1 << 10).info["tile_elems"]
    SIZES = sizes_for(m)
    x_all = workloads.host_input(max(SIZES), sig.dtype, workloads.seed_for(1))
    plan = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=max(SIZES))
    for n in SIZES:
        x = x_all[:n].copy()
        y = plan(torch.from_numpy(x).cuda()).cpu().numpy()
        check(y, oracle.recurrence(x, sig.a, sig.b, sig.dtype), sig.dtype, "%s n=%d" % (sig.name, n))


@pytest.mark.parametrize("sig", workloads.TABLE1, ids=lambda s: s.name)
@pytest.mark.parametrize("kind", ["ones", "impulse", "alternating", "extremes"])
@pytest.mark.parametrize("path", sorted(PATHS))
def test_parity_structured(cuda_plr, sig, kind, path, monkeypatch):
    import torch
    use_path(monkeypatch, path)
    n = 7 * M + 123
    x = workloads.structured_input(kind, n, sig.dtype)
    y = run(cuda_plr, torch, sig, x)
    check(y, oracle.recurrence(x, sig.a, sig.b, sig.dtype), sig.dtype, "%s %s" % (sig.name, kind))


def test_worked_example_on_gpu(cuda_plr):
    import torch
    from conftest import read_golden
    g = read_golden("worked_example.txt")
    x = np.array(g["input"], dtype=np.int32)
    y = run(cuda_plr, torch, workloads.BY_NAME["order2"], x)
    assert y.tolist() == g["expected_output"]


def test_closed_forms_on_gpu(cuda_plr):
    """ones -> i+1, C(i+2,2), C(i+3,3) mod 2^32 across ~270 tiles."""
    import torch
    n = (1 << 20) + 77
    i = np.arange(n, dtype=np.uint64)
    x = np.ones(n, dtype=np.int32)
    for b, e in (((1,), i + 1), ((2, -1), (i + 1) * (i + 2) // 2), ((3, -3, 1), (i + 1) * (i + 2) * (i + 3) // 6)):
        sig = workloads.Signature("t", (1,), b, "int32", "", "")
        y = run(cuda_plr, torch, sig, x)
        assert np.array_equal(y.view(np.uint32), (e % (1 << 32)).astype(np.uint32))


@pytest.mark.parametrize("sig", workloads.TABLE1, ids=lambda s: s.name)
def test_repeated_launches_epochs(cuda_plr, sig, monkeypatch):
    """One plan, many launches with varying n: epoch-tagged status words and
    the ticket base must never mix launches -- also across the small-n and
    the persistent kernels, which share the plan's launch state."""
    import torch
    monkeypatch.setenv("PLR_SMALL_MAX", str(60 * M))
    plan = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=200 * M)
    rng = np.random.default_rng(5)
    for t in range(12):
        n = int(rng.integers(1, 200 * M))
        x = workloads.host_input(n, sig.dtype, 100 + t)
        y = plan(torch.from_numpy(x).cuda()).cpu().numpy()
        check(y, oracle.recurrence(x, sig.a, sig.b, sig.dtype), sig.dtype, "%s launch %d n=%d" % (sig.name, t, n))


@pytest.mark.parametrize("sig", workloads.TABLE1, ids=lambda s: s.name)
@pytest.mark.parametrize("n", [5000, 3 * M + 7, (1 << 20) + 12345, (1 << 22) + 4321])
def test_cuda_graph_replay(cuda_plr, sig, n):
    """plr_execute captured in a CUDA graph: the ticket base and the epoch
    live on the device (launch_state_advance), so every replay, and eager
    launches of the same plan between replays, see a fresh launch state."""
    import torch
    plan = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
    xd = torch.from_numpy(workloads.host_input(n, sig.dtype, 300)).cuda()
    yd = torch.empty_like(xd)
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        plan(xd, yd)                                     # warm-up outside the capture
    torch.cuda.current_stream().wait_stream(s)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        plan(xd, yd)
    for t in range(4):
        x = workloads.host_input(n, sig.dtype, 301 + t)
        xd.copy_(torch.from_numpy(x))
        for _ in range(t + 1):                           # repeated replays of the same launch
            g.replay()
        check(yd.cpu().numpy(), oracle.recurrence(x, sig.a, sig.b, sig.dtype), sig.dtype,
              "%s graph replay %d n=%d" % (sig.name, t, n))
        m = max(1, n // (t + 2))                         # an eager launch of another size in between
        ye = plan(xd[:m]).cpu().numpy()
        check(ye, oracle.recurrence(x[:m], sig.a, sig.b, sig.dtype), sig.dtype,
              "%s eager after replay %d m=%d" % (sig.name, t, m))
    del g
    plan.close()


@pytest.mark.parametrize("sig", workloads.TABLE1, ids=lambda s: s.name)
def test_continue_chunks(cuda_plr, sig):
    """plr_execute_continue over chunks (history = preceding inputs/outputs)
    equals one call (P:78 zero state only at the very start)."""
    import torch
    n = 50 * M + 999
    x = workloads.host_input(n, sig.dtype, 21)
    ref = oracle.recurrence(x, sig.a, sig.b, sig.dtype)
    plan = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
    xd = torch.from_numpy(x).cuda()
    yd = torch.empty_like(xd)
    cuts = [0, 4, 4096, 4100, 20 * M + 8, 20 * M + 12, n]     # chunk starts stay 16-byte aligned

    def hist(t, s, L):
        if s == 0 or L == 0:
            return None
        if s >= L:
            return t[s - L:s]
        return torch.cat([torch.zeros(L - s, dtype=t.dtype, device="cuda"), t[:s]])
    for s, e in zip(cuts[:-1], cuts[1:]):
        plan.continue_(xd[s:e], yd[s:e], x_hist=hist(xd, s, sig.p), y_hist=hist(yd, s, sig.k))
    check(yd.cpu().numpy(), ref, sig.dtype, sig.name)


@pytest.mark.parametrize("sig", workloads.TABLE1, ids=lambda s: s.name)
def test_reduce_payload_and_combine(cuda_plr, sig):
    """Reduce-only payload = zero-history end state; device combine = host
    combine; and the full loopback of the sharded schedule on one GPU
    (reduce or local pass -> gathered payloads -> combine -> seeded pass or
    DECAY fixup) reproduces the oracle over the concatenation (reading R12)."""
    import torch
    sizes = [7 * M + 5, 3, 12 * M, M - 1, 9 * M + 1000]
    n = sum(sizes)
    x = workloads.host_input(n, sig.dtype, 31)
    ref = oracle.recurrence(x, sig.a, sig.b, sig.dtype)
    plan = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
    decay = plan.info["cls"] == "DECAY"
    starts = np.cumsum([0] + sizes)
    # each "rank" owns its segment in its own (aligned) allocation, as on a real box
    xs = [torch.from_numpy(x[starts[r]:starts[r] + nr].copy()).cuda() for r, nr in enumerate(sizes)]
    ys = [torch.empty_like(t) for t in xs]
    pls = []
    for r, nr in enumerate(sizes):
        if decay:
            plan(xs[r], ys[r])
            pl = plan.payload_from_output(xs[r], ys[r])
        else:
            pl = plan.reduce(xs[r])
        # payload == oracle zero-history tails
        yz = oracle.recurrence(x[starts[r]:starts[r] + nr], sig.a, sig.b, sig.dtype)
        got = pl.cpu().numpy()
        assert int(got[:8].view(np.uint64)[0]) == nr
        npdt = np.int32 if sig.dtype == "int32" else np.float32
        kk = min(sig.k if not decay else 4, nr)       # plr_reduce fills the last k outputs only
        yt = got[24:40].view(npdt)[4 - kk:]
        check(yt.astype(np.float64) if sig.dtype == "float32" else yt, yz[len(yz) - kk:], sig.dtype, "payload %d" % r)
        pls.append(pl)
    payloads = torch.cat(pls)
    host_pl = payloads.cpu().numpy().tobytes()
    for r, nr in enumerate(sizes):
        hist = plan.combine(payloads, r, len(sizes))
        assert hist.cpu().numpy().tobytes() == plan.combine_host(host_pl, r, len(sizes))
        if decay:
            plan.fixup(ys[r], hist)
        else:
            xh = hist[4 - sig.p:4] if sig.p else None
            plan.continue_(xs[r], ys[r], x_hist=xh, y_hist=hist[8 - sig.k:8])
    check(torch.cat(ys).cpu().numpy(), ref, sig.dtype, sig.name)


@pytest.mark.parametrize("sig", [workloads.BY_NAME[n] for n in ("prefix", "order3", "hp3")], ids=lambda s: s.name)
def test_execute_sharded_world1(cuda_plr, sig):
    import torch
    n = 40 * M + 17
    x = workloads.host_input(n, sig.dtype, 41)
    plan = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)

    class C:
        rank, world, handle = 0, 1, None
    y = plan.sharded(torch.from_numpy(x).cuda(), comm=C()).cpu().numpy()
    check(y, oracle.recurrence(x, sig.a, sig.b, sig.dtype), sig.dtype, sig.name)


@pytest.mark.parametrize("sig", [workloads.BY_NAME[n] for n in ("tuple3", "lp2")], ids=lambda s: s.name)
def test_execute_host_pipeline(cuda_plr, sig):
    """plr_execute_host: chunked H2D/compute/D2H, chunks continued."""
    import torch
    n = (1 << 26) + 3 * M + 11              # > 2 chunks of 2^25
    x = workloads.host_input(n, sig.dtype, 51)
    plan = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
    xh = torch.from_numpy(x).pin_memory()
    y = plan.execute_host(xh).numpy()
    check(y, oracle.recurrence(x, sig.a, sig.b, sig.dtype), sig.dtype, sig.name)


def test_errors(cuda_plr):
    import torch
    plan = cuda_plr.Plan((1, 1), (0.5,), "float32", n_max=1000)
    x = torch.zeros(1000, dtype=torch.float32, device="cuda")
    with pytest.raises(cuda_plr.PLRError) as e:
        plan(x, x)                               # p > 0 in place
    assert e.value.status == 5
    with pytest.raises(cuda_plr.PLRError) as e:
        plan(x[1:], torch.empty(999, device="cuda"))
    assert e.value.status == 6                   # misaligned
    big = torch.zeros(1001, dtype=torch.float32, device="cuda")
    with pytest.raises(cuda_plr.PLRError) as e:
        plan(big)
    assert e.value.status == 4
    plan2 = cuda_plr.Plan((1,), (1,), "int32", n_max=1000)
    xi = torch.arange(1000, dtype=torch.int32, device="cuda")
    ref = oracle.recurrence(xi.cpu().numpy(), (1,), (1,), "int32")
    assert np.array_equal(plan2(xi, xi).cpu().numpy(), ref)   # p == 0 in place is allowed
    assert plan2(torch.zeros(0, dtype=torch.int32, device="cuda")).numel() == 0


# ------------------------------------------------------------ full size ----
FULL = 1 << 30


def _stream_check(plr_mod, torch, sig, n, seed, seg=1 << 25):
    """Full-size run in the bench's launch configuration; the oracle streams
    over segments with its history carried (O(segment) host memory) and every
    output element is compared."""
    plan = plr_mod.Plan(sig.a, sig.b, sig.dtype, n_max=n)
    xd = workloads.device_input(n, sig.dtype, seed)
    yd = plan(xd)
    torch.cuda.synchronize()
    xh = yh = None
    worst = 0.0
    for s in range(0, n, seg):
        e = min(n, s + seg)
        x = xd[s:e].cpu().numpy()
        y = yd[s:e].cpu().numpy()
        ref = oracle.recurrence(x, sig.a, sig.b, sig.dtype, x_hist=xh, y_hist=yh)
        if sig.dtype == "int32":
            assert np.array_equal(y, ref), "%s mismatch in [%d, %d)" % (sig.name, s, e)
        else:
            worst = max(worst, rel_err(y, ref))
        xh = x[len(x) - sig.p:] if sig.p else None
        yh = ref[len(ref) - sig.k:]
    assert worst <= TOL, (sig.name, worst)
    del xd, yd
    plan.close()
    torch.cuda.empty_cache()


@pytest.mark.parametrize("name", [s.name for s in workloads.TABLE1])
def test_full_size_parity(cuda_plr, name):
    """Every Table-1 row at exactly n = 2^30, every
    output element compared."""
    import torch
    sig = workloads.BY_NAME[name]
    _stream_check(cuda_plr, torch, sig, FULL, workloads.seed_for(2))


def test_full_size_ragged(cuda_plr):
    import torch
    _stream_check(cuda_plr, torch, workloads.BY_NAME["hp3"], FULL - 12345, workloads.seed_for(6))


# ------------------------------------------------------------ ablation -----
ABLATIONS = {"generic": ("PLR_FORCE_GENERIC", "1"), "no_constsig": ("PLR_NO_CONSTSIG", "1")}


@pytest.mark.parametrize("sig", workloads.TABLE1, ids=lambda s: s.name)
@pytest.mark.parametrize("mode", sorted(ABLATIONS))
def test_ablation_modes_parity(cuda_plr, sig, mode, monkeypatch):
    """The Fig. 10 analogue (tools/ablation.py) times kernels
    with the class specialisations off (PLR_FORCE_GENERIC=1: DECAY rows on
    the generic multi-tile look-back, no compile-time tables) or the
    compile-time signature tables off (PLR_NO_CONSTSIG=1).  Those kernels
    must meet the same parity bar as the shipped ones."""
    import torch
    var, val = ABLATIONS[mode]
    monkeypatch.setenv(var, val)
    monkeypatch.setenv("PLR_SMALL_MAX", "0")          # the persistent kernels the ablation times
    probe = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=1 << 10)
    m = probe.info["tile_elems"]
    if mode == "generic":
        assert probe.info["kernel_kind"] != 0 and probe.info["const_sig"] == 0
    else:
        assert probe.info["const_sig"] == 0
    probe.close()
    sizes = [1, 5, m - 1, m + 1, 7 * m + 3, 33 * m + 5, (1 << 20) + 12345]
    x_all = workloads.host_input(max(sizes), sig.dtype, workloads.seed_for(9))
    plan = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=max(sizes))
    for n in sizes:
        x = x_all[:n].copy()
        y = plan(torch.from_numpy(x).cuda()).cpu().numpy()
        check(y, oracle.recurrence(x, sig.a, sig.b, sig.dtype), sig.dtype, "%s %s n=%d" % (sig.name, mode, n))
    xa = workloads.structured_input("alternating", 7 * m + 123, sig.dtype)
    y = plan(torch.from_numpy(xa).cuda()).cpu().numpy()
    check(y, oracle.recurrence(xa, sig.a, sig.b, sig.dtype), sig.dtype, "%s %s alternating" % (sig.name, mode))
    plan.close()


# ------------------------------------------------------------ determinism --
@pytest.mark.parametrize("sig", [s for s in workloads.TABLE1 if s.dtype == "float32"], ids=lambda s: s.name)
def test_decay_bitwise_repeatable(cuda_plr, sig):
    """DECAY float results are bitwise repeatable, because
    T(m) = 0 makes the look-back a single hop (the carry entering a tile
    never depends on which predecessor happened to be inclusive).  Repeated
    launches, with and without a concurrent memory-bound kernel on another
    stream perturbing the tile-to-CTA schedule, give identical bits."""
    import torch
    n = (1 << 24) + 777
    plan = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
    assert plan.info["cls"] == "DECAY"
    xd = workloads.device_input(n, sig.dtype, workloads.seed_for(10))
    first = plan(xd).cpu().numpy().view(np.uint32)
    noise_a = torch.empty(1 << 27, dtype=torch.float32, device="cuda")
    noise_b = torch.empty_like(noise_a)
    side = torch.cuda.Stream()
    for t in range(6):
        if t % 2:
            with torch.cuda.stream(side):
                for _ in range(3):
                    noise_b.copy_(noise_a)
        y = plan(xd).cpu().numpy().view(np.uint32)
        torch.cuda.synchronize()
        assert np.array_equal(y, first), "%s: run %d differs bitwise in %d elements" % (
            sig.name, t, int(np.count_nonzero(y != first)))
    plan.close()


# ------------------------------------------------------------ small n ------
@pytest.mark.parametrize("sig", workloads.TABLE1, ids=lambda s: s.name)
def test_small_n_sweep_points(cuda_plr, sig, monkeypatch):
    """every size of the sweep 2^10 .. 2^22
    plus ragged neighbours, through the size-dependent kernel choice, and
    the small-n kernel forced beyond its default range (2^22 + 777)."""
    import torch
    sizes = [1 << e for e in range(10, 23)] + [(1 << e) + 5 for e in (10, 16, 21)] + [(1 << 22) + 777]
    x_all = workloads.host_input(max(sizes), sig.dtype, workloads.seed_for(11))
    monkeypatch.setenv("PLR_SMALL_MAX", str(max(sizes)))
    plan = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=max(sizes))
    for n in sizes:
        x = x_all[:n].copy()
        y = plan(torch.from_numpy(x).cuda()).cpu().numpy()
        check(y, oracle.recurrence(x, sig.a, sig.b, sig.dtype), sig.dtype, "%s n=%d" % (sig.name, n))
    plan.close()


# ------------------------------------------------------------ reduce-only --
@pytest.mark.parametrize("name", ["prefix", "tuple3", "order2", "order3", "fir_order2", "fsum"])
@pytest.mark.parametrize("n", [(1 << 22) + 1, 7936 * 1000, (1 << 24) + 12345, 148 * 2 * 7936 * 3 - 4])
def test_reduce_kernel_end_state(cuda_plr, name, n):
    """plr_reduce beyond the small-n range runs the contiguous-range
    streaming fold (plr_kernels_reduce.cuh): its payload's last k outputs
    equal the oracle's y_{n-k} .. y_{n-1} of the zero-history segment (int32
    bit-exact; float within the bar), incl. ragged ends and one tile per CTA
    short of a full wave."""
    import torch
    sigs = {s.name: s for s in workloads.TABLE1}
    sigs["fir_order2"] = workloads.Signature("fir_order2", (3, -1, 2, 5), (2, -1), "int32", "", "")
    sigs["fsum"] = workloads.Signature("fsum", (1.0,), (1.0,), "float32", "", "")
    sig = sigs[name]
    x = workloads.host_input(n, sig.dtype, workloads.seed_for(14))
    plan = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
    pl = plan.reduce(torch.from_numpy(x).cuda()).cpu().numpy()
    ref = oracle.recurrence(x, sig.a, sig.b, sig.dtype)
    assert int(pl[:8].view(np.uint64)[0]) == n
    npdt = np.int32 if sig.dtype == "int32" else np.float32
    got = pl[24:40].view(npdt)[4 - sig.k:]
    xt = pl[8:24].view(npdt)
    assert np.array_equal(xt, x[n - 4:])
    check(got.astype(np.float64) if sig.dtype == "float32" else got, ref[n - sig.k:], sig.dtype, "%s n=%d" % (name, n))
    plan.close()


# ------------------------------------------------- small n: cluster launches --
CLUSTER_SIGS = {s.name: s for s in workloads.TABLE1 if s.name in ("prefix", "tuple2", "tuple3", "order2", "order3")}
CLUSTER_SIGS.update({s.name: s for s in (
    workloads.Signature("order4", (1,), (4, -6, 4, -1), "int32", "4th-order prefix sum", "P:140-143"),
    workloads.Signature("fir_order2", (3, -1, 2, 5), (2, -1), "int32", "FIR map + 2nd-order sum", "Eq. (1)"),
    workloads.Signature("fsum", (1.0,), (1.0,), "float32", "float prefix sum (FLOAT class)", "P:97"))})


@pytest.mark.parametrize("name", sorted(CLUSTER_SIGS))
@pytest.mark.parametrize("cluster", ["1", "0"])
def test_small_n_cluster_lookback(cuda_plr, name, cluster, monkeypatch):
    """Non-decaying small-n launches run in clusters of 8 tiles whose
    aggregates meet over DSMEM; the look-back runs over cluster records
    (plr_kernels_small.cuh).  Tile counts around cluster boundaries (1, 2,
    7, 8, 9, 16, 17, 64, 65, 273 and the most resident tiles) with ragged
    tails, cluster launches on and off, against the oracle; continuation
    with history enters the first cluster's carry."""
    import torch
    sig = CLUSTER_SIGS[name]
    monkeypatch.setenv("PLR_SMALL_CLUSTER", cluster)
    monkeypatch.setenv("PLR_SMALL_MAX", str(1 << 21))
    ms = 3840
    probe = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=1 << 21)
    info = probe.info
    probe.close()
    c = info["small_cluster_ctas"]
    top = info["small_clusters"] * c                     # most tiles of a cluster launch
    assert top >= 64, "cluster launches unavailable: %s" % info
    # tile counts around cluster boundaries, up to the largest cluster launch
    # and one tile beyond it (the per-tile look-back again)
    tiles = sorted({t for t in (1, 2, c - 1, c, c + 1, 2 * c, 2 * c + 1, 64, 65, 273, top - 1, top, top + 1)
                    if 1 <= t <= top + 1})
    sizes = sorted({t * ms - d for t in tiles for d in (0, 1)} | {2 * ms + 17, 9 * ms + 1})
    x_all = workloads.host_input(max(sizes) + 64, sig.dtype, workloads.seed_for(13))
    plan = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=max(sizes) + 64)
    for n in sizes:
        x = x_all[:n].copy()
        y = plan(torch.from_numpy(x).cuda()).cpu().numpy()
        check(y, oracle.recurrence(x, sig.a, sig.b, sig.dtype), sig.dtype, "%s n=%d cluster=%s" % (name, n, cluster))
    # continuation: the second chunk starts from the first chunk's history
    n1, n2 = 17 * ms + 5, 64 * ms + 3
    x = x_all[:n1 + n2].copy()
    ref = oracle.recurrence(x, sig.a, sig.b, sig.dtype)
    y1 = plan(torch.from_numpy(x[:n1].copy()).cuda()).cpu().numpy()
    xh = torch.from_numpy(x[max(0, n1 - plan.p):n1].copy()).cuda() if plan.p > 0 else None
    yh = torch.from_numpy(y1[n1 - plan.k:].copy()).cuda()
    y2 = plan.continue_(torch.from_numpy(x[n1:].copy()).cuda(), x_hist=xh, y_hist=yh).cpu().numpy()
    check(np.concatenate([y1, y2]), ref, sig.dtype, "%s continuation cluster=%s" % (name, cluster))
    plan.close()


@pytest.mark.parametrize("lag", ["0", "1", "5", "9"])
def test_rr_runtime_lag(cuda_plr, lag, monkeypatch):
    """The re-read kernel's phase-B lag at run time (PLR_RR_LAG, read at plan
    creation, honoured by PLR_RR_RUNTIME_LAG=1 builds; 0 = NS-1): the
    look-back units of one tile (medium n) and of G tiles (large n), ragged,
    against the oracle.  A lag below max(1, G-1) falls back to NS-1 (lag 0
    once ran phase B of the stop position and hung)."""
    import torch
    monkeypatch.setenv("PLR_RR_LAG", lag)
    for name in ("tuple2", "order3"):
        sig = workloads.BY_NAME[name]
        sizes = [(1 << 21) + 5, (1 << 23) + 77, (1 << 24) + 3]
        x_all = workloads.host_input(max(sizes), sig.dtype, workloads.seed_for(19))
        plan = cuda_plr.Plan(sig.a, sig.b, sig.dtype, n_max=max(sizes))
        assert plan.info["small_max"] < sizes[0]
        for n in sizes:
            x = x_all[:n].copy()
            y = plan(torch.from_numpy(x).cuda()).cpu().numpy()
            check(y, oracle.recurrence(x, sig.a, sig.b, sig.dtype), sig.dtype, "%s n=%d lag=%s" % (name, n, lag))
        plan.close()
