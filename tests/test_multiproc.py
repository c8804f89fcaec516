"""World-size-2 (and 3) gloo tests of the sharded path's host logic on CPU:
contiguous partition, 64-byte payload exchange over torch.distributed, the
segment prefix z_{r+1} = M^{n_r} z_r + payload_r (plr_combine_host, the same
arithmetic as the device combine), and the unique-id bootstrap broadcast.
Segment payloads are computed by the oracle (zero history), and every rank
checks its boundary history against the oracle over the whole sequence
(reading R12)."""
import os
import socket
import struct

import numpy as np
import pytest
import torch.multiprocessing as mp

import workloads


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, names, n_total, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch.distributed as dist

    import oracle
    import paper_conf_asplos_malekib18_b200 as plr
    import workloads as wl
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        # bootstrap: rank 0's id bytes reach everyone
        tok = plr.broadcast_bytes(bytes([7, rank]) * 64 if rank == 0 else None)
        assert tok == bytes([7, 0]) * 64
        for name in names:
            sig = wl.BY_NAME[name]
            x = wl.host_input(n_total, sig.dtype, 77)
            start, n_r = plr.shard_bounds(n_total, world, rank)
            seg = x[start:start + n_r]
            yz = oracle.recurrence(seg, sig.a, sig.b, sig.dtype)           # zero history
            npdt = np.int32 if sig.dtype == "int32" else np.float32
            xt = np.zeros(4, npdt)
            yt = np.zeros(4, npdt)
            if n_r:
                xt[4 - min(4, n_r):] = seg[-4:]
                yt[4 - min(4, n_r):] = yz[-4:].astype(npdt)
            payload = struct.pack("<Q", n_r) + xt.tobytes() + yt.tobytes() + bytes(24)
            allp = plr.gather_payloads(payload)
            plan = plr.Plan(sig.a, sig.b, sig.dtype, n_max=0)
            hist = np.frombuffer(plan.combine_host(allp, rank, world), dtype=npdt)
            yfull = oracle.recurrence(x, sig.a, sig.b, sig.dtype)
            ex_x = np.array([x[start - 4 + i] if start - 4 + i >= 0 else 0 for i in range(4)], npdt)
            ex_y = np.array([yfull[start - 4 + i] if start - 4 + i >= 0 else 0 for i in range(4)])
            assert np.array_equal(hist[:4], ex_x), (name, rank)
            if sig.dtype == "int32":
                assert np.array_equal(hist[4:], ex_y.astype(np.int32)), (name, rank)
            else:
                assert np.allclose(hist[4:], ex_y, rtol=1e-5, atol=1e-5), (name, rank, hist, ex_y)
            # continuing the rank's segment from the combined history reproduces
            # the global result (the seeded pass of the non-DECAY schedule)
            ys = oracle.recurrence(seg, sig.a, sig.b, sig.dtype,
                                   x_hist=hist[4 - sig.p:4] if sig.p else None,
                                   y_hist=hist[8 - sig.k:8].astype(np.float64) if sig.dtype == "float32"
                                   else hist[8 - sig.k:8])
            ref = yfull[start:start + n_r]
            if sig.dtype == "int32":
                assert np.array_equal(ys, ref), (name, rank)
            else:
                assert np.max(np.abs(ys - ref) / np.maximum(1, np.abs(ref))) < 1e-4, (name, rank)
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,n_total", [(2, 20011), (3, 9)])
def test_gloo_sharded_host_logic(world, n_total):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    names = [s.name for s in workloads.TABLE1]
    procs = [ctx.Process(target=_worker, args=(r, world, port, names, n_total, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=240) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    assert all(v == "ok" for v in res.values()), res


def test_shard_bounds_partition():
    import paper_conf_asplos_malekib18_b200 as plr
    for n in (0, 1, 7, 1 << 20, (1 << 20) + 5):
        for w in (1, 2, 3, 8):
            segs = [plr.shard_bounds(n, w, r) for r in range(w)]
            assert segs[0][0] == 0
            for (s0, n0), (s1, _) in zip(segs, segs[1:]):
                assert s0 + n0 == s1
            assert sum(nr for _, nr in segs) == n
