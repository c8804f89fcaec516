"""Size sweep 2^10..2^30 (paper's protocol P:909-921: powers of two plus a
non-power-of-two) for every Table-1 signature, with the in-run memcpy
yardstick at each size.  Inputs <= 2^24 are L2-resident; L2 is flushed
between timed repetitions (a 256 MiB write) so the numbers are HBM numbers.
Prints one JSON line per (signature, n)."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_asplos_malekib18_b200 as plr  # noqa: E402
import workloads  # noqa: E402

names = sys.argv[1].split(",") if len(sys.argv) > 1 else [s.name for s in workloads.TABLE1]
lo = int(sys.argv[2]) if len(sys.argv) > 2 else 10
hi = int(sys.argv[3]) if len(sys.argv) > 3 else 30
sizes = [1 << e for e in range(lo, hi + 1, 2)] + [(1 << hi) - 12345]
nmax = max(sizes)
xi = workloads.device_input(nmax, "int32", 3)
xf = workloads.device_input(nmax, "float32", 4)
y = torch.empty_like(xi)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")


def timed(fn, n, reps):
    ts = []
    for r in range(reps + 2):
        flush.fill_(r & 0xff)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        if r >= 2:
            ts.append(e0.elapsed_time(e1))
    return sum(ts) / len(ts)


for n in sizes:
    reps = 10 if n <= (1 << 24) else 5
    ms_cp = timed(lambda: y[:n].copy_(xi[:n]), n, reps)
    for name in names:
        sig = workloads.BY_NAME[name]
        x = (xi if sig.dtype == "int32" else xf)[:n]
        yy = (y if sig.dtype == "int32" else y.view(torch.float32))[:n]
        plan = plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
        ms = timed(lambda: plan(x, yy), n, reps)
        print(json.dumps({"sig": name, "n": n, "ms": round(ms, 5), "GB/s": round(8 * n / ms / 1e6, 1),
                          "Gelem/s": round(n / ms / 1e6, 2), "memcpy_GB/s": round(8 * n / ms_cp / 1e6, 1),
                          "frac_memcpy": round(ms_cp / ms, 3), "tile": plan.info["tile_elems"]}), flush=True)
        plan.close()
