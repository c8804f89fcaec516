"""Small-n device time: is the gap to a copy at
2^10..2^22 on the device or in the host launch path?

Run under `ncu --metrics gpu__time_duration.sum --csv` (ncu flushes caches
between kernels, so every launch is a cold HBM launch) and summarise with
`python tools/small_n.py --parse launches.csv` (run with SMALLN_HOST=0
under ncu).  Each (n, signature) runs
REPS launches; the yardstick is an elementwise int32 -> fp32 copy kernel
(reads 4 B, writes 4 B per element, like the scan).  Without --parse the
script also prints the host-side per-call time (events around a batch of
back-to-back calls, which is host-bound when the kernel is shorter than
the launch path)."""
import csv
import json
import os
import sys

SIGS = ["prefix", "tuple2", "order3", "lp1", "hp3"]
SIZES = [1 << e for e in range(10, 23, 2)] + [(1 << 20) + 12345]
REPS = 3


def parse(path):
    with open(path) as f:
        lines = [l for l in f if l.startswith('"')]
    scan, copy = [], []
    for r in csv.DictReader(lines):
        if r["Metric Name"] != "gpu__time_duration.sum":
            continue
        v = float(r["Metric Value"].replace(",", ""))
        u = r["Metric Unit"]
        us = v / 1000.0 if u in ("ns", "nsecond") else v * 1000.0 if u in ("ms", "msecond") else v
        (scan if "plr_scan" in r["Kernel Name"] else copy).append(us)
    print("# small-n device time (ncu gpu__time_duration, cold cache, serialised)\n")
    print("| n | copy us | " + " | ".join("%s us (frac)" % s for s in SIGS) + " |")
    print("|---|---|" + "---|" * len(SIGS))
    ci = si = 0
    for n in SIZES:
        c = copy[ci:ci + REPS]
        ci += REPS
        cm = sorted(c)[len(c) // 2]
        cells = []
        for _ in SIGS:
            s = scan[si:si + REPS]
            si += REPS
            sm = sorted(s)[len(s) // 2]
            cells.append("%.2f (%.2f)" % (sm, cm / sm))
        print("| %d | %.2f | %s |" % (n, cm, " | ".join(cells)))
    print("\n(median of %d launches each; frac = copy time / scan time)" % REPS)


def run():
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch
    import paper_conf_asplos_malekib18_b200 as plr
    import workloads

    nmax = max(SIZES)
    xi = workloads.device_input(nmax, "int32", 3)
    xf = workloads.device_input(nmax, "float32", 4)
    yi = torch.empty_like(xi)
    yf = torch.empty_like(xf)
    plans = {}
    for n in SIZES:
        for _ in range(REPS):
            yf[:n].copy_(xi[:n])
        for name in SIGS:
            sig = workloads.BY_NAME[name]
            x = (xi if sig.dtype == "int32" else xf)[:n]
            y = (yi if sig.dtype == "int32" else yf)[:n]
            if (name, n) not in plans:
                plans[(name, n)] = plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
            for _ in range(REPS):
                plans[(name, n)](x, y)
    torch.cuda.synchronize()
    if os.environ.get("SMALLN_HOST", "1") == "1":
        for n in SIZES:
            for name in SIGS:
                sig = workloads.BY_NAME[name]
                x = (xi if sig.dtype == "int32" else xf)[:n]
                y = (yi if sig.dtype == "int32" else yf)[:n]
                plan = plans[(name, n)]
                for _ in range(20):
                    plan(x, y)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                torch.cuda.synchronize()
                e0.record()
                for _ in range(200):
                    plan(x, y)
                e1.record()
                torch.cuda.synchronize()
                b2b = e0.elapsed_time(e1) * 5
                # the same launch captured 20x in a CUDA graph (launch state lives on the device)
                g = torch.cuda.CUDAGraph()
                with torch.cuda.graph(g):
                    for _ in range(20):
                        plan(x, y)
                g.replay()
                torch.cuda.synchronize()
                e0.record()
                for _ in range(10):
                    g.replay()
                e1.record()
                torch.cuda.synchronize()
                print(json.dumps({"sig": name, "n": n, "back_to_back_us_per_call": round(b2b, 2),
                                  "graph_us_per_call": round(e0.elapsed_time(e1) * 1000 / 200, 2)}), flush=True)
                del g
    for p in plans.values():
        p.close()


if __name__ == "__main__":
    if len(sys.argv) > 2 and sys.argv[1] == "--parse":
        parse(sys.argv[2])
    else:
        run()
