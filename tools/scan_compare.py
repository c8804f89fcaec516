"""PLR vs the paper's Scan comparator (Blelloch matrix-vector scan through
CUB, Figs. 1-9 "Scan" curves) and the device copy, per Table-1
signature at n (default 2^26 and 2^30): ms, GB/s (8 B/element), fraction of
the copy.  Usage: python tools/scan_compare.py [n,n,...] [sig,...]"""
import json
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_asplos_malekib18_b200 as plr  # noqa: E402
import workloads  # noqa: E402

sizes = [int(v) for v in sys.argv[1].split(",")] if len(sys.argv) > 1 else [1 << 26, 1 << 30]
names = sys.argv[2].split(",") if len(sys.argv) > 2 else [s.name for s in workloads.TABLE1]


def timed(fn, reps=5):
    for _ in range(2):
        fn()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


for n in sizes:
    xi = workloads.device_input(n, "int32", 1)
    xf = workloads.device_input(n, "float32", 2)
    y = torch.empty_like(xi)
    ms_cp = timed(lambda: y.copy_(xi))
    for name in names:
        sig = workloads.BY_NAME[name]
        x = xi if sig.dtype == "int32" else xf
        yy = y if sig.dtype == "int32" else y.view(torch.float32)
        plan = plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
        ms_plr = timed(lambda: plan(x, yy))
        ms_scan = timed(lambda: plan.scan_comparator(x, yy))
        print(json.dumps({"sig": name, "n": n, "memcpy_ms": round(ms_cp, 4), "plr_ms": round(ms_plr, 4),
                          "scan_ms": round(ms_scan, 4), "plr_GBs": round(8 * n / ms_plr / 1e6, 1),
                          "scan_GBs": round(8 * n / ms_scan / 1e6, 1), "plr_frac_memcpy": round(ms_cp / ms_plr, 3),
                          "scan_frac_memcpy": round(ms_cp / ms_scan, 3),
                          "plr_over_scan": round(ms_scan / ms_plr, 2)}), flush=True)
        plan.close()
    del xi, xf, y
    torch.cuda.empty_cache()
