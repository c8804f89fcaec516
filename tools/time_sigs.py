"""Time signatures at n (no debug stats): ms, GB/s, fraction of an in-run memcpy.
Usage: python tools/time_sigs.py [n] [sig,sig,...] [scan|reverse|bidir]   (PLR_LIB selects a variant library)
reverse: the anticausal pass; bidir: forward + anticausal (two passes, 16 B per element counted)"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_asplos_malekib18_b200 as plr  # noqa: E402
import workloads  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 30
names = sys.argv[2].split(",") if len(sys.argv) > 2 and sys.argv[2] else [s.name for s in workloads.TABLE1]
mode = sys.argv[3] if len(sys.argv) > 3 else "scan"
passes = 2 if mode == "bidir" else 1
xi = workloads.device_input(n, "int32", 1)
xf = workloads.device_input(n, "float32", 2)
y = torch.empty_like(xi)


def timed(fn, reps=10):
    for _ in range(3):
        fn()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps


ms_cp = timed(lambda: y.copy_(xi))
print("%-7s %8.3f ms %7.1f GB/s" % ("memcpy", ms_cp, n * 8 / ms_cp / 1e6), flush=True)
for name in names:
    sig = workloads.BY_NAME[name]
    x = xi if sig.dtype == "int32" else xf
    yy = y if sig.dtype == "int32" else y.view(torch.float32)
    plan = plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
    if mode == "reverse":
        ms = timed(lambda: plan.reverse(x, yy))
    elif mode == "bidir":
        tmp = torch.empty_like(yy)
        ms = timed(lambda: plan.bidirectional(x, yy, tmp=tmp))
    else:
        ms = timed(lambda: plan(x, yy))
    print("%-7s %8.3f ms %7.1f GB/s  %.3f of memcpy  %s" % (name, ms, passes * n * 8 / ms / 1e6, passes * ms_cp / ms,
          {k: plan.info[k] for k in ("ctas_per_sm", "cls", "tile_elems")}), flush=True)
    plan.close()
