"""Look-back statistics + timing per signature at a given n (PLR_STATS=1)."""
import os
import sys
os.environ["PLR_STATS"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_asplos_malekib18_b200 as plr  # noqa: E402
import workloads  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 30
names = sys.argv[2].split(",") if len(sys.argv) > 2 else ["prefix", "tuple2", "tuple3", "order3"]
xi = workloads.device_input(n, "int32", 1)
xf = workloads.device_input(n, "float32", 2)
y = torch.empty_like(xi)
for name in names:
    sig = workloads.BY_NAME[name]
    x = xi if sig.dtype == "int32" else xf
    yy = y if sig.dtype == "int32" else y.view(torch.float32)
    plan = plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
    for _ in range(3):
        plan(x, yy)
    torch.cuda.synchronize()
    plan.debug_stats(reset=True)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    reps = 5
    for _ in range(reps):
        plan(x, yy)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / reps
    st = plan.debug_stats()
    lb = max(1, st["lookbacks"])
    print("%-7s %8.3f ms %7.1f GB/s  lb/launch %d  polls/lb %.2f  waits/lb %.2f  depth/lb %.1f  "
          "cyc: agg %.0f lb %.0f sleep %.0f load %.0f fold %.0f  info %s" % (
              name, ms, n * 8 / ms / 1e6, st["lookbacks"] // reps, st["windows"] / lb, st["waits"] / lb,
              st["depth_sum"] / lb, st["cyc_agg"] / lb, st["cyc_lookback"] / lb, st["cyc_sleep"] / lb,
              st["cyc_load"] / lb, st["cyc_fold"] / lb,
              {k: plan.info[k] for k in ("ctas_per_sm", "cls")}), flush=True)
    plan.close()
