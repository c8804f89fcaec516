"""Critical path of the LAST tile of one small-n launch (plr_kernels_small.cuh):
globaltimer stamps (PLR_TRACE variant build, PLR_STATS=1), ns after that
CTA's entry, median of 5 launches, L2 flushed before each.
Usage: PLR_LIB=.../libplr_b200_trace.so python tools/trace_small.py"""
import json
import os
import sys
os.environ["PLR_STATS"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_asplos_malekib18_b200 as plr  # noqa: E402
import workloads  # noqa: E402

NAMES = ["entry", "ticket", "loaded", "phaseA_sync", "lookback_done", "phaseB_done", "store_read"]
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for name in ["prefix", "tuple2", "order3", "lp1", "hp3"]:
    for n in [3840 * 4, 3840 * 68, 3840 * 273, 3840 * 1092]:
        sig = workloads.BY_NAME[name]
        x = workloads.device_input(n, sig.dtype, 1)
        y = torch.empty_like(x)
        plan = plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
        rows = []
        lb = []
        for r in range(7):
            flush.fill_(r)
            torch.cuda.synchronize()
            plan(x, y)
            torch.cuda.synchronize()
            st = plan.debug_stats(reset=True)
            t = st["trace"]
            if r >= 2:
                rows.append([(v - t[0]) if v else -1 for v in t])
                lb.append(st)
        med = [sorted(c)[len(c) // 2] for c in zip(*rows)]
        nl = max(1, sum(s["lookbacks"] for s in lb))
        per = {k: round(sum(s[k] for s in lb) / nl, 2) for k in ("windows", "waits", "depth_sum", "cyc_lookback",
                                                                  "cyc_sleep", "cyc_load", "cyc_fold")}
        print(json.dumps({"sig": name, "n": n, "ns_after_entry": dict(zip(NAMES, med)),
                          "per_lookback_mean": per}), flush=True)
        plan.close()
