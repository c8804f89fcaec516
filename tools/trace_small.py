"""Critical path of CTA 0 in one small launch of the re-read kernel: globaltimer
stamps (PLR_TRACE variant build, PLR_STATS=1), ns after the init barrier.
Usage: PLR_LIB=.../libplr_b200_trace.so python tools/trace_small.py"""
import json
import os
import sys
os.environ["PLR_STATS"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_asplos_malekib18_b200 as plr  # noqa: E402
import workloads  # noqa: E402

NAMES = ["init", "entry", "lookback_unit0_done", "lookback_warp_exit", "storer_saw_stop", "storer_exit", "compute_end"]
for name in ["tuple2", "order3"]:
    for n in [1024, 7936 * 4, 1 << 20, 1 << 22]:
        sig = workloads.BY_NAME[name]
        x = workloads.device_input(n, sig.dtype, 1)
        y = torch.empty_like(x)
        plan = plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
        rows = []
        for r in range(6):
            plan(x, y)
            torch.cuda.synchronize()
            t = plan.debug_stats(reset=True)["trace"]
            if r >= 2:
                rows.append([(v - t[0]) if v else -1 for v in t])
        med = [sorted(c)[len(c) // 2] for c in zip(*rows)]
        print(json.dumps({"sig": name, "n": n, "ns_after_init": dict(zip(NAMES, med))}), flush=True)
        plan.close()
