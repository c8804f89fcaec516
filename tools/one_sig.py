"""Run one Table-1 signature a few times at n (default 2^30): profiling target.
Usage: python tools/one_sig.py sig [n] [scan|reduce|reverse]"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_asplos_malekib18_b200 as plr  # noqa: E402
import workloads  # noqa: E402

name = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 1 << 30
mode = sys.argv[3] if len(sys.argv) > 3 else "scan"
sig = workloads.BY_NAME[name]
x = workloads.device_input(n, sig.dtype, 1)
y = torch.empty_like(x)
plan = plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
for _ in range(4):
    if mode == "reduce":
        plan.reduce(x)
    elif mode == "reverse":
        plan.reverse(x, y)
    else:
        plan(x, y)
torch.cuda.synchronize()
print("done", name, n)
