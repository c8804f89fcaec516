"""Repeat one signature at given sizes and count mismatching runs vs the oracle.
Usage: python tools/stress.py sig n1,n2,... reps"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
import oracle  # noqa: E402
import paper_conf_asplos_malekib18_b200 as plr  # noqa: E402
import workloads  # noqa: E402

sig = workloads.BY_NAME[sys.argv[1]]
sizes = [int(v) for v in sys.argv[2].split(",")]
reps = int(sys.argv[3])
x_all = workloads.host_input(max(sizes), sig.dtype, workloads.seed_for(1))
plan = plr.Plan(sig.a, sig.b, sig.dtype, n_max=max(sizes))
for n in sizes:
    x = x_all[:n].copy()
    ref = oracle.recurrence(x, sig.a, sig.b, sig.dtype)
    xd = torch.from_numpy(x).cuda()
    bad = []
    for r in range(reps):
        y = plan(xd).cpu().numpy()
        if sig.dtype == "int32":
            nb = int(np.count_nonzero(y != ref))
        else:
            nb = int(np.count_nonzero(np.abs(y - ref) / np.maximum(1, np.abs(ref)) > 1e-4))
        if nb:
            bad.append((r, nb, int(np.flatnonzero(y != ref)[0]) if sig.dtype == "int32" else -1))
    print(sig.name, n, "bad runs %d/%d" % (len(bad), reps), bad[:5], flush=True)
