"""Small-grid launches of every scan-kernel family for compute-sanitizer
(memcheck / racecheck / synccheck): a few tiles each, checked against the
oracle.  Usage: compute-sanitizer --tool T python tools/sanitize_run.py
(PLR_SMALL_MAX=0: the persistent kernels; default: the small-n kernel,
cluster launches for the non-decaying rows)"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_asplos_malekib18_b200 as plr  # noqa: E402
import workloads  # noqa: E402

CASES = [("prefix", 40000), ("tuple3", 70000), ("order2", 9000), ("lp1", 30000), ("hp3", 30000), ("hp2", 12345)]
bad = 0
for name, n in CASES:
    sig = workloads.BY_NAME[name]
    x = workloads.host_input(n, sig.dtype, 77)
    plan = plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
    for _ in range(2):
        y = plan(torch.from_numpy(x).cuda()).cpu().numpy()
    ref = oracle.recurrence(x, sig.a, sig.b, sig.dtype)
    if sig.dtype == "int32":
        ok = np.array_equal(y, ref)
    else:
        ok = float(np.max(np.abs(y - ref) / np.maximum(1, np.abs(ref)))) <= 1e-4
    info = plan.info
    kern = plan.kernel_name() if n > info["small_max"] else (
        "plr_small_kernel" + (" (clusters of %d)" % info["small_cluster_ctas"]
                              if info["small_clusters"] > 0 and os.environ.get("PLR_SMALL_CLUSTER", "1") != "0" else ""))
    print(name, n, kern, "ok" if ok else "MISMATCH", flush=True)
    bad += not ok
    plan.close()
torch.cuda.synchronize()
print("cases", len(CASES), "bad", bad)
