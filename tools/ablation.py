"""Fig. 10 analogue on B200: every Table-1
signature at n (default 2^30) with the class specialisations on (default),
with compile-time signature tables off (PLR_NO_CONSTSIG=1: tables read from
kernel parameters) and with every specialisation off (PLR_FORCE_GENERIC=1:
generic multi-tile look-back kernel, no DECAY single hop, no constant
tables).  Prints one JSON line per (signature, mode)."""
import json
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_asplos_malekib18_b200 as plr  # noqa: E402
import workloads  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 30
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
MODES = {"specialised": {}, "no_constsig": {"PLR_NO_CONSTSIG": "1"}, "generic": {"PLR_FORCE_GENERIC": "1"}}
for sig in workloads.TABLE1:
    x = xi if sig.dtype == "int32" else xf
    yy = y if sig.dtype == "int32" else y.view(torch.float32)
    for mode, env in MODES.items():
        for k in ("PLR_NO_CONSTSIG", "PLR_FORCE_GENERIC"):
            os.environ.pop(k, None)
        os.environ.update(env)
        plan = plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
        ms = timed(lambda: plan(x, yy))
        print(json.dumps({"sig": sig.name, "mode": mode, "n": n, "ms": round(ms, 4),
                          "GB/s": round(8 * n / ms / 1e6, 1), "frac_memcpy": round(ms_cp / ms, 4),
                          "kernel": plan.kernel_name(), "tile": plan.info["tile_elems"]}), flush=True)
        plan.close()
for k in ("PLR_NO_CONSTSIG", "PLR_FORCE_GENERIC"):
    os.environ.pop(k, None)
