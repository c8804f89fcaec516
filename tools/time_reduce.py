"""Time the reduce-only pass (plr_reduce, reads n) against the single pass
and a read-only torch reduction at n (default 2^30): the sharded schedule's
first leg for non-decaying signatures.
Usage: python tools/time_reduce.py [n] [sig,sig,...]"""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_asplos_malekib18_b200 as plr  # noqa: E402
import workloads  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 1 << 30
names = sys.argv[2].split(",") if len(sys.argv) > 2 else ["prefix", "tuple2", "tuple3", "order2", "order3"]
xi = workloads.device_input(n, "int32", 1)
y = torch.empty_like(xi)
pl = torch.empty(64, dtype=torch.uint8, device="cuda")


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
ms_rd = timed(lambda: torch.sum(xi, dtype=torch.int64))
print("memcpy %.3f ms (%.0f GB/s r+w)   torch.sum %.3f ms (%.0f GB/s read)" % (
    ms_cp, 8 * n / ms_cp / 1e6, ms_rd, 4 * n / ms_rd / 1e6), flush=True)
for name in names:
    sig = workloads.BY_NAME[name]
    plan = plr.Plan(sig.a, sig.b, sig.dtype, n_max=n)
    ms_scan = timed(lambda: plan(xi, y))
    ms_red = timed(lambda: plan.reduce(xi, pl))

    class One:
        rank, world, handle = 0, 1, None
    ms_sh = timed(lambda: plan.sharded(xi, y, comm=One()), reps=5)
    print("%-7s scan %.3f ms  reduce %.3f ms (%.0f GB/s read, %.2f of torch.sum)  sharded(w=1) %.3f ms "
          "-> vs single %.3f (bound 2n/3n = 0.667 at equal rates)" % (
              name, ms_scan, ms_red, 4 * n / ms_red / 1e6, ms_rd / ms_red, ms_sh, ms_scan / ms_sh), flush=True)
    plan.close()
