"""Dynamic SASS opcode mix of an ncu capture (source page, sass view):
warp-level instructions executed per opcode, and per element of the launch.
Usage: python tools/ncu_ops.py rep.ncu-rep [n_elements] [top]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
n = float(sys.argv[2]) if len(sys.argv) > 2 else float(1 << 30)
top = int(sys.argv[3]) if len(sys.argv) > 3 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = rows[1]
iS, iE, iT = hdr.index("Source"), hdr.index("Instructions Executed"), hdr.index("Thread Instructions Executed")
agg, tagg = {}, {}
for r in rows[2:]:
    if len(r) <= iT:
        continue
    src = r[iS].strip()
    toks = src.split()
    if not toks:
        continue
    op = toks[1] if toks[0].startswith("@") and len(toks) > 1 else toks[0]
    op = op.split(".")[0].rstrip(";")
    try:
        e, t = int(r[iE]), int(r[iT])
    except ValueError:
        continue
    agg[op] = agg.get(op, 0) + e
    tagg[op] = tagg.get(op, 0) + t
tot = sum(agg.values())
print("total warp inst %.3e  = %.2f warp-inst/elt, %.1f thread-inst/elt (32x)" % (tot, tot / n, 32 * tot / n))
print("%-10s %10s %8s %10s" % ("op", "warp-inst", "%", "thr/elt"))
for op, e in sorted(agg.items(), key=lambda kv: -kv[1])[:top]:
    print("%-10s %10.3e %7.1f%% %10.2f" % (op, e, 100.0 * e / tot, tagg[op] / n))
