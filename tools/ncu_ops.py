"""Per-opcode executed warp instructions per unit of work from an ncu capture.
Usage: python tools/ncu_ops.py rep.ncu-rep units [top]"""
import collections
import csv
import io
import subprocess
import sys

rep, units = sys.argv[1], float(sys.argv[2])
top = int(sys.argv[3]) if len(sys.argv) > 3 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = next(r for r in rows if r and r[0] == "Address")
isrc, iex = hdr.index("Source"), hdr.index("Instructions Executed")
ops = collections.Counter()
for r in rows:
    if len(r) <= iex or not r[iex].isdigit():
        continue
    toks = [t for t in r[isrc].split() if not t.startswith("@")]
    if toks:
        ops[toks[0].split(".")[0]] += int(r[iex])
tot = sum(ops.values())
print("total %.0f warp-inst per unit" % (tot / units))
for op, c in ops.most_common(top):
    print("%-10s %8.1f  %4.1f%%" % (op, c / units, 100.0 * c / tot))
