"""Per-source-line warp-stall samples of an ncu capture (cuda,sass view).
Usage: python tools/ncu_lines.py rep.ncu-rep [top]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 and sys.argv[2].isdigit() else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
agg = {}
inst = {}
cur = None
fname = "?"
for row in csv.reader(io.StringIO(out)):
    if len(row) == 2 and row[0] == "File Path":
        fname = row[1].split("/")[-1]
        continue
    if len(row) < 5 or row[0] == "Line No":
        continue
    if row[0]:
        cur = (fname, row[0], row[1].strip()[:90])
    try:
        s = int(row[4])
    except ValueError:
        continue
    try:
        ie = int(row[7])
    except (ValueError, IndexError):
        ie = 0
    if cur:
        agg[cur] = agg.get(cur, 0) + s
        inst[cur] = inst.get(cur, 0) + ie
tot = sum(agg.values()) or 1
itot = sum(inst.values()) or 1
key = (lambda kv: -inst[kv[0]]) if "--inst" in sys.argv else (lambda kv: -kv[1])
print("stall%  inst%  line")
for (f, ln, src), s in sorted(agg.items(), key=key)[:top]:
    print("%5.1f%% %5.1f%%  %s:%s  %s" % (100.0 * s / tot, 100.0 * inst[(f, ln, src)] / itot, f, ln, src))
