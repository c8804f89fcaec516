"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) of a
bench.py run: per kernel name, launches and total/avg duration, plus the
scan kernel's share of the first timed-step window.
Usage: python tools/launch_list.py gpurun_out/launches.csv > profiles/<tag>_launches.md"""
import csv
import sys

rows = []
with open(sys.argv[1]) as f:
    lines = [l for l in f if l.startswith('"')]
for r in csv.DictReader(lines):
    if r["Metric Name"] != "gpu__time_duration.sum":
        continue
    v = float(r["Metric Value"].replace(",", ""))
    unit = r["Metric Unit"]
    us = v / 1000.0 if unit in ("ns", "nsecond") else v * 1000.0 if unit in ("ms", "msecond") else v
    name = r["Kernel Name"]
    short = name.split("(")[0].replace("void ", "")[:110]
    rows.append((int(r["ID"]), short, us, r["Grid Size"], r["Block Size"]))
agg = {}
for _, n, us, g, b in rows:
    a = agg.setdefault(n, [0, 0.0, g, b])
    a[0] += 1
    a[1] += us
tot = sum(a[1] for a in agg.values())
print("# ncu launch list (%d launches, %.1f ms total kernel time)\n" % (len(rows), tot / 1000))
print("| kernel | launches | total ms | avg us | share | grid | block |")
print("|---|---|---|---|---|---|---|")
for n, (c, t, g, b) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    print("| `%s` | %d | %.2f | %.1f | %.1f%% | %s | %s |" % (n, c, t / 1000, t / c, 100 * t / tot, g, b))
print("\n## first 60 launches in order\n")
for i, n, us, g, b in rows[:60]:
    print("- %d `%s` %.1f us grid %s block %s" % (i, n, us, g, b))
