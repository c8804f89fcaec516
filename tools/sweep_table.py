"""Render a sweep.py JSONL file as a markdown table of fractions of memcpy.
Usage: python tools/sweep_table.py gpurun_out/<tag>_sweep.jsonl"""
import json
import sys

rows = [json.loads(l) for l in open(sys.argv[1]) if l.startswith("{")]
sigs, ns = [], []
for r in rows:
    if r["sig"] not in sigs:
        sigs.append(r["sig"])
    if r["n"] not in ns:
        ns.append(r["n"])
d = {(r["sig"], r["n"]): r for r in rows}
print("| n | memcpy GB/s | " + " | ".join(sigs) + " |")
print("|---|---|" + "---|" * len(sigs))
for n in ns:
    first = d.get((sigs[0], n))
    cells = [("%.2f" % d[(s, n)]["frac_memcpy"]) if (s, n) in d else "-" for s in sigs]
    print("| %d | %.0f | %s |" % (n, first["memcpy_GB/s"] if first else 0, " | ".join(cells)))
print()
print("(fraction of an in-run device-to-device copy of the same bytes at each n; L2 flushed between repetitions)")
