"""Render tools/ablation.py JSONL as markdown.  Usage: python tools/ablation_table.py file.jsonl"""
import json
import sys

rows = [json.loads(l) for l in open(sys.argv[1]) if l.startswith("{")]
modes = []
for r in rows:
    if r["mode"] not in modes:
        modes.append(r["mode"])
d = {(r["sig"], r["mode"]): r for r in rows}
sigs = []
for r in rows:
    if r["sig"] not in sigs:
        sigs.append(r["sig"])
print("| signature | " + " | ".join("%s (frac memcpy, kernel)" % m for m in modes) + " |")
print("|---|" + "---|" * len(modes))
for s in sigs:
    cells = []
    for m in modes:
        r = d.get((s, m))
        cells.append("%.3f, %s" % (r["frac_memcpy"], r["kernel"].split(" ")[0]) if r else "-")
    print("| %s | %s |" % (s, " | ".join(cells)))
print()
print("n = %d; specialised = default plans; no_constsig = PLR_NO_CONSTSIG=1 (transfer tables from kernel "
      "parameters instead of compile-time constants); generic = PLR_FORCE_GENERIC=1 (no DECAY single-hop "
      "look-back / hierarchy specialisation, no constant tables: the multi-tile look-back kernel)" % rows[0]["n"])
