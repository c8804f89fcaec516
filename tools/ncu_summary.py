"""Summarise ncu --set full captures (.ncu-rep) into profiles/: key metrics,
stall reasons and the top SASS stall sites.  Usage:
    python tools/ncu_summary.py <tag> gpurun_out/<tag>_<sig>.ncu-rep ...
"""
import csv
import io
import json
import os
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread", "launch__grid_size",
        "launch__block_size", "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
        "lts__t_sectors_srcunit_tex.sum", "lts__t_sectors_srcunit_tex_evict_normal_lookup_hit.sum",
        "smsp__inst_executed.sum", "sm__cycles_elapsed.avg.per_second"]


def ncu(rep, page, extra=()):
    r = subprocess.run(["ncu", "-i", rep, "--page", page, "--csv", *extra], capture_output=True, text=True)
    return list(csv.reader(io.StringIO(r.stdout)))


def summarise(rep):
    rows = ncu(rep, "raw")
    hdr, units, vals = rows[0], rows[1], rows[2]
    kv = {h: (vals[i], units[i]) for i, h in enumerate(hdr)}
    out = {"kernel": kv.get("Kernel Name", ("?",))[0]}
    for k in KEYS:
        if k in kv:
            out[k] = kv[k][0] + (" " + kv[k][1] if kv[k][1] else "")
    stalls = []
    for i, h in enumerate(hdr):
        if "pcsamp_warps_issue_stalled" in h and not h.endswith("not_issued"):
            try:
                stalls.append((float(vals[i].replace(",", "")), h.split("stalled_")[-1]))
            except ValueError:
                pass
    tot = sum(v for v, _ in stalls) or 1
    out["stalls_pct"] = {n: round(100 * v / tot, 1) for v, n in sorted(stalls, reverse=True)[:8]}
    src = ncu(rep, "source", ["--print-source", "sass"])
    h2 = src[1]
    isrc, iss = h2.index("Source"), h2.index("Warp Stall Sampling (All Samples)")
    data = [r for r in src[2:] if len(r) > iss and r[iss].isdigit()]
    tot2 = sum(int(r[iss]) for r in data) or 1
    top = sorted(data, key=lambda r: -int(r[iss]))[:8]
    out["top_sass_stall_sites"] = ["%.1f%% %s" % (100 * int(r[iss]) / tot2, r[isrc].strip()) for r in top]

    def num(k):
        return float(kv[k][0].replace(",", ""))
    unit = {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1.0}
    rd = num("dram__bytes_read.sum") * unit.get(kv["dram__bytes_read.sum"][1], 1)
    wr = num("dram__bytes_write.sum") * unit.get(kv["dram__bytes_write.sum"][1], 1)
    out["dram_bytes_per_launch"] = rd + wr
    return out


def main():
    tag = sys.argv[1]
    res = {}
    for rep in sys.argv[2:]:
        name = os.path.basename(rep).replace(".ncu-rep", "")
        res[name] = summarise(rep)
    os.makedirs("profiles", exist_ok=True)
    with open("profiles/%s_ncu_summary.json" % tag, "w") as f:
        json.dump(res, f, indent=1)
    with open("profiles/%s_ncu_summary.md" % tag, "w") as f:
        for name, d in res.items():
            f.write("## %s\n\n" % name)
            for k, v in d.items():
                if isinstance(v, (list, dict)):
                    f.write("- %s:\n" % k)
                    for item in (v.items() if isinstance(v, dict) else enumerate(v)):
                        f.write("  - %s: %s\n" % item if isinstance(v, dict) else "  - %s\n" % item[1])
                else:
                    f.write("- %s: %s\n" % (k, v))
            f.write("\n")
    print(json.dumps(res, indent=1)[:3000])


if __name__ == "__main__":
    main()
