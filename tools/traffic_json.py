"""Write profiles/ncu_scan_traffic.json (bench.py's roofline "traffic") from an
ncu summary of the bench kernels: dram read+write bytes per launch, averaged
over the captures whose name ends with one of the bench signatures.
Usage: python tools/traffic_json.py profiles/<tag>_ncu_summary.json [sig,sig]"""
import json
import sys

src = sys.argv[1]
sigs = (sys.argv[2] if len(sys.argv) > 2 else "tuple2,tuple3").split(",")
d = json.load(open(src))
d = {k: v for k, v in d.items() if any(k.endswith("_" + s) for s in sigs)}
per = {k: v["dram_bytes_per_launch"] for k, v in d.items()}
out = {"bytes_per_launch": sum(per.values()) / len(per), "per_capture": per,
       "kernels": {k: v["kernel"] for k, v in d.items()},
       "source": src + " (ncu --set full --clock-control none, one launch each, n = 2^30)"}
json.dump(out, open("profiles/ncu_scan_traffic.json", "w"), indent=1)
print(json.dumps(out, indent=1))
