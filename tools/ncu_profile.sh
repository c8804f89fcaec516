# ncu evidence for the scan kernel (one GPU).  Usage: bash tools/ncu_profile.sh <tag>
set -x
TAG=${1:-r01}
mkdir -p gpurun_out
# 1) launch list of a short bench run (cold-cache, serialised: compare shares)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv \
    --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 3 --warmup 3 --no-extras > gpurun_out/${TAG}_launches_bench.log 2>&1
# 2) full capture of one scan launch per signature class at 2^30
for sig in tuple2 prefix lp1 hp3; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:plr_scan_kernel -s 2 -c 1 \
      -o gpurun_out/${TAG}_${sig} python tools/one_sig.py $sig > gpurun_out/${TAG}_${sig}.log 2>&1
done
