# ncu evidence for the scan kernel (one GPU).  Usage: bash tools/ncu_profile.sh <tag> [sigs]
set -x
TAG=${1:-r01}
SIGS=${2:-tuple2 prefix lp1 hp3}
mkdir -p gpurun_out
for sig in $SIGS; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:plr_scan -s 2 -c 1 \
      -o gpurun_out/${TAG}_${sig} python tools/one_sig.py $sig > gpurun_out/${TAG}_${sig}.log 2>&1
done
