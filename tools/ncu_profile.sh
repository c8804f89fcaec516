# ncu evidence for the scan kernel (one GPU).  Usage: bash tools/ncu_profile.sh <tag> [sigs]
# Each capture is summarised on the box (profiles-style markdown, opcode mix,
# per-line stalls); the .ncu-rep is kept only for sigs listed in $KEEP_REPS
# (gpurun copies back at most 64 MiB).
set -x
TAG=${1:-r01}
SIGS=${2:-tuple2 prefix lp1 hp3}
mkdir -p gpurun_out
for sig in $SIGS; do
  rep=gpurun_out/${TAG}_${sig}
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:plr_scan -s 2 -c 1 \
      -o $rep python tools/one_sig.py $sig > ${rep}.log 2>&1
  python tools/ncu_ops.py ${rep}.ncu-rep > ${rep}_ops.txt 2>&1
  python tools/ncu_lines.py ${rep}.ncu-rep 40 > ${rep}_lines.txt 2>&1
  case " $KEEP_REPS " in *" $sig "*) ;; *) mkdir -p gpurun_out/reps_${TAG}; mv ${rep}.ncu-rep gpurun_out/reps_${TAG}/ ;; esac
done
# summaries need the reps: summarise everything captured this call, then drop the unkept ones
python tools/ncu_summary.py ${TAG} $(ls gpurun_out/${TAG}_*.ncu-rep gpurun_out/reps_${TAG}/*.ncu-rep 2>/dev/null) > gpurun_out/${TAG}_ncu_summary.log 2>&1
cp profiles/${TAG}_ncu_summary.* gpurun_out/ 2>/dev/null
rm -rf gpurun_out/reps_${TAG}
