# round-2 batch q: the TMEM generic kernel for k >= 2 at its default geometry
# (tmk: G=3, tmkg2: G=2) vs the re-read kernel; ncu of the small-n kernel at 2^20
set -x
TAG=${TAG:-r03q}
mkdir -p gpurun_out
TAG=${TAG} VARS="base tmk tmkg2" SIGS=tuple2,tuple3,order2,order3 bash tools/gpu_cmp.sh
for sig in prefix tuple2; do
  rep=gpurun_out/${TAG}_small_${sig}
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:plr_small -s 2 -c 1 \
      -o $rep python tools/one_sig.py $sig 1048576 > ${rep}.log 2>&1
  python tools/ncu_lines.py ${rep}.ncu-rep 40 > ${rep}_lines.txt 2>&1
done
python tools/ncu_summary.py ${TAG}s gpurun_out/${TAG}_small_*.ncu-rep > gpurun_out/${TAG}s_ncu_summary.log 2>&1
cp profiles/${TAG}s_ncu_summary.* gpurun_out/ 2>/dev/null
true
