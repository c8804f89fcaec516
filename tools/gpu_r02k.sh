# small-n ncu --set full captures (where the fixed per-launch device time goes)
set -x
mkdir -p gpurun_out
for spec in "tuple2 1024" "tuple2 1048576" "prefix 1024" "lp1 1024"; do
  set -- $spec
  rep=gpurun_out/r02k_${1}_n$2
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:plr_scan -s 2 -c 1 \
      -o $rep python tools/one_sig.py $1 $2 > ${rep}.log 2>&1
  python tools/ncu_lines.py ${rep}.ncu-rep 40 > ${rep}_lines.txt 2>&1
done
python tools/ncu_summary.py r02k gpurun_out/r02k_*.ncu-rep > gpurun_out/r02k_ncu_summary.log 2>&1
cp profiles/r02k_ncu_summary.* gpurun_out/ 2>/dev/null
rm -f gpurun_out/r02k_*.ncu-rep
true
