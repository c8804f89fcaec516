set -x
mkdir -p gpurun_out
for sig in prefix order3; do
  rep=gpurun_out/r04r_small_${sig}
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:plr_small -s 2 -c 1 -o $rep python tools/one_sig.py $sig 1048576 > ${rep}.log 2>&1
  python tools/ncu_lines.py ${rep}.ncu-rep 30 > ${rep}_lines.txt 2>&1
done
python tools/ncu_summary.py r04rs gpurun_out/r04r_small_*.ncu-rep > gpurun_out/r04rs_ncu_summary.log 2>&1
cp profiles/r04rs_ncu_summary.* gpurun_out/ 2>/dev/null
rm -f gpurun_out/r04r_small_*.ncu-rep
true
