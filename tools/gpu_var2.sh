# time variants (PLR_LIB) and collect look-back stats for each
set -x
mkdir -p gpurun_out
rm -f gpurun_out/variants4.log
for v in $VARS; do
  [ "$v" = "base" ] && v=""
  echo "== variant '$v'" >> gpurun_out/variants4.log
  PLR_LIB=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200$v.so timeout 300 python tools/lookback_stats.py $((1<<30)) ${SIGS:-prefix,tuple2,tuple3,order2,order3} >> gpurun_out/variants4.log 2>&1
done
[ -n "$NCU" ] && bash tools/ncu_profile.sh r01e "$NCU"
