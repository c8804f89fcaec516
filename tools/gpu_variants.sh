set -x
rm -f gpurun_out/lbstats.log
for v in "" _nt7 _nt5; do
  echo "== variant '$v'" >> gpurun_out/lbstats.log
  PLR_LIB=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200$v.so timeout 300 python tools/lookback_stats.py $((1<<30)) prefix,tuple2,tuple3 >> gpurun_out/lbstats.log 2>&1
done
