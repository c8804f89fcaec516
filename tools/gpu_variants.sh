set -x
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "not full_size and not host_pipeline" > gpurun_out/pytest_quick.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_quick.log
rm -f gpurun_out/lbstats.log
for v in "" _t1 _t2 _t3; do
  echo "== variant '$v'" >> gpurun_out/lbstats.log
  PLR_LIB=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200$v.so timeout 300 python tools/lookback_stats.py $((1<<30)) prefix,tuple2,tuple3,order2 >> gpurun_out/lbstats.log 2>&1
done
