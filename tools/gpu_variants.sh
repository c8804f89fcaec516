set -x
timeout 120 python tools/one_sig.py prefix 100000 > gpurun_out/tmem_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/tmem_smoke.log
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "not full_size and not host_pipeline" > gpurun_out/pytest_quick.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_quick.log
rm -f gpurun_out/lbstats.log
timeout 300 python tools/lookback_stats.py $((1<<30)) prefix,tuple2,tuple3,order2,order3,lp1,lp3,hp3 >> gpurun_out/lbstats.log 2>&1
