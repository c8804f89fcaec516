set -x
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "not full_size and not host_pipeline" > gpurun_out/pytest_quick.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_quick.log
timeout 300 python tools/lookback_stats.py $((1<<30)) prefix,tuple2,tuple3,order3,lp3,hp3 > gpurun_out/lbstats.log 2>&1; echo "rc=$?" >> gpurun_out/lbstats.log
