set -x
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "not full_size" > gpurun_out/pytest_q.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_q.log
timeout 300 python tools/time_sigs.py $((1<<30)) > gpurun_out/times_q.log 2>&1
timeout 300 python tools/lookback_stats.py $((1<<30)) prefix,tuple2,tuple3,order2,order3 > gpurun_out/lb_q.log 2>&1
