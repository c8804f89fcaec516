timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r01r_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r01r_pytest.log
timeout 300 python tools/time_sigs.py 1073741824 > gpurun_out/r01r_times.log 2>&1
TAG=r01r VARS="rx31w8 rx23w8 rns9" SIGS=tuple2,tuple3,order2,order3 bash tools/gpu_cmp.sh
