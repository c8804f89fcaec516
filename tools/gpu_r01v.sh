mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r01v_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r01v_pytest.log
timeout 300 python tools/time_sigs.py 1073741824 > gpurun_out/r01v_times.log 2>&1
for s in order3 tuple2; do timeout 200 python tools/stress.py $s 1060921,33554432,7937,40000000 10 >> gpurun_out/r01v_stress.log 2>&1; done
TAG=r01v VARS="h1 h3 h4 h5" SIGS=hp3 bash tools/gpu_cmp.sh
timeout 600 python tools/sweep.py > gpurun_out/r01v_sweep.jsonl 2> gpurun_out/r01v_sweep.err
