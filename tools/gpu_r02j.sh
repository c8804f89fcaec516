# device-side launch state (CUDA-graph replayable launches): gpu tests, smoke, small-n timings, bench
set -x
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02j_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/r02j_smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r02j_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r02j_pytest_gpu.log
timeout 600 python bench.py > gpurun_out/r02j_bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/r02j_bench.log
timeout 300 python tools/small_n.py > gpurun_out/r02j_small_n_host.jsonl 2>&1
SMALLN_HOST=0 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02j_small_n.csv python tools/small_n.py > gpurun_out/r02j_small_n_ncu.log 2>&1
python tools/small_n.py --parse gpurun_out/r02j_small_n.csv > gpurun_out/r02j_small_n.md 2>&1
timeout 300 python tools/time_sigs.py $((1<<30)) > gpurun_out/r02j_times.log 2>&1
true
