# final check of the round's tree: smoke, all gpu tests, bench
set -x
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02q_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/r02q_smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r02q_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r02q_pytest_gpu.log
timeout 600 python bench.py > gpurun_out/r02q_bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/r02q_bench.log
true
