timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r02h_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r02h_pytest.log
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/r02h_bench.log 2>&1; echo rc=$? >> gpurun_out/r02h_bench.log
