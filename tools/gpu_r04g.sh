# round-2 batch 04g: the zero-lag fix -- runtime-lag parity, the whole GPU suite, sweep
set -x
TAG=${TAG:-r04g}
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x --timeout 120 -p no:cacheprovider -k "runtime_lag" > gpurun_out/${TAG}_pytest_lag.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_lag.log
timeout 1800 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 900 python tools/sweep.py > gpurun_out/${TAG}_sweep.jsonl 2> gpurun_out/${TAG}_sweep.err
true
