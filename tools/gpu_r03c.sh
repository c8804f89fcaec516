# round-2 batch c: full GPU suite, Scan comparison, big-kernel sweep
set -x
TAG=${TAG:-r03c}
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 600 python tools/scan_compare.py > gpurun_out/${TAG}_scan_compare.jsonl 2> gpurun_out/${TAG}_scan_compare.err
PLR_SMALL_MAX=0 timeout 500 python tools/sweep.py prefix,tuple2,order3,lp1,hp3 10 22 > gpurun_out/${TAG}_sweep_big.jsonl 2> gpurun_out/${TAG}_sweep_big.err
true
