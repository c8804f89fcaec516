# round-2 batch 04e: re-read kernel runtime phase-B lag (PLR_RR_LAG 5..9, default 9) at medium and large n
set -x
TAG=${TAG:-r04e}
mkdir -p gpurun_out
for lg in 9 7 5; do
  PLR_RR_LAG=$lg timeout 400 python tools/sweep.py tuple2,tuple3,order2,order3 21 25 > gpurun_out/${TAG}_sweep_l$lg.jsonl 2> gpurun_out/${TAG}_sweep_l$lg.err
  PLR_RR_LAG=$lg timeout 400 python tools/sweep.py tuple2,tuple3,order2,order3 22 28 > gpurun_out/${TAG}_sweep_e_l$lg.jsonl 2> gpurun_out/${TAG}_sweep_e_l$lg.err
done
PLR_RR_LAG=5 timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x --timeout 300 -p no:cacheprovider -k "(tuple or order) and (sizes or structured or graph or continue)" > gpurun_out/${TAG}_pytest_l5.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_l5.log
true
