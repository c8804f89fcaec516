# round-2 batch n: re-read kernel stage split / width variants at 2^30
# (rra3: SA=3 SB=4, rra4: SA=4 SB=3, rrw16: W=16 X=15), reduce-pass parity
set -x
TAG=${TAG:-r03n}
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q -x --timeout 300 -p no:cacheprovider -k "reduce or sharded" \
    > gpurun_out/${TAG}_pytest_sel.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_sel.log
TAG=${TAG} VARS="base rra3 rra4 rrw16 base" SIGS=tuple2,tuple3,order2,order3 bash tools/gpu_cmp.sh
true
