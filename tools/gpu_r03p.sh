# round-2 batch p: small-n cluster look-back (parity, sweep on/off), TMEM
# generic kernel at the wide geometry (tmw16: X=31 W=16 SL=2 ST=1 G=1; tmw16g2: G=2)
set -x
TAG=${TAG:-r03p}
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x --timeout 300 -p no:cacheprovider \
    -k "cluster or small_n or parity_sizes or continue or graph" > gpurun_out/${TAG}_pytest_sel.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_sel.log
for c in 1 0; do
  PLR_SMALL_CLUSTER=$c timeout 400 python tools/sweep.py prefix,tuple2,tuple3,order2,order3 10 22 > gpurun_out/${TAG}_sweep_c$c.jsonl 2> gpurun_out/${TAG}_sweep_c$c.err
done
TAG=${TAG} VARS="base tmw16 tmw16g2" SIGS=prefix,tuple2,tuple3,order2,order3 bash tools/gpu_cmp.sh
true
