# round-2 batch m: small-n prefetch (constant-cache warm-up, lane_T via smem,
# deferred launch-state read) and the reduce pass's parallel record fold,
# A/B against the HEAD library (libplr_b200_base.so)
set -x
TAG=${TAG:-r03m}
mkdir -p gpurun_out
L=paper_conf_asplos_malekib18_b200
timeout 900 python -m pytest tests -m gpu -q -x --timeout 300 -p no:cacheprovider \
    -k "small_n or reduce or sharded or graph or parity_sizes or structured or repeated or continue" \
    > gpurun_out/${TAG}_pytest_sel.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_sel.log
for v in base ""; do
  lib=$L/libplr_b200${v:+_$v}.so
  PLR_LIB=$lib timeout 400 python tools/sweep.py prefix,tuple2,order3,lp1,hp3 10 22 > gpurun_out/${TAG}_sweep_${v:-new}.jsonl 2> gpurun_out/${TAG}_sweep_${v:-new}.err
  PLR_LIB=$lib timeout 300 python tools/time_reduce.py > gpurun_out/${TAG}_reduce_${v:-new}.log 2>&1
done
PLR_LIB=$L/libplr_b200_trace.so timeout 300 python tools/trace_small.py > gpurun_out/${TAG}_trace_small.jsonl 2>&1
true
