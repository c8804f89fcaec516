# round-2 batch c: DECAY fp64 geometry variants, full GPU suite, Scan comparison, big-kernel sweep
set -x
TAG=${TAG:-r03c}
mkdir -p gpurun_out
timeout 120 python tools/time_sigs.py $((1<<30)) lp1,lp2,hp1,hp2,lp3,hp3 > gpurun_out/${TAG}_times_base.log 2>&1
for v in d64a d64b d64c; do
  PLR_LIB=paper_conf_asplos_malekib18_b200/libplr_b200_$v.so timeout 120 python tools/time_sigs.py $((1<<30)) lp3,hp3 > gpurun_out/${TAG}_times_$v.log 2>&1
done
PLR_LIB=paper_conf_asplos_malekib18_b200/libplr_b200_trace.so timeout 300 python tools/trace_small.py > gpurun_out/${TAG}_trace_small.jsonl 2>&1
PLR_SMALL_MAX=0 timeout 500 python tools/sweep.py prefix,tuple2,order3,lp1,hp3 10 22 > gpurun_out/${TAG}_sweep_big.jsonl 2> gpurun_out/${TAG}_sweep_big.err
timeout 600 python tools/scan_compare.py > gpurun_out/${TAG}_scan_compare.jsonl 2> gpurun_out/${TAG}_scan_compare.err
timeout 2300 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
true
