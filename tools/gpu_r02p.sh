# stop-aware wait experiment: PLR_POLL_HINT_NS 0 (trace) vs 200 vs 2000 ns: trace, small-n graph times, 2^30 times
mkdir -p gpurun_out
for v in trace h200 h2000; do
  lib=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200_$v.so
  PLR_LIB=$lib timeout 120 python tools/trace_small.py > gpurun_out/r02p_trace_$v.jsonl 2>&1
  PLR_LIB=$lib timeout 200 python tools/small_n.py > gpurun_out/r02p_small_n_host_$v.jsonl 2>&1
  PLR_LIB=$lib timeout 200 python tools/time_sigs.py 1073741824 > gpurun_out/r02p_times_$v.txt 2>&1
done
true
