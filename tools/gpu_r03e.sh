# round-2 batch e: fp64 DECAY geometry variants, fp32 DECAY A/B vs the round-1 library, small-n v2 (+ geometry variants), 2^30 times, full suite
set -x
TAG=${TAG:-r03e}
mkdir -p gpurun_out
L=paper_conf_asplos_malekib18_b200
for v in "" d64e d64f; do
  lib=$L/libplr_b200${v:+_$v}.so
  [ -f $lib ] && PLR_LIB=$lib timeout 120 python tools/time_sigs.py $((1<<30)) lp3,hp3 > gpurun_out/${TAG}_times_dec64_${v:-base}.log 2>&1
done
timeout 120 python tools/time_sigs.py $((1<<30)) lp1,lp2,hp1,hp2 > gpurun_out/${TAG}_times_dec32_now.log 2>&1
[ -d ab_r1 ] && timeout 120 python ab_r1/tools/time_sigs.py $((1<<30)) lp1,lp2,hp1,hp2 > gpurun_out/${TAG}_times_dec32_r1.log 2>&1
timeout 120 python tools/time_sigs.py $((1<<30)) lp1,lp2,hp1,hp2 > gpurun_out/${TAG}_times_dec32_now2.log 2>&1
PLR_LIB=$L/libplr_b200_trace.so timeout 300 python tools/trace_small.py > gpurun_out/${TAG}_trace_small.jsonl 2>&1
PLR_LIB=$L/libplr_b200_sm16t.so timeout 300 python tools/trace_small.py > gpurun_out/${TAG}_trace_small_sm16.jsonl 2>&1
timeout 400 python tools/sweep.py prefix,tuple2,order3,lp1,hp3 10 22 > gpurun_out/${TAG}_sweep_auto.jsonl 2> gpurun_out/${TAG}_sweep_auto.err
for v in sm16; do
  PLR_LIB=$L/libplr_b200_$v.so timeout 400 python tools/sweep.py prefix,tuple2,order3,lp1,hp3 16 22 > gpurun_out/${TAG}_sweep_$v.jsonl 2> gpurun_out/${TAG}_sweep_$v.err
done
timeout 400 python tools/time_sigs.py $((1<<30)) > gpurun_out/${TAG}_times.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
true
