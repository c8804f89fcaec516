# round-2 batch d: bench (+ reference arm), launch list, ncu captures, float error table
set -x
TAG=${TAG:-r03d}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${TAG}_smi.txt
timeout 900 python bench.py > gpurun_out/${TAG}_bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/${TAG}_bench.log
timeout 300 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/${TAG}_bench_ref.log 2>&1
for v in "" rrA rrB rrC rrD; do
  lib=paper_conf_asplos_malekib18_b200/libplr_b200${v:+_$v}.so
  [ -f $lib ] && PLR_LIB=$lib timeout 150 python tools/time_sigs.py $((1<<30)) tuple2,tuple3,order2,order3 > gpurun_out/${TAG}_times_rr${v:-base}.log 2>&1
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 3 --warmup 3 --no-extras > gpurun_out/${TAG}_bench_ncu.log 2>&1
KEEP_REPS="" bash tools/ncu_profile.sh ${TAG} "${NCU_SIGS:-tuple2 tuple3 hp3 lp3}"
PLR_LIB=paper_conf_asplos_malekib18_b200/libplr_b200_trace.so timeout 300 python tools/trace_small.py > gpurun_out/${TAG}_trace_small.jsonl 2>&1
timeout 600 python tools/sweep.py prefix,tuple2,order3,lp1,hp3 10 22 > gpurun_out/${TAG}_sweep_auto.jsonl 2> gpurun_out/${TAG}_sweep_auto.err
timeout 900 python tools/float_err.py > gpurun_out/${TAG}_float_err.md 2> gpurun_out/${TAG}_float_err.err
true
