# the measurement set at HEAD -- bench (+ reference arm), launch list, ncu captures
# (bench kernels, fp64 DECAY, reduce-only), worst float error, ablation, size sweep, reduce timing
set -x
TAG=${TAG:-head}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${TAG}_smi.txt
timeout 1200 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 200 python tools/time_sigs.py $((1<<30)) > gpurun_out/${TAG}_times.log 2>&1
timeout 300 python tools/time_sigs.py $((1<<30)) "" reverse > gpurun_out/${TAG}_times_reverse.log 2>&1
timeout 300 python tools/time_sigs.py $((1<<30)) "" bidir > gpurun_out/${TAG}_times_bidir.log 2>&1
timeout 900 python bench.py > gpurun_out/${TAG}_bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/${TAG}_bench.log
timeout 300 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/${TAG}_bench_ref.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 3 --warmup 3 --no-extras > gpurun_out/${TAG}_bench_ncu.log 2>&1
KEEP_REPS="" bash tools/ncu_profile.sh ${TAG} "tuple2 tuple3 hp3 lp3 order3"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:plr_reduce -s 2 -c 1 -o gpurun_out/${TAG}_reduce_prefix python tools/one_sig.py prefix $((1<<30)) reduce > gpurun_out/${TAG}_reduce_prefix.log 2>&1
python tools/ncu_summary.py ${TAG}r gpurun_out/${TAG}_reduce_prefix.ncu-rep > gpurun_out/${TAG}r_ncu_summary.log 2>&1; cp profiles/${TAG}r_ncu_summary.* gpurun_out/ 2>/dev/null; rm -f gpurun_out/${TAG}_reduce_prefix.ncu-rep
timeout 900 python tools/float_err.py > gpurun_out/${TAG}_float_err.md 2> gpurun_out/${TAG}_float_err.err
timeout 600 python tools/ablation.py > gpurun_out/${TAG}_ablation.jsonl 2> gpurun_out/${TAG}_ablation.err
timeout 900 python tools/sweep.py > gpurun_out/${TAG}_sweep.jsonl 2> gpurun_out/${TAG}_sweep.err
timeout 300 python tools/time_reduce.py > gpurun_out/${TAG}_reduce.log 2>&1
true
