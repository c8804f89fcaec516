# full GPU check: smoke, all -m gpu tests, per-signature timings, bench, ncu
# (launch list of the bench command + full captures), ablation, size sweep
# usage: TAG=r01x [NCU_SIGS="..."] [NONCU=1] [NOEXTRA=1] bash tools/gpu_round.sh
set -x
TAG=${TAG:-r01}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${TAG}_smi.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${TAG}_smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 300 python tools/time_sigs.py $((1<<30)) > gpurun_out/${TAG}_times.log 2>&1
timeout 600 python bench.py > gpurun_out/${TAG}_bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/${TAG}_bench.log
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/${TAG}_bench_ref.log 2>&1
if [ -z "$NONCU" ]; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 3 --warmup 3 > gpurun_out/${TAG}_bench_ncu.log 2>&1
  bash tools/ncu_profile.sh ${TAG} "${NCU_SIGS:-tuple2 tuple3}"
fi
if [ -z "$NOEXTRA" ]; then
  timeout 300 python tools/small_n.py > gpurun_out/${TAG}_small_n_host.jsonl 2>&1
  SMALLN_HOST=0 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_small_n.csv python tools/small_n.py > gpurun_out/${TAG}_small_n_ncu.log 2>&1
  python tools/small_n.py --parse gpurun_out/${TAG}_small_n.csv > gpurun_out/${TAG}_small_n.md 2>&1
  timeout 600 python tools/ablation.py > gpurun_out/${TAG}_ablation.jsonl 2> gpurun_out/${TAG}_ablation.err
  timeout 600 python tools/sweep.py > gpurun_out/${TAG}_sweep.jsonl 2> gpurun_out/${TAG}_sweep.err
fi
true
[ -n "$CMP_VARS" ] && TAG=${TAG} VARS="$CMP_VARS" SIGS=${CMP_SIGS:-prefix,tuple2,tuple3,order2,order3} bash tools/gpu_cmp.sh
true
