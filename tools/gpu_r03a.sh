# round-2 batch a: smoke, hang variants stress, full GPU suite, float error table, sanitizers
set -x
TAG=${TAG:-r03a}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/${TAG}_smi.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${TAG}_smoke.log
SIZES=1183745,7936005,4195081,16777216
for v in "" _hangA _hangB _hangC; do
  for s in tuple3 order3 prefix; do
    PLR_LIB=paper_conf_asplos_malekib18_b200/libplr_b200$v.so timeout 240 python tools/stress.py $s $SIZES 250 >> gpurun_out/${TAG}_stress$v.log 2>&1
    echo "$s rc=$?" >> gpurun_out/${TAG}_stress$v.log
  done
done
for t in memcheck synccheck racecheck; do
  timeout 600 compute-sanitizer --tool $t --kernel-regex kns=plr_ python tools/sanitize_run.py > gpurun_out/${TAG}_sanitize_$t.log 2>&1
  echo "rc=$?" >> gpurun_out/${TAG}_sanitize_$t.log
done
timeout 3000 python -m pytest tests -m gpu -q --timeout 1200 -p no:cacheprovider > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 1200 python tools/float_err.py > gpurun_out/${TAG}_float_err.md 2> gpurun_out/${TAG}_float_err.err
true
