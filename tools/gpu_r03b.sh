# round-2 batch b: new kernels (small-n, seeded DECAY, reduce-only, cascade, NCCL leg, reverse, Scan comparator)
set -x
TAG=${TAG:-r03b}
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${TAG}_smoke.log
PLR_SMALL_MAX=0 timeout 200 python tools/stress.py prefix 1183745,7936005,4195081,16777216 200 > gpurun_out/${TAG}_stress.log 2>&1; echo "prefix rc=$?" >> gpurun_out/${TAG}_stress.log
[ -f paper_conf_asplos_malekib18_b200/libplr_b200_hangA.so ] && PLR_SMALL_MAX=0 PLR_LIB=paper_conf_asplos_malekib18_b200/libplr_b200_hangA.so timeout 200 python tools/stress.py prefix 1183745,7936005,4195081,16777216 200 > gpurun_out/${TAG}_stress_hangA.log 2>&1; echo "prefix rc=$?" >> gpurun_out/${TAG}_stress_hangA.log
timeout 600 python tools/time_sigs.py $((1<<30)) > gpurun_out/${TAG}_times.log 2>&1
timeout 300 python tools/time_reduce.py > gpurun_out/${TAG}_reduce.log 2>&1
timeout 600 python tools/sweep.py prefix,tuple2,order3,lp1,hp3 10 22 > gpurun_out/${TAG}_sweep_auto.jsonl 2> gpurun_out/${TAG}_sweep_auto.err
timeout 1500 python -m pytest tests/test_gpu_cascade.py tests/test_gpu_nccl.py tests/test_gpu_bidir.py tests/test_gpu_scan_comparator.py tests/test_gpu_parity.py -q -rs --timeout 600 -p no:cacheprovider \
   -k "small_n or reduce_kernel or decay_bitwise or parity_sizes or structured or cascade or nccl or reverse or bidirectional or comparator" > gpurun_out/${TAG}_pytest_new.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_pytest_new.log
true
