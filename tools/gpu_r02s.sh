# stop-aware waits by test_wait + 64 ns sleep: trace, small-n, 2^30 times, all gpu tests, smoke, bench
mkdir -p gpurun_out
PLR_LIB=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200_trace.so timeout 120 python tools/trace_small.py > gpurun_out/r02s_trace.jsonl 2>&1
timeout 200 python tools/small_n.py > gpurun_out/r02s_small_n_host.jsonl 2>&1
timeout 200 python tools/time_sigs.py 1073741824 > gpurun_out/r02s_times.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02s_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/r02s_smoke.log
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/r02s_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r02s_pytest_gpu.log
timeout 600 python bench.py > gpurun_out/r02s_bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/r02s_bench.log
true
