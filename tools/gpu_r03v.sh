# round-2 batch v: compute-sanitizer on the small-n cluster launches and the persistent kernels
set -x
TAG=${TAG:-r03v}
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool python tools/sanitize_run.py > gpurun_out/${TAG}_sanitize_small_$tool.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_sanitize_small_$tool.log
done
PLR_SMALL_MAX=0 timeout 900 compute-sanitizer --tool memcheck python tools/sanitize_run.py > gpurun_out/${TAG}_sanitize_big_memcheck.log 2>&1; echo "rc=$?" >> gpurun_out/${TAG}_sanitize_big_memcheck.log
true
