# round-2 batch 04a: REV instantiations of the persistent kernels (anticausal pass beyond small_max):
# full GPU suite, forward and reverse timings at 2^30, forward-backward timings
set -x
TAG=${TAG:-r04a}
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q -x --timeout 900 -p no:cacheprovider > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 400 python tools/time_sigs.py $((1<<30)) > gpurun_out/${TAG}_times.log 2>&1
timeout 400 python tools/time_sigs.py $((1<<30)) "" reverse > gpurun_out/${TAG}_times_reverse.log 2>&1
timeout 400 python tools/time_sigs.py $((1<<30)) "" bidir > gpurun_out/${TAG}_times_bidir.log 2>&1
true
