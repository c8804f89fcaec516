# round-2 batch y: anticausal pass and forward-backward filtering at 2^30
set -x
TAG=${TAG:-r03y}
mkdir -p gpurun_out
timeout 400 python tools/time_sigs.py $((1<<30)) "" reverse > gpurun_out/${TAG}_times_reverse.log 2>&1
timeout 300 python tools/time_sigs.py $((1<<30)) lp2,hp3,prefix,order2 bidir > gpurun_out/${TAG}_times_bidir.log 2>&1
true
