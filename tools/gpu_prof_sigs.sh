# ncu full captures of chosen signatures + the size sweep.  Usage: TAG=r01k SIGS="hp3 lp3" [SWEEP=1] bash tools/gpu_prof_sigs.sh
set -x
TAG=${TAG:-r01k}
mkdir -p gpurun_out
[ -n "$SWEEP" ] && timeout 900 python tools/sweep.py > gpurun_out/${TAG}_sweep.jsonl 2> gpurun_out/${TAG}_sweep.err
bash tools/ncu_profile.sh ${TAG} "${SIGS:-hp3 lp3 order3}"
