# one build->measure iteration on the GPU box.
# usage: TAG=r01x [TESTK="lp or hp"] [TSIGS=a,b] [PROF="hp3 lp3"] bash tools/gpu_iter.sh
set -x
TAG=${TAG:-iter}
mkdir -p gpurun_out
if [ -n "$TESTK" ]; then
  timeout 900 python -m pytest tests -m gpu -x -q -k "$TESTK" > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest.log
fi
timeout 300 python tools/time_sigs.py ${N:-1073741824} $TSIGS > gpurun_out/${TAG}_times.log 2>&1
[ -n "$PROF" ] && bash tools/ncu_profile.sh ${TAG} "$PROF"
true
