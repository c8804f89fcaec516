# round-2 batch w: stress of the small-n cluster launches (compute-sanitizer is closed on this pool)
# 1000 launches per size at tile counts around cluster boundaries, every output vs the oracle
set -x
TAG=${TAG:-r03w}
mkdir -p gpurun_out
S=$(python -c "print(','.join(str(t*3840-d) for t in (2,3,4,5,8,9,64,65,273,283,284) for d in (0,1)))")
for sig in prefix tuple3 order3; do
  timeout 600 python tools/stress.py $sig $S 1000 >> gpurun_out/${TAG}_stress_cluster.log 2>&1; echo "$sig rc=$?" >> gpurun_out/${TAG}_stress_cluster.log
done
true
