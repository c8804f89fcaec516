set -x
mkdir -p gpurun_out
timeout 300 python tools/lookback_stats.py $((1<<30)) prefix,tuple2,tuple3,order2,order3 > gpurun_out/lbstats2.log 2>&1
bash tools/ncu_profile.sh r01d "tuple2 tuple3"
