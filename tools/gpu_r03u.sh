# round-2 batch u: re-read kernel geometry with more phase-B stages
# (x27s6: X=27 SB=6; x23s7: X=23 SB=7; ns12: X=27 SB=6 NS=12 G=8)
set -x
TAG=${TAG:-r03u}
mkdir -p gpurun_out
TAG=${TAG} VARS="base x27s6 x23s7 ns12 base" SIGS=tuple2,tuple3,order2,order3 bash tools/gpu_cmp.sh
true
