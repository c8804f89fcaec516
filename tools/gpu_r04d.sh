# round-2 batch 04d: medium n -- look-back units of one tile up to PLR_UNIT1_WAVES x grid x G tiles (default 1)
set -x
TAG=${TAG:-r04d}
mkdir -p gpurun_out
for w in 1 2 4 8; do
  PLR_UNIT1_WAVES=$w timeout 400 python tools/sweep.py prefix,tuple2,tuple3,order3 21 25 > gpurun_out/${TAG}_sweep_w$w.jsonl 2> gpurun_out/${TAG}_sweep_w$w.err
  PLR_UNIT1_WAVES=$w timeout 400 python tools/sweep.py prefix,tuple2,tuple3,order3 22 24 > gpurun_out/${TAG}_sweep_e_w$w.jsonl 2> gpurun_out/${TAG}_sweep_e_w$w.err
done
true
