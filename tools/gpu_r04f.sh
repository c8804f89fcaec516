# round-2 batch 04f: re-read kernel with more slots / a longer lag (ns11: NS=11 lag 10; ns12: NS=12 lag 11; G=6)
set -x
TAG=${TAG:-r04f}
mkdir -p gpurun_out
TAG=${TAG} VARS="base ns11 ns12 base ns11 ns12" SIGS=tuple2,tuple3,order2,order3 bash tools/gpu_cmp.sh
for v in ns11 ns12; do
  PLR_LIB=paper_conf_asplos_malekib18_b200/libplr_b200_$v.so timeout 400 python tools/sweep.py tuple2,order3 22 26 > gpurun_out/${TAG}_sweep_$v.jsonl 2> gpurun_out/${TAG}_sweep_$v.err
done
timeout 400 python tools/sweep.py tuple2,order3 22 26 > gpurun_out/${TAG}_sweep_base.jsonl 2> gpurun_out/${TAG}_sweep_base.err
true
