# round-2 batch s: small-n clusters of 4 (main) vs 8 (c8) vs off; k>=2 small-n kernel beyond 2^17
set -x
TAG=${TAG:-r03s}
mkdir -p gpurun_out
L=paper_conf_asplos_malekib18_b200
python -c "
import paper_conf_asplos_malekib18_b200 as plr, workloads
s=workloads.BY_NAME['prefix']; p=plr.Plan(s.a,s.b,s.dtype,n_max=1<<20); print(p.info)" > gpurun_out/${TAG}_info.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x --timeout 300 -p no:cacheprovider -k "cluster or small_n" \
    > gpurun_out/${TAG}_pytest_cluster.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_cluster.log
for c in 1 0; do
  PLR_SMALL_CLUSTER=$c timeout 400 python tools/sweep.py prefix,tuple2,tuple3,order2,order3 10 20 > gpurun_out/${TAG}_sweep_c$c.jsonl 2> gpurun_out/${TAG}_sweep_c$c.err
done
PLR_LIB=$L/libplr_b200_c8.so timeout 400 python tools/sweep.py prefix,tuple2,tuple3,order2,order3 10 20 > gpurun_out/${TAG}_sweep_c8.jsonl 2> gpurun_out/${TAG}_sweep_c8.err
PLR_SMALL_MAX=2097152 timeout 400 python tools/sweep.py tuple2,tuple3,order2,order3 16 20 > gpurun_out/${TAG}_sweep_smallk2.jsonl 2> gpurun_out/${TAG}_sweep_smallk2.err
true
