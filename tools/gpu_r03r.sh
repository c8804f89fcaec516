# round-2 batch r: is the small-n cluster launch taken? plan info, launch list, parity, sweep on/off
set -x
TAG=${TAG:-r03r}
mkdir -p gpurun_out
PLR_DEBUG=1 python -c "
import paper_conf_asplos_malekib18_b200 as plr, workloads
for nm in ('prefix','tuple2','order3','lp1'):
    s=workloads.BY_NAME[nm]; p=plr.Plan(s.a,s.b,s.dtype,n_max=1<<20); i=p.info
    print(nm, {k:i[k] for k in ('small_clusters','small_ctas_per_sm','small_max','num_sms','kernel_kind')}); p.close()
" > gpurun_out/${TAG}_info.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_small_launches.csv \
    python tools/one_sig.py prefix 1048576 > gpurun_out/${TAG}_ncu_small.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x --timeout 300 -p no:cacheprovider -k "cluster" \
    > gpurun_out/${TAG}_pytest_cluster.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_cluster.log
for c in 1 0; do
  PLR_SMALL_CLUSTER=$c timeout 400 python tools/sweep.py prefix,tuple2,tuple3,order2,order3 10 20 > gpurun_out/${TAG}_sweep_c$c.jsonl 2> gpurun_out/${TAG}_sweep_c$c.err
done
true
