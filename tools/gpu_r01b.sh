set -x
mkdir -p gpurun_out
for v in "" _nl3 _nl4 _nl4s4; do
  echo "== variant '$v'" >> gpurun_out/variants.log
  PLR_LIB=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200$v.so timeout 300 python tools/time_sigs.py $((1<<30)) prefix,tuple2,tuple3,order2,order3,lp3,hp3 >> gpurun_out/variants.log 2>&1
done
bash tools/ncu_profile.sh r01c "tuple2 prefix hp3"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 1000 --csv --log-file gpurun_out/launches_r01.csv python bench.py --steps 3 --warmup 3 > gpurun_out/bench_ncu.log 2>&1
