# round-2 batch f: TMEM-parked DECAY kernel A/B (+ fp32 DECAY status sizing A/B vs round 1), full suite, sweep, bench
set -x
TAG=${TAG:-r03f}
mkdir -p gpurun_out
L=paper_conf_asplos_malekib18_b200
for v in "" dt0 dtd2 dtsl3 dt32; do
  lib=$L/libplr_b200${v:+_$v}.so
  [ -f $lib ] && PLR_LIB=$lib timeout 150 python tools/time_sigs.py $((1<<30)) lp1,lp2,hp1,hp2,lp3,hp3 > gpurun_out/${TAG}_times_dec_${v:-main}.log 2>&1
done
[ -d ab_r1 ] && timeout 150 python ab_r1/tools/time_sigs.py $((1<<30)) lp1,lp2,hp1,hp2,lp3,hp3 > gpurun_out/${TAG}_times_dec_r1.log 2>&1
timeout 1800 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
timeout 400 python tools/sweep.py prefix,tuple2,order3,lp1,hp3 10 22 > gpurun_out/${TAG}_sweep_auto.jsonl 2> gpurun_out/${TAG}_sweep_auto.err
timeout 400 python tools/time_sigs.py $((1<<30)) > gpurun_out/${TAG}_times.log 2>&1
true
