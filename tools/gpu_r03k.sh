# round-2 batch k: TMEM-parked DECAY geometries around X=27 (fp64) and for the fp32 rows
set -x
TAG=${TAG:-r03k}
mkdir -p gpurun_out
L=paper_conf_asplos_malekib18_b200
for v in "" dtI dtJ dtK; do
  lib=$L/libplr_b200${v:+_$v}.so
  PLR_LIB=$lib timeout 120 python tools/time_sigs.py $((1<<30)) lp3,hp3 > gpurun_out/${TAG}_times64_${v:-main}.log 2>&1
done
for v in "" dt32b; do
  lib=$L/libplr_b200${v:+_$v}.so
  PLR_LIB=$lib timeout 120 python tools/time_sigs.py $((1<<30)) lp1,lp2,hp1,hp2 > gpurun_out/${TAG}_times32_${v:-main}.log 2>&1
done
PLR_LIB=$L/libplr_b200_dt32b.so timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "(lp1 or hp2) and (sizes or structured)" --timeout 300 -p no:cacheprovider > gpurun_out/${TAG}_pytest_dt32b.log 2>&1
true
