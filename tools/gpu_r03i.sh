# round-2 batch i: more TMEM-parked DECAY geometries, then the full suite on the new default
set -x
TAG=${TAG:-r03i}
mkdir -p gpurun_out
L=paper_conf_asplos_malekib18_b200
for v in "" dtE dtF dtG dtH; do
  lib=$L/libplr_b200${v:+_$v}.so
  [ -f $lib ] && PLR_LIB=$lib timeout 120 python tools/time_sigs.py $((1<<30)) lp3,hp3 > gpurun_out/${TAG}_times_${v:-main}.log 2>&1
done
timeout 1800 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > gpurun_out/${TAG}_pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_gpu.log
true
