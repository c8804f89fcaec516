# round-2 batch h: TMEM-parked DECAY kernel geometries at 1 CTA/SM (lp3, hp3) + parity of each
set -x
TAG=${TAG:-r03h}
mkdir -p gpurun_out
L=paper_conf_asplos_malekib18_b200
for v in dtA dtB dtC dtD; do
  PLR_LIB=$L/libplr_b200_$v.so timeout 120 python tools/time_sigs.py $((1<<30)) lp3,hp3 > gpurun_out/${TAG}_times_$v.log 2>&1
done
for v in dtA dtB dtC dtD; do
  PLR_LIB=$L/libplr_b200_$v.so timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "(hp3 or lp3) and (sizes or structured or full_size)" --timeout 300 -p no:cacheprovider > gpurun_out/${TAG}_pytest_$v.log 2>&1
done
true
