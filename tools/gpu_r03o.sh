# round-2 batch o: re-read kernel storer with STQ bulk stores in flight
# (stq2, stq3) and X=27 with 6 phase-B stages (x27, STQ=2), at 2^30; parity of stq2
set -x
TAG=${TAG:-r03o}
mkdir -p gpurun_out
L=paper_conf_asplos_malekib18_b200
TAG=${TAG} VARS="base stq2 stq3 x27 base" SIGS=tuple2,tuple3,order2,order3 bash tools/gpu_cmp.sh
PLR_LIB=$L/libplr_b200_stq2.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x --timeout 300 -p no:cacheprovider \
    -k "tuple or order" > gpurun_out/${TAG}_pytest_stq2.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_stq2.log
true
