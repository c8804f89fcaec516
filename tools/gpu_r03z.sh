# round-2 batch z: re-read kernel phase A as two independent chains (split) vs base
set -x
TAG=${TAG:-r03z}
mkdir -p gpurun_out
L=paper_conf_asplos_malekib18_b200
TAG=${TAG} VARS="base split base split" SIGS=tuple2,tuple3,order2,order3 bash tools/gpu_cmp.sh
PLR_LIB=$L/libplr_b200_split.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_wider.py -m gpu -q -x --timeout 300 -p no:cacheprovider \
    -k "tuple or order or fir or full_size" > gpurun_out/${TAG}_pytest_split.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_split.log
true
