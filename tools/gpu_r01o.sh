timeout 900 python -m pytest tests -m gpu -x -q -k "prefix or tuple or order" > gpurun_out/r01o_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r01o_pytest.log
TAG=r01o VARS="base blk0" SIGS=prefix,tuple2,tuple3,order2,order3 bash tools/gpu_cmp.sh
bash tools/ncu_profile.sh r01o "order3"
