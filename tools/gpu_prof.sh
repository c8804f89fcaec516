set -x
bash tools/ncu_profile.sh r01 "tuple2 prefix"
timeout 1200 python -m pytest tests -m gpu -x -q -k "full_size" > gpurun_out/pytest_full.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_full.log
