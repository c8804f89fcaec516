for s in order3 tuple3 order2 prefix; do
  timeout 300 python tools/stress.py $s 1060921,1048576,7680,15361,7681 20 >> gpurun_out/r01q_stress.log 2>&1
done
timeout 900 python -m pytest tests -m gpu -x -q -k "prefix or tuple or order" > gpurun_out/r01q_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r01q_pytest.log
TAG=r01q VARS="base x31w4 x31w8 x23w8" SIGS=lp1,lp2,lp3,hp1,hp2,hp3 bash tools/gpu_cmp.sh
timeout 300 python tools/time_sigs.py 1073741824 prefix,tuple2,tuple3,order2,order3 > gpurun_out/r01q_times_int.log 2>&1
