timeout 900 python -m pytest tests -m gpu -x -q -k "order or prefix or tuple or smoke or worked or closed or wider or unit" > gpurun_out/r02a_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r02a_pytest.log
for s in order3 order2; do timeout 200 python tools/stress.py $s 1060921,33554432,7937,40000000 10 >> gpurun_out/r02a_stress.log 2>&1; done
timeout 300 python tools/time_sigs.py 1073741824 prefix,tuple2,tuple3,order2,order3 > gpurun_out/r02a_times.log 2>&1
