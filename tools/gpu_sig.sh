set -x
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "not full_size" > gpurun_out/pytest_sig.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_sig.log
rm -f gpurun_out/variants3.log
echo "== base" >> gpurun_out/variants3.log
timeout 300 python tools/time_sigs.py $((1<<30)) prefix,tuple2,tuple3,order2,order3 >> gpurun_out/variants3.log 2>&1
echo "== base PLR_NO_CONSTSIG" >> gpurun_out/variants3.log
PLR_NO_CONSTSIG=1 timeout 300 python tools/time_sigs.py $((1<<30)) prefix,tuple2,tuple3,order2,order3 >> gpurun_out/variants3.log 2>&1
echo "== nl3" >> gpurun_out/variants3.log
PLR_LIB=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200_nl3.so timeout 300 python tools/time_sigs.py $((1<<30)) prefix,tuple2,tuple3,order2,order3 >> gpurun_out/variants3.log 2>&1
