# time variants + dram bytes of one tuple2 launch per variant
mkdir -p gpurun_out
rm -f gpurun_out/variants5.log
for v in $VARS; do
  [ "$v" = "base" ] && v=""
  echo "== variant '$v'" >> gpurun_out/variants5.log
  export PLR_LIB=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200$v.so
  timeout 300 python tools/time_sigs.py $((1<<30)) ${SIGS:-prefix,tuple2,tuple3,order3} >> gpurun_out/variants5.log 2>&1
  timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum -k regex:plr_scan -s 2 -c 1 python tools/one_sig.py tuple2 2>&1 | grep -E "dram__|gpu__time" >> gpurun_out/variants5.log
done
unset PLR_LIB
