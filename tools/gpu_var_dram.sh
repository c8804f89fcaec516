# time variants + dram bytes of one launch per variant and signature
# usage: TAG=x VARS="base p1" SIGS="tuple2 tuple3" bash tools/gpu_var_dram.sh
mkdir -p gpurun_out
out=gpurun_out/${TAG}_vardram.log; rm -f $out
for v in $VARS; do
  lib=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200.so
  [ "$v" != "base" ] && lib=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200_$v.so
  echo "== variant $v" >> $out
  PLR_LIB=$lib timeout 200 python tools/time_sigs.py 1073741824 $(echo $SIGS | tr ' ' ',') >> $out 2>&1
  for s in $SIGS; do
    PLR_LIB=$lib timeout 200 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum -k regex:plr_scan -s 2 -c 1 python tools/one_sig.py $s 2>&1 | grep -E "dram__|gpu__time" | sed "s/^/$s /" >> $out
  done
done
