# time every variant library in $VARS (space separated suffixes) on the given signatures
set -x
mkdir -p gpurun_out
for v in $VARS; do
  [ "$v" = "base" ] && v=""
  echo "== variant '$v'" >> gpurun_out/variants2.log
  PLR_LIB=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200$v.so timeout 300 python tools/time_sigs.py $((1<<30)) ${SIGS:-prefix,tuple2,tuple3,order3} >> gpurun_out/variants2.log 2>&1
done
