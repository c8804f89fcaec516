# time every Table-1 signature at 2^30 for several library variants.
# usage: TAG=r01x VARS="base spin" [SIGS=a,b] bash tools/gpu_cmp.sh
mkdir -p gpurun_out
out=gpurun_out/${TAG:-cmp}_cmp.log
rm -f $out
for v in $VARS; do
  lib=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200.so
  [ "$v" != "base" ] && lib=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200_$v.so
  echo "== variant $v" >> $out
  PLR_LIB=$lib timeout 300 python tools/time_sigs.py ${N:-1073741824} $SIGS >> $out 2>&1
done
