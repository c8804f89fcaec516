for v in base v1 v2 v3 v4; do
  lib=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200.so
  [ "$v" != "base" ] && lib=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200_$v.so
  echo "== variant $v" >> gpurun_out/r02d_cmp.log
  PLR_LIB=$lib timeout 60 python tools/time_sigs.py 1073741824 tuple2,tuple3,order2,order3 >> gpurun_out/r02d_cmp.log 2>&1
  echo "rc=$?" >> gpurun_out/r02d_cmp.log
done
