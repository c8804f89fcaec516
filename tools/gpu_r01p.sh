for v in base blk0; do
  lib=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200.so
  [ "$v" != "base" ] && lib=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200_$v.so
  echo "== $v" >> gpurun_out/r01p_stress.log
  for s in order3 tuple3 order2; do
    PLR_LIB=$lib timeout 300 python tools/stress.py $s 1060921,1048576,7680,15361 20 >> gpurun_out/r01p_stress.log 2>&1
  done
done
