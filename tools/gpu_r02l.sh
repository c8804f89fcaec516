# small-n wait experiment: suspend-hint waits (base) vs spin waits (PLR_WAIT_HINT_NS=0)
mkdir -p gpurun_out
for v in base spin; do
  lib=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200.so
  [ "$v" != "base" ] && lib=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200_$v.so
  PLR_LIB=$lib timeout 300 python tools/small_n.py > gpurun_out/r02l_small_n_host_$v.jsonl 2>&1
  PLR_LIB=$lib timeout 300 python tools/time_sigs.py 1073741824 > gpurun_out/r02l_times_$v.txt 2>&1
done
true
