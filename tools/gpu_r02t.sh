# poll sleep 64 ns (base) vs 256 ns: small-n per-call, 2^30 times (twice each)
mkdir -p gpurun_out
for v in base s256 base s256; do
  lib=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200.so
  [ "$v" != "base" ] && lib=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200_$v.so
  PLR_LIB=$lib timeout 200 python tools/time_sigs.py 1073741824 >> gpurun_out/r02t_times_$v.txt 2>&1
done
for v in base s256; do
  lib=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200.so
  [ "$v" != "base" ] && lib=$PWD/paper_conf_asplos_malekib18_b200/libplr_b200_$v.so
  PLR_LIB=$lib timeout 200 python tools/small_n.py > gpurun_out/r02t_small_n_host_$v.jsonl 2>&1
done
true
