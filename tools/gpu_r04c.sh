# round-2 batch 04c: small-n kernel geometry (sw16: W=16 X=15 m=7680; sx31: W=8 X=31 m=7936) vs main (W=8 X=15 m=3840)
set -x
TAG=${TAG:-r04c}
mkdir -p gpurun_out
L=paper_conf_asplos_malekib18_b200
for v in "" sw16 sx31; do
  lib=$L/libplr_b200${v:+_$v}.so
  PLR_LIB=$lib timeout 400 python tools/sweep.py prefix,tuple2,order3,lp1,hp3 12 20 > gpurun_out/${TAG}_sweep_${v:-main}.jsonl 2> gpurun_out/${TAG}_sweep_${v:-main}.err
done
PLR_LIB=$L/libplr_b200_sw16.so timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x --timeout 300 -p no:cacheprovider -k "small_n or cluster" > gpurun_out/${TAG}_pytest_sw16.log 2>&1; echo "pytest rc=$?" >> gpurun_out/${TAG}_pytest_sw16.log
true
