for w in 0 1 4; do
  echo "== waves $w" >> gpurun_out/r02c_waves.log
  PLR_UNIT1_WAVES=$w timeout 300 python tools/sweep.py prefix,tuple2,order3,hp3 16 26 >> gpurun_out/r02c_waves.log 2>&1
done
