mkdir -p gpurun_out
HGEMM_SK_HM=1 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "splitk or small_problems" > gpurun_out/s2_hm_tests.log 2>&1; tail -3 gpurun_out/s2_hm_tests.log
for v in base hm; do
  if [ $v = hm ]; then export HGEMM_SK_HM=1; else unset HGEMM_SK_HM; fi
  for wl in cfg3_lstm_b64 cfg1_256_NN_f32 sq384 sq512; do
    python tools/ncu_configs.py $wl > /dev/null 2>&1 || echo "plain $wl $v failed"
    ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/hm_${v}_$wl.csv \
       python tools/ncu_configs.py $wl > gpurun_out/hm_${v}_${wl}_order.txt 2>/dev/null
    echo "== $v $wl"; python tools/launch_cost_join.py gpurun_out/hm_${v}_$wl.csv gpurun_out/hm_${v}_${wl}_order.txt | grep -E "auto|splitk/64|cublas"
  done
done
