mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "splitk or small_problems" > gpurun_out/s2_hm2_tests.log 2>&1; tail -2 gpurun_out/s2_hm2_tests.log
HGEMM_SK_HM=1 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "splitk_splits or random_ragged or integer or alpha_beta" > gpurun_out/s2_hm2_tests_forced.log 2>&1; tail -2 gpurun_out/s2_hm2_tests_forced.log
for wl in cfg1_256_NN_f32 sq384 sq512 cfg3_lstm_b64; do
  python tools/ncu_configs.py $wl > /dev/null 2>&1 || echo "plain $wl failed"
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/hm2_$wl.csv \
     python tools/ncu_configs.py $wl > gpurun_out/hm2_${wl}_order.txt 2>/dev/null
  python tools/launch_cost_join.py gpurun_out/hm2_$wl.csv gpurun_out/hm2_${wl}_order.txt | grep -E "auto|cublas"
done
