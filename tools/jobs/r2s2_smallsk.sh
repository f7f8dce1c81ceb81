mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "small_problems or splitk or random_ragged" > gpurun_out/s2_smallsk_tests.log 2>&1; tail -2 gpurun_out/s2_smallsk_tests.log
for wl in cfg1_256_NN_f32 sq384 sq512 sq512_NN_f32 sq768 sq1024; do
  python tools/ncu_configs.py $wl > /dev/null 2>&1 || echo "plain $wl failed"
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/cfgncu2_$wl.csv \
     python tools/ncu_configs.py $wl > gpurun_out/cfgncu2_${wl}_order.txt 2>/dev/null
  python tools/launch_cost_join.py gpurun_out/cfgncu2_$wl.csv gpurun_out/cfgncu2_${wl}_order.txt | grep -E "auto|cublas"
done
