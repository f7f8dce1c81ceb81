mkdir -p gpurun_out
for wl in cfg1_256_NN_f32 cfg3_lstm_b64 cfg3_lstm_b256; do
  python tools/ncu_configs.py $wl > /dev/null 2>&1 || echo "plain $wl failed"
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/cfgncu_$wl.csv \
     python tools/ncu_configs.py $wl > gpurun_out/cfgncu_${wl}_order.txt 2>/dev/null
  python tools/launch_cost_join.py gpurun_out/cfgncu_$wl.csv gpurun_out/cfgncu_${wl}_order.txt
done
