mkdir -p gpurun_out
for wl in sq256_NN_f32 sq384 sq512 sq512_NN_f32 sq768 sq1024 sq1280; do
  python tools/ncu_configs.py $wl > /dev/null 2>&1 || echo "plain $wl failed"
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/cfgncu_$wl.csv \
     python tools/ncu_configs.py $wl > gpurun_out/cfgncu_${wl}_order.txt 2>/dev/null
  python tools/launch_cost_join.py gpurun_out/cfgncu_$wl.csv gpurun_out/cfgncu_${wl}_order.txt
done
