mkdir -p gpurun_out
python tools/chooser_probe.py > /dev/null 2>&1 || echo "plain failed"
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/chooser.csv python tools/chooser_probe.py > gpurun_out/chooser_order.txt 2>/dev/null
python tools/launch_cost_join.py gpurun_out/chooser.csv gpurun_out/chooser_order.txt
