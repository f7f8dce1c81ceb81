mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_large.py -q -x 2>&1 | tail -2
python tools/chooser_probe.py > /dev/null 2>&1 || echo "plain failed"
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/chooser2.csv python tools/chooser_probe.py > gpurun_out/chooser2_order.txt 2>/dev/null
python tools/launch_cost_join.py gpurun_out/chooser2.csv gpurun_out/chooser2_order.txt | grep "auto"
