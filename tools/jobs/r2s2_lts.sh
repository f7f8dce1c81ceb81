mkdir -p gpurun_out
python tools/lts_probe.py > /dev/null 2>&1 || echo "plain failed"
ncu --metrics gpu__time_duration.sum,sm__cycles_active.max,gpc__cycles_elapsed.max,lts__t_sectors_srcunit_tex_op_read.sum --clock-control none --csv --log-file gpurun_out/lts_probe.csv python tools/lts_probe.py > gpurun_out/lts_probe_order.txt 2>/dev/null
python tools/launch_cost_join.py gpurun_out/lts_probe.csv gpurun_out/lts_probe_order.txt
