mkdir -p gpurun_out
python tools/lts_probe.py --warm > /dev/null 2>&1 || echo "plain failed"
ncu --metrics gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_read.sum --cache-control none --clock-control none --csv --log-file gpurun_out/warm_probe.csv python tools/lts_probe.py --warm > gpurun_out/warm_order.txt 2>/dev/null
echo "== warm (no flush, ncu cache-control none)"; python tools/launch_cost_join.py gpurun_out/warm_probe.csv gpurun_out/warm_order.txt
