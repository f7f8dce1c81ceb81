mkdir -p gpurun_out
python tools/launch_cost_ncu.py > /dev/null 2>&1 || echo "plain run failed"
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s2_launchcost.csv \
  python tools/launch_cost_ncu.py > gpurun_out/s2_launchcost_order.txt 2> gpurun_out/s2_launchcost.err
python tools/launch_cost_join.py gpurun_out/s2_launchcost.csv gpurun_out/s2_launchcost_order.txt > gpurun_out/s2_launchcost.log 2>&1
cat gpurun_out/s2_launchcost.log
timeout 600 python tools/headline_ab.py --blocks 8 --block 50 --variants ours,cublas,ours:gm=8,ours:gm=32 > gpurun_out/s2_headline_ab.log 2>&1
cat gpurun_out/s2_headline_ab.log | tail -12
