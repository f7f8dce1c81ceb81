mkdir -p gpurun_out
python tools/lts_probe.py > /dev/null 2>&1 || echo "plain failed"
for v in 2 1; do
HGEMM_TC_KG=$v ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/lts2_$v.csv python tools/lts_probe.py > gpurun_out/lts2_order_$v.txt 2>/dev/null
echo "== KG=$v"; python tools/launch_cost_join.py gpurun_out/lts2_$v.csv gpurun_out/lts2_order_$v.txt
done
