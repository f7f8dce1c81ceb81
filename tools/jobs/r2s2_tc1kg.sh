mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "kgroup" 2>&1 | tail -2
for v in 1 0; do
  HGEMM_TC1_KG=$v python tools/chooser_probe.py > /dev/null 2>&1 || echo "plain failed"
  HGEMM_TC1_KG=$v ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/tc1kg_$v.csv python tools/chooser_probe.py > gpurun_out/tc1kg_order_$v.txt 2>/dev/null
  python tools/launch_cost_join.py gpurun_out/tc1kg_$v.csv gpurun_out/tc1kg_order_$v.txt > gpurun_out/tc1kg_$v.log
done
paste gpurun_out/tc1kg_1.log gpurun_out/tc1kg_0.log | grep -E "auto|tc1/block_n128 |cublas" | awk -F'\t' '{print substr($1,1,86) " || off " substr($2, 76, 12)}'
