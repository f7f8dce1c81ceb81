mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/s2_kg3_tests.log 2>&1; tail -3 gpurun_out/s2_kg3_tests.log
HGEMM_TC_KG=1 python tools/ncu_shapes.py > /dev/null 2>&1
for v in 2 1; do
  HGEMM_TC_KG=$v ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s2_kgt_$v.csv \
    python tools/ncu_shapes.py > gpurun_out/s2_kgt_${v}_order.txt 2> /dev/null
  python tools/launch_cost_join.py gpurun_out/s2_kgt_$v.csv gpurun_out/s2_kgt_${v}_order.txt > gpurun_out/s2_kgt_$v.log 2>&1
done
paste gpurun_out/s2_kgt_2.log gpurun_out/s2_kgt_1.log | awk -F'\t' '{print substr($1,1,92) " || kg1 " substr($2, 76, 12) " " substr($2,1,45)}'
