mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "stream_k or kgroup or half or ragged or integer" > gpurun_out/s2_kgsk_tests.log 2>&1; tail -2 gpurun_out/s2_kgsk_tests.log
for v in 1 0; do
  HGEMM_TC_KG_SK=$v python tools/ncu_shapes.py > /dev/null 2>&1 || echo "plain $v failed"
  HGEMM_TC_KG_SK=$v ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s2_kgsk_$v.csv \
    python tools/ncu_shapes.py > gpurun_out/s2_kgsk_${v}_order.txt 2> /dev/null
  python tools/launch_cost_join.py gpurun_out/s2_kgsk_$v.csv gpurun_out/s2_kgsk_${v}_order.txt > gpurun_out/s2_kgsk_$v.log 2>&1
done
paste gpurun_out/s2_kgsk_1.log gpurun_out/s2_kgsk_0.log | awk -F'\t' '{print substr($1,1,92) " || off " substr($2, 76, 12)}'
