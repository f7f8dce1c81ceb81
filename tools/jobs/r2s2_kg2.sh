mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_large.py -x -q -k "baseline_configs" > gpurun_out/s2_kg2_tests.log 2>&1; tail -3 gpurun_out/s2_kg2_tests.log
for v in new base; do
  if [ $v = base ]; then export HGEMM_LIB=ab_libs/base3.so; else unset HGEMM_LIB; fi
  python tools/launch_cost_ncu.py --gemm-only > /dev/null 2>&1 || echo "plain run $v failed"
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s2_kg_$v.csv \
    python tools/launch_cost_ncu.py --gemm-only > gpurun_out/s2_kg_${v}_order.txt 2> /dev/null
  python tools/launch_cost_join.py gpurun_out/s2_kg_$v.csv gpurun_out/s2_kg_${v}_order.txt > gpurun_out/s2_kg_$v.log 2>&1
done
unset HGEMM_LIB
paste gpurun_out/s2_kg_new.log gpurun_out/s2_kg_base.log | awk -F'\t' '{print substr($1,1,92) " || base " substr($2, 76, 12)}'
