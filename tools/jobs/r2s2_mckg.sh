mkdir -p gpurun_out
export HGEMM_LIB=ab_libs/mc.so
HGEMM_MC=2 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "kgroup or random_ragged or integer_bit_exact or alpha_beta" > gpurun_out/s2_mckg_tests.log 2>&1; tail -3 gpurun_out/s2_mckg_tests.log
for v in 2 1; do
  HGEMM_MC=$v python tools/ncu_shapes.py > /dev/null 2>&1 || echo "plain $v failed"
  HGEMM_MC=$v ncu --metrics gpu__time_duration.sum,launch__cluster_dim_x --clock-control none --csv --log-file gpurun_out/s2_mckg_$v.csv \
    python tools/ncu_shapes.py > gpurun_out/s2_mckg_${v}_order.txt 2> /dev/null
  python tools/launch_cost_join.py gpurun_out/s2_mckg_$v.csv gpurun_out/s2_mckg_${v}_order.txt > gpurun_out/s2_mckg_$v.log 2>&1
done
paste gpurun_out/s2_mckg_2.log gpurun_out/s2_mckg_1.log | awk -F'\t' '{print substr($1,1,92) " || mc1 " substr($2, 76, 12)}'
