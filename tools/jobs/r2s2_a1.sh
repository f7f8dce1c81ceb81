mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/s2_a1_parity.log 2>&1; tail -2 gpurun_out/s2_a1_parity.log
for v in new base; do
  if [ $v = base ]; then export HGEMM_LIB=ab_libs/base.so; else unset HGEMM_LIB; fi
  python tools/launch_cost_ncu.py --gemm-only > /dev/null 2>&1 || echo "plain run $v failed"
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s2_a1_$v.csv \
    python tools/launch_cost_ncu.py --gemm-only > gpurun_out/s2_a1_${v}_order.txt 2> gpurun_out/s2_a1_$v.err
  python tools/launch_cost_join.py gpurun_out/s2_a1_$v.csv gpurun_out/s2_a1_${v}_order.txt > gpurun_out/s2_a1_$v.log 2>&1
done
unset HGEMM_LIB
export HGEMM_LIB=ab_libs/trace.so
for s in "256 256 256" "4096 1024 4096 --beta 1"; do
  python tools/trace_cta2.py $s >> gpurun_out/s2_a1_trace.log 2>&1
done
paste gpurun_out/s2_a1_new.log gpurun_out/s2_a1_base.log | awk -F'\t' '{print $1 " || base " substr($2, 76, 12)}'
cat gpurun_out/s2_a1_trace.log
