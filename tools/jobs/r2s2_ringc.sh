mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "beta or alpha or ragged or half or flexible" > gpurun_out/s2_ringc_tests.log 2>&1; tail -2 gpurun_out/s2_ringc_tests.log
for v in new base; do
  if [ $v = base ]; then export HGEMM_LIB=ab_libs/base2.so; else unset HGEMM_LIB; fi
  python tools/launch_cost_ncu.py --gemm-only > /dev/null 2>&1 || echo "plain run $v failed"
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s2_rc_$v.csv \
    python tools/launch_cost_ncu.py --gemm-only > gpurun_out/s2_rc_${v}_order.txt 2> /dev/null
  python tools/launch_cost_join.py gpurun_out/s2_rc_$v.csv gpurun_out/s2_rc_${v}_order.txt > gpurun_out/s2_rc_$v.log 2>&1
done
unset HGEMM_LIB
paste gpurun_out/s2_rc_new.log gpurun_out/s2_rc_base.log | grep ours | awk -F'\t' '{print substr($1,1,90) " || base " substr($2, 76, 12)}'
