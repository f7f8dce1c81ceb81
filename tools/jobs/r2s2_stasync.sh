mkdir -p gpurun_out
HGEMM_EXP=64 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "splitk" > gpurun_out/s2_sa_parity.log 2>&1; tail -2 gpurun_out/s2_sa_parity.log
for v in bulk direct; do
  if [ $v = direct ]; then export HGEMM_EXP=64; else unset HGEMM_EXP; fi
  python tools/launch_cost_ncu.py --gemm-only > /dev/null 2>&1 || echo "plain run $v failed"
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s2_sa_$v.csv \
    python tools/launch_cost_ncu.py --gemm-only > gpurun_out/s2_sa_${v}_order.txt 2> gpurun_out/s2_sa_$v.err
  python tools/launch_cost_join.py gpurun_out/s2_sa_$v.csv gpurun_out/s2_sa_${v}_order.txt > gpurun_out/s2_sa_$v.log 2>&1
  HGEMM_LIB=ab_libs/trace.so python tools/trace_sk.py 64 4096 2048 > gpurun_out/s2_sa_trace_$v.log 2>&1
  HGEMM_LIB=ab_libs/trace.so python tools/trace_sk.py 256 4096 2048 >> gpurun_out/s2_sa_trace_$v.log 2>&1
done
unset HGEMM_EXP
paste gpurun_out/s2_sa_bulk.log gpurun_out/s2_sa_direct.log | head -6 | awk -F'\t' '{print $1 " || direct " substr($2, 76, 12)}'
for v in bulk direct; do echo "== $v"; grep -E "^(start|setup|data0|mma_issued|tfull|sent|epi_done|end) " gpurun_out/s2_sa_trace_$v.log; done
