mkdir -p gpurun_out
for v in relaxed release; do
  if [ $v = release ]; then export HGEMM_LIB=ab_libs/release.so; else unset HGEMM_LIB; fi
  python tools/launch_cost_ncu.py --gemm-only > /dev/null 2>&1 || echo "plain run $v failed"
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s2_lc_$v.csv \
    python tools/launch_cost_ncu.py --gemm-only > gpurun_out/s2_lc_${v}_order.txt 2> gpurun_out/s2_lc_$v.err
  python tools/launch_cost_join.py gpurun_out/s2_lc_$v.csv gpurun_out/s2_lc_${v}_order.txt > gpurun_out/s2_lc_$v.log 2>&1
done
unset HGEMM_LIB
for v in trace trace_release; do
  echo "== $v" >> gpurun_out/s2_trace_rel.log
  HGEMM_LIB=ab_libs/$v.so python tools/trace_sk.py 64 4096 2048 >> gpurun_out/s2_trace_rel.log 2>&1
done
paste gpurun_out/s2_lc_relaxed.log gpurun_out/s2_lc_release.log | awk -F'\t' '{print $1 " || " substr($2, 76, 12)}'
grep -v "^ *[0-9]" gpurun_out/s2_trace_rel.log
