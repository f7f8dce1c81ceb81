mkdir -p gpurun_out
python -m paper_conf_ipps_00020c20_b200.build -DHGEMM_TRACE --out=/tmp/libhgemm_trace.so > /dev/null 2>&1
for g in 1 4 8; do
  echo "G $g"
  HGEMM_STREAM_G=$g HGEMM_LIB=/tmp/libhgemm_trace.so timeout 120 python tools/trace_stream.py 64 4096 2048 1.0 32
done > gpurun_out/j46_trace_swapped.log 2>&1
cat gpurun_out/j46_trace_swapped.log
