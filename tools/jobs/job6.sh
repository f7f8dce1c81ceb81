mkdir -p gpurun_out
timeout 300 python tools/stream_sweep.py > gpurun_out/j6_stream_sweep.log 2>&1
python -m paper_conf_ipps_00020c20_b200.build -DHGEMM_TRACE --out=/tmp/libhgemm_trace.so > /dev/null 2>&1
for s in "16384 64 4096" "16384 256 4096" "64 4096 2048 1.0 32" "256 4096 2048 1.0 32"; do
  HGEMM_LIB=/tmp/libhgemm_trace.so timeout 120 python tools/trace_stream.py $s
done > gpurun_out/j6_trace_stream.log 2>&1
cat gpurun_out/j6_*.log
