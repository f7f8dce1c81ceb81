mkdir -p gpurun_out
export HGEMM_LIB=ab_libs/trace.so
for pdl in 0 1; do for n in 64 128; do echo "PDL=$pdl"; HGEMM_PDL=$pdl python tools/trace_stream.py 16384 $n 4096; done; done > gpurun_out/s2_trace_stream.log 2>&1
cat gpurun_out/s2_trace_stream.log
