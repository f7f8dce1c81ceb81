mkdir -p gpurun_out
export HGEMM_LIB=ab_libs/trace.so
for s in "64 4096 2048" "256 4096 2048"; do python tools/trace_sk.py $s; python tools/trace_sk.py $s --warm; done > gpurun_out/s2_trace3.log 2>&1
grep -v "^ *[0-9]" gpurun_out/s2_trace3.log
