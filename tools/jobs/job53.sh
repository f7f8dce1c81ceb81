mkdir -p gpurun_out
python -m paper_conf_ipps_00020c20_b200.build -DHGEMM_TRACE --out=/tmp/libhgemm_trace.so > /dev/null 2>&1
for s in "64 4096 2048" "256 4096 2048"; do HGEMM_LIB=/tmp/libhgemm_trace.so timeout 120 python tools/trace_sk.py $s; done > gpurun_out/j53_trace_sk.log 2>&1
cat gpurun_out/j53_trace_sk.log | grep -v "^ *[0-9]* *[0-9]"
