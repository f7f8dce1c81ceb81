# skinny streaming study: TMA read curve, per-CTA trace, ncu ours vs cuBLAS
mkdir -p gpurun_out
timeout 300 python tools/stream_study.py --quick > gpurun_out/j37_stream_study.log 2>&1
python -m paper_conf_ipps_00020c20_b200.build -DHGEMM_TRACE --out=/tmp/libhgemm_trace.so > /dev/null 2>&1
for s in "16384 64 4096" "16384 256 4096"; do
  HGEMM_LIB=/tmp/libhgemm_trace.so timeout 120 python tools/trace_stream.py $s
done > gpurun_out/j37_trace_stream.log 2>&1
bash tools/ncu_cfg.sh j37 cfg4_skinny_n64 > /dev/null 2>&1
cat gpurun_out/j37_*.log
