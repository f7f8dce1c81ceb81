mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/s2_gpu_tests_relaxed.log 2>&1
tail -3 gpurun_out/s2_gpu_tests_relaxed.log
export HGEMM_LIB=ab_libs/trace.so
for s in "256 256 256" "1024 1024 1024" "4096 1024 4096 --beta 1" "2048 2048 2048"; do
  python tools/trace_cta2.py $s >> gpurun_out/s2_trace_tc.log 2>&1
done
cat gpurun_out/s2_trace_tc.log
