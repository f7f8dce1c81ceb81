mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_large.py -x -q -k "stream or skinny or cfg4" > gpurun_out/s2_a3d_tests.log 2>&1; tail -2 gpurun_out/s2_a3d_tests.log
for v in 1 0; do
  HGEMM_STREAM_A3D=$v python tools/launch_cost_ncu.py --gemm-only > /dev/null 2>&1
  HGEMM_STREAM_A3D=$v ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s2_a3d_$v.csv \
    python tools/launch_cost_ncu.py --gemm-only > gpurun_out/s2_a3d_${v}_order.txt 2> /dev/null
  python tools/launch_cost_join.py gpurun_out/s2_a3d_$v.csv gpurun_out/s2_a3d_${v}_order.txt > gpurun_out/s2_a3d_$v.log 2>&1
done
paste gpurun_out/s2_a3d_1.log gpurun_out/s2_a3d_0.log | grep "16384\|1024x" | awk -F'\t' '{print substr($1,1,92) " || a3d=0 " substr($2, 76, 12)}'
for n in 64 128; do for v in 1 0; do
 echo "== n=$n A3D=$v"; HGEMM_STREAM_A3D=$v HGEMM_LIB=ab_libs/trace.so python tools/trace_stream.py 16384 $n 4096 | grep -E "data0|mma_done|epi_done"
done; done
