mkdir -p gpurun_out
for i in 1 2; do
python tools/mid_shapes.py staged6 > gpurun_out/s2_direct_$i.log 2>&1
HGEMM_LIB=ab_libs/direct.so HGEMM_EPI_DIRECT=1 python tools/mid_shapes.py direct7 --no-cublas >> gpurun_out/s2_direct_$i.log 2>&1
done
cat gpurun_out/s2_direct_*.log
