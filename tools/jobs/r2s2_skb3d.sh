mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_large.py -x -q -k "splitk or lstm or small_problems or baseline" > gpurun_out/s2_skb3d_tests.log 2>&1; tail -2 gpurun_out/s2_skb3d_tests.log
for v in 1 0; do
  HGEMM_SK_B3D=$v python tools/launch_cost_ncu.py --gemm-only > /dev/null 2>&1
  HGEMM_SK_B3D=$v ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s2_skb_$v.csv \
    python tools/launch_cost_ncu.py --gemm-only > gpurun_out/s2_skb_${v}_order.txt 2> /dev/null
  python tools/launch_cost_join.py gpurun_out/s2_skb_$v.csv gpurun_out/s2_skb_${v}_order.txt > gpurun_out/s2_skb_$v.log 2>&1
done
paste gpurun_out/s2_skb_1.log gpurun_out/s2_skb_0.log | grep "ours" | awk -F'\t' '{print substr($1,1,92) " || b3d=0 " substr($2, 76, 12)}'
