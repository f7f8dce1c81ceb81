# streaming-pattern study: 3-D TMA boxes (G k-blocks per load) and plain LDG; L2 promotion on the skinny kernel
mkdir -p gpurun_out
timeout 300 python tools/stream_study.py --3d > gpurun_out/j40_stream3d.log 2>&1
for pr in 0 128 256; do
  echo "L2_PROMO $pr"
  HGEMM_L2_PROMO=$pr timeout 300 python tools/stream_sweep.py --skinny
done > gpurun_out/j40_promo.log 2>&1
cat gpurun_out/j40_*.log
