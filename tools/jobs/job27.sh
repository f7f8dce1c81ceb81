# direct-store epilogue (7 ring stages) for the 256-wide CTA-pair kernel: parity + timing
mkdir -p gpurun_out
HGEMM_EPI_DIRECT=1 timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "tc2-256 or stream_k or half or flexible" 2>&1 | tail -3 > gpurun_out/j27_tests.log
HGEMM_EPI_DIRECT=1 timeout 1200 python -m pytest tests/test_gpu_large.py -q -x -k "baseline_configs" 2>&1 | tail -2 >> gpurun_out/j27_tests.log
for r in 1 2; do
  timeout 300 python tools/mid_variants.py staged
  HGEMM_EPI_DIRECT=1 timeout 300 python tools/mid_variants.py direct
done > gpurun_out/j27_mid.log 2>&1
cat gpurun_out/j27_*.log
