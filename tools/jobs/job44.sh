# swapped streaming for the LSTM gates with 64-row Ak boxes at every chunk width + G sweep
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "stream_kernel or stream_swapped" 2>&1 | tail -3 > gpurun_out/j44_tests.log
for g in 1 2 4 8; do
  echo "G $g"
  HGEMM_STREAM_G=$g timeout 300 python tools/stream_sweep.py --mean
done > gpurun_out/j44_g.log 2>&1
cat gpurun_out/j44_*.log
