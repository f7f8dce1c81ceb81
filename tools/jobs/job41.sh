# streaming kernel: k-blocks per stage G (3-D Bk map), same box A/B
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "stream_kernel or stream_swapped" 2>&1 | tail -3 > gpurun_out/j41_tests.log
HGEMM_STREAM_G=4 timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "stream_kernel or stream_swapped" 2>&1 | tail -3 >> gpurun_out/j41_tests.log
for rep in 1 2; do for g in 1 2 4; do
  echo "G $g"
  HGEMM_STREAM_G=$g timeout 300 python tools/stream_sweep.py --skinny
done; done > gpurun_out/j41_g.log 2>&1
for g in 1 2 4 8; do
  echo "G $g (all shapes incl. swapped LSTM)"
  HGEMM_STREAM_G=$g timeout 300 python tools/stream_sweep.py
done >> gpurun_out/j41_g.log 2>&1
cat gpurun_out/j41_*.log
