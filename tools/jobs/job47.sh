# streaming kernel: Ak multicast clusters (MC 1/2/4) and pre-barrier issue count; parity under each MC
mkdir -p gpurun_out
for mc in 1 2 4; do
  echo "MC $mc"
  HGEMM_STREAM_MC=$mc timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -k "stream_kernel or stream_swapped" 2>&1 | tail -3
done > gpurun_out/j47_tests.log 2>&1
for mc in 1 2 4; do for pre in 2 16; do
  echo "MC $mc PRE $pre"
  HGEMM_STREAM_MC=$mc HGEMM_STREAM_PRE=$pre timeout 300 python tools/stream_sweep.py --mean
done; done > gpurun_out/j47_sweep.log 2>&1
cat gpurun_out/j47_*.log
