# streaming kernel: first-ring issue before the CTA barrier, all stages (default) vs 2
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -k "stream_kernel or stream_swapped" 2>&1 | tail -2 > gpurun_out/j48_tests.log
for rep in 1 2; do for pre in 0 2; do
  echo "PRE $pre"
  HGEMM_STREAM_PRE=$pre timeout 200 python tools/stream_sweep.py --skinny --mean
done; done > gpurun_out/j48_pre.log 2>&1
cat gpurun_out/j48_*.log
