# decoupled Ak/Bk rings in the streaming kernel: parity + A/B
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "stream_kernel or stream_swapped" 2>&1 | tail -3 > gpurun_out/j39_tests.log
for a in 0 2 6; do
  echo "ASTAGES $a"
  HGEMM_STREAM_ASTAGES=$a timeout 300 python tools/stream_sweep.py --skinny
done > gpurun_out/j39_skinny.log 2>&1
timeout 300 python tools/stream_sweep.py >> gpurun_out/j39_skinny.log 2>&1
cat gpurun_out/j39_*.log
