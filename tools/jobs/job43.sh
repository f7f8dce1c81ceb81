# skinny: new defaults (G auto with >= 3 stages, stream only for n <= 128) vs G = 1, mean of 40 launches
mkdir -p gpurun_out
for rep in 1 2; do for g in 1 -1; do
  echo "G $g"
  HGEMM_STREAM_G=$g timeout 300 python tools/stream_sweep.py --skinny --mean
done; done > gpurun_out/j43_g.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -q -m gpu -x 2>&1 | tail -3 > gpurun_out/j43_tests.log
cat gpurun_out/j43_*.log
