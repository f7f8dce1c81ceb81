# skinny: G=1 vs auto (G=2), mean of 40 event-timed launches; tc2 flexible-width arm at n=256
mkdir -p gpurun_out
for rep in 1 2; do for g in 1 -1; do
  echo "G $g"
  HGEMM_STREAM_G=$g timeout 300 python tools/stream_sweep.py --skinny --mean
done; done > gpurun_out/j42_g.log 2>&1
cat gpurun_out/j42_*.log
