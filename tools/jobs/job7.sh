# NEXT-3: the paper's full evaluation sweep (square + six rectangular shapes, W = 1024..16384 step 256)
mkdir -p gpurun_out
timeout 3000 python tools/paper_sweep.py --square-step 256 --rect-step 256 --out gpurun_out/j7_paper_sweep.jsonl \
  --md gpurun_out/j7_paper_sweep.md > gpurun_out/j7_paper_sweep.log 2>&1
tail -n 3 gpurun_out/j7_paper_sweep.log; head -12 gpurun_out/j7_paper_sweep.md
