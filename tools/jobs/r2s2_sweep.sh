mkdir -p gpurun_out
timeout 3300 python tools/paper_sweep.py --square-step 256 --rect-step 256 --out gpurun_out/s2_paper_sweep.jsonl \
  --md gpurun_out/s2_paper_sweep.md > gpurun_out/s2_paper_sweep.log 2>&1
tail -n 3 gpurun_out/s2_paper_sweep.log; head -30 gpurun_out/s2_paper_sweep.md
