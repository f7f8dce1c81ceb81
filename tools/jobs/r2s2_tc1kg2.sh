mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
python tools/chooser_probe.py > /dev/null 2>&1 || echo "plain failed"
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/tc1kg2.csv python tools/chooser_probe.py > gpurun_out/tc1kg2_order.txt 2>/dev/null
python tools/launch_cost_join.py gpurun_out/tc1kg2.csv gpurun_out/tc1kg2_order.txt | grep -E "auto|cublas"
timeout 3300 python tools/paper_sweep.py --square-step 256 --rect-step 256 --out gpurun_out/s3_paper_sweep.jsonl --md gpurun_out/s3_paper_sweep.md > gpurun_out/s3_paper_sweep.log 2>&1
grep -A10 "^| shape | points" gpurun_out/s3_paper_sweep.md | head -11
