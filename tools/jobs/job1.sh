set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv
timeout 600 python -m pytest tests/test_gpu_acc16.py -x -q 2>&1 | tail -30 > gpurun_out/j1_acc16.log
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -30 > gpurun_out/j1_gpu_tests.log
timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu > gpurun_out/j1_bench.log 2>&1
timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python tools/sanitize_cases.py > gpurun_out/j1_memcheck.log 2>&1
tail -3 gpurun_out/j1_*.log
