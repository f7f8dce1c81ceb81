mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -3 > gpurun_out/fc_gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/fc_smoke.log 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/fc_bench20.log 2>&1
cat gpurun_out/fc_gpu_tests.log; tail -1 gpurun_out/fc_smoke.log; tail -1 gpurun_out/fc_bench20.log | cut -c1-220
