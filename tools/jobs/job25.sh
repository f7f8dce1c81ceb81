mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/j25_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/j25_smoke.log
timeout 3000 python -m pytest tests -m gpu -q -x 2>&1 | tail -4 > gpurun_out/j25_gpu_tests.log
cat gpurun_out/j25_*.log
