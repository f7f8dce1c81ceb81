mkdir -p gpurun_out
timeout 3000 python -m pytest tests -m gpu -q -x 2>&1 | tail -15 > gpurun_out/j15_gpu_tests.log
cat gpurun_out/j15_gpu_tests.log
