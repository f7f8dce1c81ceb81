mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -k "stream" 2>&1 | tail -3 > gpurun_out/j49_tests.log
cat gpurun_out/j49_tests.log
