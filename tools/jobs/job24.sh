mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "stream" 2>&1 | tail -3 > gpurun_out/j24_tests.log
timeout 600 python tools/stream_sweep.py > gpurun_out/j24_stream_sweep.log 2>&1
cat gpurun_out/j24_*.log
