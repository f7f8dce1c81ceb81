mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_allgather.py tests/test_gpu_sharded.py -q -x 2>&1 | tail -3 > gpurun_out/j22_tests.log
HGEMM_WSYNC=0 timeout 600 python -m pytest tests/test_gpu_allgather.py -q -x -k long_k 2>&1 | tail -2 >> gpurun_out/j22_tests.log
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --no-side --no-strong --ag-virtual 8 > gpurun_out/j22_agv.log 2>&1
HGEMM_WSYNC=0 timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --no-side --no-strong --ag-virtual 8 > gpurun_out/j22_agv_nowsync.log 2>&1
cat gpurun_out/j22_tests.log; grep -o '"allgather_fused_virtual": {[^}]*}' gpurun_out/j22_agv*.log
