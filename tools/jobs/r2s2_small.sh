mkdir -p gpurun_out
timeout 600 python tools/small_configs.py > gpurun_out/s2_small.log 2>&1
cat gpurun_out/s2_small.log
