mkdir -p gpurun_out
timeout 600 python tools/code_warm.py > gpurun_out/j45_code_warm.log 2>&1
cat gpurun_out/j45_code_warm.log
