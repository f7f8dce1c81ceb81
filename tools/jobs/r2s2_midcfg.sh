mkdir -p gpurun_out
timeout 600 python tools/mid_configs.py > gpurun_out/s2_midcfg.log 2>&1
cat gpurun_out/s2_midcfg.log
