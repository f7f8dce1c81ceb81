mkdir -p gpurun_out
timeout 300 python tools/l2_ingest_study.py > gpurun_out/s2_ingest.log 2>&1
cat gpurun_out/s2_ingest.log
