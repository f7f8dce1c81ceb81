mkdir -p gpurun_out
python tools/sanitize_cases.py > gpurun_out/s2_sanitize_plain.log 2>&1 && \
timeout 1500 compute-sanitizer --tool synccheck python tools/sanitize_cases.py > gpurun_out/s2_synccheck.log 2>&1
tail -3 gpurun_out/s2_sanitize_plain.log; tail -4 gpurun_out/s2_synccheck.log
