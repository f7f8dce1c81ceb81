set -x
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_acc16.py -q 2>&1 | tail -30 > gpurun_out/j2_acc16.log
timeout 1500 python -m pytest tests -m gpu -q 2>&1 | tail -30 > gpurun_out/j2_gpu_tests.log
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_cases.py > gpurun_out/j2_$tool.log 2>&1
done
for f in gpurun_out/j2_*.log; do echo "== $f"; tail -n 4 $f; done
