mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke(); print('SMOKE OK')" > gpurun_out/s2_smoke.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/s2_gpu_tests.log 2>&1
timeout 900 python bench.py > gpurun_out/s2_bench_default.log 2>&1
tail -2 gpurun_out/s2_gpu_tests.log; tail -1 gpurun_out/s2_bench_default.log | cut -c1-400
