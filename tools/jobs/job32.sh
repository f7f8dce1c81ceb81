mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "hgemm_host" 2>&1 | tail -3 > gpurun_out/j32_tests.log
for r in 1 2 3; do timeout 600 python bench.py --steps 20 --no-cpu --no-side --no-strong --no-cublas 2>/dev/null | python -c "import json,sys; d=json.loads([l for l in sys.stdin if l.startswith('{')][-1]); print('e2e', d['e2e']['value'], d['e2e']['ms_per_step'])"; done >> gpurun_out/j32_tests.log
cat gpurun_out/j32_tests.log
