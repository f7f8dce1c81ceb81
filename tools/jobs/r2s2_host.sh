mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "hgemm_host" > gpurun_out/s2_host_tests.log 2>&1; tail -2 gpurun_out/s2_host_tests.log
for rep in 1 2; do
for v in new base; do
  if [ $v = base ]; then export HGEMM_LIB=ab_libs/base_host.so; else unset HGEMM_LIB; fi
  python bench.py --steps 10 --warmup 3 --no-cpu --no-cublas --no-side --no-strong 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', 'e2e', round(d['e2e']['value'],1), d['e2e']['ms_per_step'])"
done; done
