# round-2 measurement package: full GPU suite, default bench line, reference arm, ncu launch list,
# ncu --set full of the headline kernel (ours and cuBLAS)
mkdir -p gpurun_out
timeout 3000 python -m pytest tests -m gpu -q -x 2>&1 | tail -4 > gpurun_out/j20_gpu_tests.log
timeout 1200 python bench.py > gpurun_out/j20_bench_default.log 2>&1
timeout 900 python bench.py --impl reference > gpurun_out/j20_bench_reference.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/j20_launches.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e > gpurun_out/j20_launches_bench.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:hgemm_tc -s 3 -c 1 -o gpurun_out/j20_ours_8192 \
  python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e --no-cublas --no-side --no-strong > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none -k regex:nvjet -s 2 -c 1 -o gpurun_out/j20_cublas_8192 \
  python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e --no-side --no-strong > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none -k regex:hgemm_tc -s 3 -c 1 -o gpurun_out/j20_ours_32768 \
  python bench.py --workload cfg5_sharded_32768 --steps 1 --warmup 3 --no-cpu --no-e2e --no-cublas --no-side --no-strong > /dev/null 2>&1
ls -la gpurun_out/j20*
cat gpurun_out/j20_gpu_tests.log; tail -c 600 gpurun_out/j20_bench_default.log
