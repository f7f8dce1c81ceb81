# round-2 final measurement package
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/f_smoke.log 2>&1; echo "rc=$?" >> gpurun_out/f_smoke.log
timeout 3000 python -m pytest tests -m gpu -q 2>&1 | tail -4 > gpurun_out/f_gpu_tests.log
timeout 1200 python bench.py > gpurun_out/f_bench_default.log 2>&1
timeout 900 python bench.py --impl reference > gpurun_out/f_bench_reference.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/f_launches.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:hgemm_tc -s 3 -c 1 -o gpurun_out/f_ours_8192 \
  python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e --no-cublas --no-side --no-strong > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none -k regex:hgemm_tc -s 3 -c 1 -o gpurun_out/f_ours_32768 \
  python bench.py --workload cfg5_sharded_32768 --steps 1 --warmup 3 --no-cpu --no-e2e --no-cublas --no-side --no-strong > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none -k regex:splitk -s 3 -c 1 -o gpurun_out/f_ours_lstm64 \
  python bench.py --workload cfg3_lstm_b64 --steps 2 --warmup 3 --no-cpu --no-e2e --no-cublas --no-side --no-strong > /dev/null 2>&1
ls gpurun_out/f_*; cat gpurun_out/f_smoke.log gpurun_out/f_gpu_tests.log
