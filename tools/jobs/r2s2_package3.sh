# round-2 (last session) measurement package: full GPU suite + smoke, default bench line, reference arm,
# ncu launch list of the bench, ncu --set full of the headline (ours, cuBLAS) and of LSTM b64 / BERT-FFN2
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -3 > gpurun_out/r_gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r_smoke.log 2>&1
timeout 1200 python bench.py > gpurun_out/r_bench_default.log 2>&1
timeout 900 python bench.py --impl reference > gpurun_out/r_bench_reference.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r_launches.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e > gpurun_out/r_launches_bench.log 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:hgemm_tc -s 3 -c 1 -o gpurun_out/r_ours_8192 \
  python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e --no-cublas --no-side --no-strong > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none -k regex:nvjet -s 2 -c 1 -o gpurun_out/r_cublas_8192 \
  python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e --no-side --no-strong > /dev/null 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:hgemm -s 2 -c 1 -o gpurun_out/r_ours_lstm64 \
  python tools/run_workload.py cfg3_lstm_b64 3 --no-cublas > /dev/null 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:hgemm -s 2 -c 1 -o gpurun_out/r_ours_ffn2 \
  python tools/run_workload.py cfg3_bert_ffn2_4096 3 --no-cublas > /dev/null 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:hgemm -s 2 -c 1 -o gpurun_out/r_ours_cfg1 \
  python tools/run_workload.py cfg1_256_NN_f32 3 --no-cublas > /dev/null 2>&1
ls -la gpurun_out/r_*
cat gpurun_out/r_gpu_tests.log; tail -1 gpurun_out/r_smoke.log; tail -c 400 gpurun_out/r_bench_default.log
