mkdir -p gpurun_out
timeout 600 ncu --set full --import-source on --clock-control none -k regex:hgemm_tc -s 3 -c 1 -o gpurun_out/j29_ours_ffn2 \
  python bench.py --workload cfg3_bert_ffn2_4096 --steps 2 --warmup 3 --no-cpu --no-e2e --no-cublas --no-side --no-strong > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none -k regex:nvjet -s 2 -c 1 -o gpurun_out/j29_cublas_ffn2 \
  python bench.py --workload cfg3_bert_ffn2_4096 --steps 2 --warmup 3 --no-cpu --no-e2e --no-side --no-strong > /dev/null 2>&1
ls -la gpurun_out/j29*
