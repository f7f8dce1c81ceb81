set -x
for w in cfg3_bert_ffn1_16384 cfg4_skinny_n64; do
timeout 300 ncu --set full --import-source on --clock-control none -k regex:hgemm -s 3 -c 1 -o gpurun_out/r01_ours_$w python bench.py --workload $w --steps 2 --warmup 3 --no-cpu --no-e2e --no-cublas --no-side > /dev/null 2>&1
timeout 300 ncu --set full --clock-control none -k regex:'nvjet|cutlass|sm100' -s 2 -c 1 -o gpurun_out/r01_cublas_$w python bench.py --workload $w --steps 2 --warmup 3 --no-cpu --no-e2e --no-side > /dev/null 2>&1
done
ls -la gpurun_out
