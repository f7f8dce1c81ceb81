# ncu --set full of our kernel and of cuBLAS (nvjet) on bench workloads:
#   bash tools/ncu_cfg.sh <tag> <workload>...   -> gpurun_out/<tag>_{ours,cublas}_<workload>.ncu-rep
tag=$1; shift
for w in "$@"; do
timeout 300 ncu --set full --import-source on --clock-control none -k regex:hgemm -s 3 -c 1 -o gpurun_out/${tag}_ours_$w python bench.py --workload $w --steps 2 --warmup 3 --no-cpu --no-e2e --no-cublas --no-side --no-strong > /dev/null 2>&1
timeout 300 ncu --set full --clock-control none -k regex:nvjet -s 2 -c 1 -o gpurun_out/${tag}_cublas_$w python bench.py --workload $w --steps 2 --warmup 3 --no-cpu --no-e2e --no-side --no-strong > /dev/null 2>&1
done
ls gpurun_out/${tag}_*
