mkdir -p gpurun_out
python tools/cluster_occupancy.py > gpurun_out/j16_cluster_occupancy.log 2>&1
for rep in 1 2; do
for v in "0 16" "32 16" "0 32" "32 32" "32 24" "32 12"; do set -- $v
  HGEMM_EXP=$1 timeout 200 python tools/sustained.py --m 32768 --warm 2 --iters 12 --order ours --group-m $2 | sed "s/^/32768 exp$1 gm$2 /"
done
timeout 200 python tools/sustained.py --m 32768 --warm 2 --iters 12 --order cublas | sed "s/^/32768 /"
for v in "0 16" "32 16" "0 32" "32 32" "32 24" "32 12"; do set -- $v
  HGEMM_EXP=$1 timeout 200 python tools/sustained.py --m 16384 --warm 2 --iters 100 --order ours --group-m $2 | sed "s/^/16384 exp$1 gm$2 /"
done
timeout 200 python tools/sustained.py --m 16384 --warm 2 --iters 100 --order cublas | sed "s/^/16384 /"
done > gpurun_out/j16_sustained_raster.log 2>&1
cat gpurun_out/j16_*.log
