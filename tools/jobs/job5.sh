# energy-relevant traffic at 16384^3 (ours per raster vs cuBLAS); per-CTA phases of small launches
mkdir -p gpurun_out
bash tools/ncu_energy.sh sq_16384 > gpurun_out/j5_energy.log 2>&1
python -m paper_conf_ipps_00020c20_b200.build -DHGEMM_TRACE --out=/tmp/libhgemm_trace.so > /dev/null 2>&1
for s in "256 256 256" "4096 1024 4096 --beta 1" "1024 4096 2048 --beta 1"; do
  HGEMM_LIB=/tmp/libhgemm_trace.so timeout 120 python tools/trace_cta2.py $s
done > gpurun_out/j5_trace_cta.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/j5_launches.csv \
  python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e --no-strong > /dev/null 2>&1
cat gpurun_out/j5_energy.log gpurun_out/j5_trace_cta.log
