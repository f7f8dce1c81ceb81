# raster study at 32768^3 (config 5, one GPU): DRAM / L2 / fabric traffic under ncu, sustained throughput
mkdir -p gpurun_out
M="gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_ltcfabric.sum"
B="python bench.py --workload cfg5_sharded_32768 --steps 1 --warmup 3 --no-cpu --no-e2e --no-side --no-strong --no-cublas"
for exp in 0 32; do for gm in 8 16 32; do
  HGEMM_EXP=$exp timeout 300 ncu --metrics $M --clock-control none -k regex:hgemm_tc -s 3 -c 1 --csv \
    --log-file gpurun_out/r32_e${exp}_gm$gm.csv $B --group-m $gm > /dev/null 2>&1
done; done
timeout 300 ncu --metrics $M --clock-control none -k regex:nvjet -s 2 -c 1 --csv --log-file gpurun_out/r32_cublas.csv \
  python bench.py --workload cfg5_sharded_32768 --steps 1 --warmup 3 --no-cpu --no-e2e --no-side --no-strong > /dev/null 2>&1
python - <<'PY' > gpurun_out/j14_raster32768.log
import csv, glob
for f in sorted(glob.glob("gpurun_out/r32_*.csv")):
    rows = [r for r in csv.reader(open(f)) if r]
    try:
        i = [k for k, r in enumerate(rows) if r[0] == "ID"][0]
    except IndexError:
        print(f, "no data"); continue
    hdr = rows[i]; d = {}
    for r in rows[i + 1:]:
        x = dict(zip(hdr, r)); d[x["Metric Name"]] = float(x["Metric Value"].replace(",", ""))
    print(f"{f.split('/')[-1]:22s} t {d['gpu__time_duration.sum']/1e3:9.1f} us  dram_rd {d['dram__bytes_read.sum']/1e9:7.2f} GB  "
          f"L2rd {d['lts__t_sectors_srcunit_tex_op_read.sum']*32/1e9:7.2f} GB  fabric {d['lts__t_sectors_srcunit_ltcfabric.sum']*32/1e9:7.2f} GB")
PY
for v in "0 16" "32 16" "32 8" "32 32"; do set -- $v
  HGEMM_EXP=$1 timeout 200 python tools/sustained.py --m 32768 --warm 2 --iters 15 --order ours --group-m $2 | sed "s/^/exp$1 gm$2 /"
done > gpurun_out/j14_sustained32768.log 2>&1
timeout 200 python tools/sustained.py --m 32768 --warm 2 --iters 15 --order cublas >> gpurun_out/j14_sustained32768.log 2>&1
cat gpurun_out/j14_*.log
