# raster study at 16384^3: DRAM / fabric / L2 traffic (ncu) and sustained throughput per variant;
# also the early-TMA split-K / streaming kernels (tests + sweep)
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -k "splitk or stream" 2>&1 | tail -3 > gpurun_out/j8_tests.log
timeout 300 python tools/stream_sweep.py > gpurun_out/j8_stream_sweep.log 2>&1
M="gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_ltcfabric.sum"
B="python bench.py --workload sq_16384 --steps 2 --warmup 3 --no-cpu --no-e2e --no-side --no-strong --no-cublas"
for exp in 0 32; do for gm in 4 8 12 16 24; do
  HGEMM_EXP=$exp timeout 300 ncu --metrics $M --clock-control none -k regex:hgemm_tc -s 3 -c 1 --csv \
    --log-file gpurun_out/r_e${exp}_gm$gm.csv $B --group-m $gm > /dev/null 2>&1
done; done
python - <<'PY' > gpurun_out/j8_raster.log
import csv, glob, collections
for f in sorted(glob.glob("gpurun_out/r_e*_gm*.csv")):
    rows = [r for r in csv.reader(open(f)) if r]
    try:
        i = [k for k, r in enumerate(rows) if r[0] == "ID"][0]
    except IndexError:
        print(f, "no data"); continue
    hdr = rows[i]; d = {}
    for r in rows[i + 1:]:
        x = dict(zip(hdr, r)); d[x["Metric Name"]] = float(x["Metric Value"].replace(",", ""))
    print(f"{f.split('/')[-1]:22s} t {d['gpu__time_duration.sum']/1e3:8.1f} us  dram_rd {d['dram__bytes_read.sum']/1e9:6.2f} GB  "
          f"L2rd {d['lts__t_sectors_srcunit_tex_op_read.sum']*32/1e9:6.2f} GB  fabric {d['lts__t_sectors_srcunit_ltcfabric.sum']*32/1e9:6.2f} GB")
PY
for gm in 8 16; do for exp in 0 32; do
  HGEMM_EXP=$exp timeout 120 python tools/sustained.py --m 16384 --warm 3 --iters 150 --order ours --group-m $gm | sed "s/^/gm$gm exp$exp /"
done; done > gpurun_out/j8_sustained.log 2>&1
timeout 120 python tools/sustained.py --m 16384 --warm 3 --iters 150 --order cublas >> gpurun_out/j8_sustained.log 2>&1
cat gpurun_out/j8_*.log
