# intra-tile k alignment on top of the wave barrier (HGEMM_WSYNC_K): traffic + sustained
mkdir -p gpurun_out
HGEMM_WSYNC_K=64 timeout 600 python -m pytest tests/test_gpu_large.py -q -x -k "metric_config or cfg5_full_32768_one_gpu" 2>&1 | tail -2 > gpurun_out/j19_tests.log
M="gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_ltcfabric.sum"
for kk in 0 128 64 32; do
  HGEMM_WSYNC_K=$kk timeout 300 ncu --metrics $M --clock-control none -k regex:hgemm_tc -s 3 -c 1 --csv \
    --log-file gpurun_out/wk_$kk.csv python bench.py --workload cfg5_sharded_32768 --steps 1 --warmup 3 --no-cpu \
    --no-e2e --no-side --no-strong --no-cublas > /dev/null 2>&1
done
python - <<'PY' > gpurun_out/j19_ncu.log
import csv, glob
for f in sorted(glob.glob("gpurun_out/wk_*.csv")):
    rows = [r for r in csv.reader(open(f)) if r]
    try:
        i = [k for k, r in enumerate(rows) if r[0] == "ID"][0]
    except IndexError:
        print(f, "no data"); continue
    hdr = rows[i]; d = {}
    for r in rows[i + 1:]:
        x = dict(zip(hdr, r)); d[x["Metric Name"]] = float(x["Metric Value"].replace(",", ""))
    print(f"{f.split('/')[-1]:12s} t {d['gpu__time_duration.sum']/1e3:9.1f} us  dram_rd {d['dram__bytes_read.sum']/1e9:7.2f} GB  "
          f"L2rd {d['lts__t_sectors_srcunit_tex_op_read.sum']*32/1e9:7.2f} GB  fabric {d['lts__t_sectors_srcunit_ltcfabric.sum']*32/1e9:7.2f} GB")
PY
for rep in 1 2; do for kk in 0 128 64; do
  HGEMM_WSYNC_K=$kk timeout 200 python tools/sustained.py --m 32768 --warm 2 --iters 12 --order ours | sed "s/^/32768 k$kk /"
  HGEMM_WSYNC_K=$kk timeout 200 python tools/sustained.py --m 16384 --warm 2 --iters 100 --order ours | sed "s/^/16384 k$kk /"
  HGEMM_WSYNC_K=$kk timeout 200 python tools/sustained.py --m 8192 --warm 2 --iters 300 --order ours | sed "s/^/8192 k$kk /"
done; done > gpurun_out/j19_sustained.log 2>&1
cat gpurun_out/j19_*.log
