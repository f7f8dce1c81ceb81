# 8192^3: intra-tile meetings (HGEMM_WSYNC_K) -> L2 / fabric traffic (ncu) and the default bench line
mkdir -p gpurun_out
M="gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_ltcfabric.sum"
for kk in 0 64 32 16; do
  HGEMM_WSYNC_K=$kk timeout 300 ncu --metrics $M --clock-control none -k regex:hgemm_tc -s 3 -c 3 --csv \
    --log-file gpurun_out/k8_$kk.csv python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e --no-side --no-strong --no-cublas > /dev/null 2>&1
done
python - <<'PY' > gpurun_out/j23_ncu.log
import csv, glob, collections
for f in sorted(glob.glob("gpurun_out/k8_*.csv")):
    rows = [r for r in csv.reader(open(f)) if r]
    try:
        i = [k for k, r in enumerate(rows) if r[0] == "ID"][0]
    except IndexError:
        print(f, "no data"); continue
    hdr = rows[i]; d = collections.defaultdict(list)
    for r in rows[i + 1:]:
        x = dict(zip(hdr, r)); d[x["Metric Name"]].append(float(x["Metric Value"].replace(",", "")))
    g = lambda k: sum(d[k]) / len(d[k])
    print(f"{f.split('/')[-1]:10s} t {g('gpu__time_duration.sum')/1e3:8.1f} us  dram_rd {g('dram__bytes_read.sum')/1e6:7.1f} MB  "
          f"L2rd {g('lts__t_sectors_srcunit_tex_op_read.sum')/1e6:7.1f} Msec  fabric {g('lts__t_sectors_srcunit_ltcfabric.sum')/1e6:6.1f} Msec")
PY
for r in 1 2; do for kk in 0 32; do
  HGEMM_WSYNC_K=$kk timeout 600 python bench.py --no-cpu --no-side --no-strong --no-e2e > gpurun_out/j23_bench_k${kk}_$r.log 2>&1
done; done
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/j23_bench_*.log")):
    l = [x for x in open(f) if x.startswith("{")]
    d = json.loads(l[-1])
    print(f.split("/")[-1], f"value {d['value']:.1f} cublas {d['cublas']['value']:.1f} clk {d['clocks'].get('sm_mhz_in_kernel_median', 0):.0f}")
PY
cat gpurun_out/j23_ncu.log
