mkdir -p gpurun_out
M="gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_ltcfabric.sum,sm__cycles_active.avg,gpc__cycles_elapsed.max"
run() {  # tag, env...
  tag=$1; shift
  env "$@" timeout 300 ncu --metrics $M --clock-control none -k regex:hgemm_tc -s 3 -c 3 --csv --log-file gpurun_out/ws_$tag.csv \
    python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e --no-cublas --no-side --no-strong > /dev/null 2>&1
}
python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e --no-cublas --no-side --no-strong > /dev/null 2>&1 || echo "plain failed"
run base X=1
run minw6 HGEMM_WSYNC_MINW=6
run minw6_k32 HGEMM_WSYNC_MINW=6 HGEMM_WSYNC_K=32
run minw6_k64 HGEMM_WSYNC_MINW=6 HGEMM_WSYNC_K=64
run minw4 HGEMM_WSYNC_MINW=4
python - <<'PY'
import csv, glob, collections, statistics
for f in sorted(glob.glob("gpurun_out/ws_*.csv")):
    rows = [r for r in csv.reader(open(f)) if r]
    i = [k for k, r in enumerate(rows) if r[0] == "ID"][0]
    hdr = rows[i]; d = collections.defaultdict(list)
    for r in rows[i + 1:]:
        x = dict(zip(hdr, r)); d[x["Metric Name"]].append(float(x["Metric Value"].replace(",", "")))
    m = {k: statistics.median(v) for k, v in d.items()}
    print(f"{f:32s} t {m['gpu__time_duration.sum']/1e3 if m['gpu__time_duration.sum']>1e4 else m['gpu__time_duration.sum']:8.1f} us  dram_rd {m['dram__bytes_read.sum']/1e6:7.1f} MB  dram_wr {m['dram__bytes_write.sum']/1e6:6.1f} MB  L2rd {m['lts__t_sectors_srcunit_tex_op_read.sum']*32/1e9:6.2f} GB  fabric {m['lts__t_sectors_srcunit_ltcfabric.sum']*32/1e9:6.2f} GB  active {m['sm__cycles_active.avg']:.0f}")
PY
for rep in 1 2; do
for v in base minw6; do
  if [ $v = minw6 ]; then export HGEMM_WSYNC_MINW=6; else unset HGEMM_WSYNC_MINW; fi
  python tools/headline_ab.py --blocks 3 --block 100 --variants ours | tail -1 | sed "s/^/$v /"
done; done
