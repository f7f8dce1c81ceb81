# DRAM traffic / duration of the 8192^3 tile kernel with TMA L2 cache hints (cold, ncu)
M="gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_srcunit_ltcfabric.sum"
for h in 0 1 2; do
  HGEMM_L2_HINT=$h timeout 200 ncu --metrics $M --clock-control none -k regex:hgemm_tc -s 3 -c 3 --csv --log-file gpurun_out/l2hint_$h.csv \
    python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e --no-cublas --no-side > /dev/null 2>&1
done
python - <<'PY'
import csv, glob, collections
for f in sorted(glob.glob("gpurun_out/l2hint_*.csv")):
    rows = [r for r in csv.reader(open(f)) if r]
    i = [k for k, r in enumerate(rows) if r[0] == "ID"][0]
    hdr = rows[i]
    d = collections.defaultdict(list)
    for r in rows[i + 1:]:
        x = dict(zip(hdr, r))
        d[x["Metric Name"]].append(float(x["Metric Value"].replace(",", "")))
    print(f, {k: round(sum(v) / len(v), 2) for k, v in d.items()})
PY
