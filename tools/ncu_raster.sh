# DRAM traffic and duration of the 8192^3 tile kernel per raster grouping (cold, ncu):
#   bash tools/ncu_raster.sh  -> gpurun_out/raster_<variant>.csv, summary on stdout
M="gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct"
for gm in 4 8 16 32; do
  timeout 200 ncu --metrics $M --clock-control none -k regex:hgemm_tc -s 3 -c 3 --csv --log-file gpurun_out/raster_gm$gm.csv \
    python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e --no-cublas --no-side --no-strong --group-m $gm > /dev/null 2>&1
done
for gn in 4 8 16; do
  HGEMM_GROUP_N=$gn timeout 200 ncu --metrics $M --clock-control none -k regex:hgemm_tc -s 3 -c 3 --csv \
    --log-file gpurun_out/raster_gn$gn.csv python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e --no-cublas --no-side --no-strong > /dev/null 2>&1
done
python - <<'PY'
import csv, glob, collections
for f in sorted(glob.glob("gpurun_out/raster_*.csv")):
    rows = [r for r in csv.reader(open(f)) if r]
    i = [k for k, r in enumerate(rows) if r[0] == "ID"][0]
    hdr = rows[i]
    d = collections.defaultdict(list)
    for r in rows[i + 1:]:
        x = dict(zip(hdr, r))
        d[x["Metric Name"]].append((float(x["Metric Value"].replace(",", "")), x["Metric Unit"]))
    print(f, {k: (round(sum(v for v, _ in xs) / len(xs), 2), xs[0][1]) for k, xs in d.items()})
PY
