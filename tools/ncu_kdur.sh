# per-kernel device durations (ncu, cold, serialised) for a few bench workloads
for w in "$@"; do
  timeout 200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum --clock-control none --csv \
     python bench.py --workload $w --steps 3 --warmup 3 --no-cpu --no-e2e 2>/dev/null > /tmp/k_$w.csv
  python - "$w" <<'PY'
import csv, sys, collections
w = sys.argv[1]
rows = [r for r in csv.reader(open(f"/tmp/k_{w}.csv")) if r]
i = [k for k, r in enumerate(rows) if r[0] == "ID"][0]
hdr = rows[i]
d = collections.defaultdict(lambda: collections.defaultdict(list))
for r in rows[i + 1:]:
    x = dict(zip(hdr, r))
    d[x["Kernel Name"][:70]][x["Metric Name"]].append(float(x["Metric Value"].replace(",", "")))
for k, m in d.items():
    if "hgemm" in k or "nvjet" in k or "gemm" in k:
        t = m["gpu__time_duration.sum"]
        print(f"{w:20s} {k:70s} n={len(t):3d} dur_us={sum(t)/len(t)/1000:8.2f} dram_MB={sum(m['dram__bytes_read.sum'])/len(t)/1e6:8.2f}")
PY
done
