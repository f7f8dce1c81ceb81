mkdir -p gpurun_out
M="gpu__time_duration.sum,smsp__inst_executed.sum,sm__cycles_active.avg,gpc__cycles_elapsed.max"
python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e --no-cublas --no-side --no-strong > /dev/null 2>&1 || echo "plain failed"
for e in 0 128 256 384; do
  HGEMM_EXP=$e timeout 300 ncu --metrics $M --clock-control none -k regex:hgemm_tc -s 3 -c 3 --csv --log-file gpurun_out/bo_$e.csv \
    python bench.py --steps 3 --warmup 3 --no-cpu --no-e2e --no-cublas --no-side --no-strong > /dev/null 2>&1
done
python - <<'PY'
import csv, glob, collections, statistics
for f in sorted(glob.glob("gpurun_out/bo_*.csv")):
    rows = [r for r in csv.reader(open(f)) if r]
    i = [k for k, r in enumerate(rows) if r[0] == "ID"][0]
    hdr = rows[i]; d = collections.defaultdict(list)
    for r in rows[i + 1:]:
        x = dict(zip(hdr, r)); d[x["Metric Name"]].append(float(x["Metric Value"].replace(",", "")))
    m = {k: statistics.median(v) for k, v in d.items()}
    print(f, {k: round(v, 1) for k, v in m.items()})
PY
for e in 0 384; do
  HGEMM_EXP=$e python tools/launch_cost_ncu.py --gemm-only > /dev/null 2>&1
  HGEMM_EXP=$e ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/bo_lc_$e.csv \
    python tools/launch_cost_ncu.py --gemm-only > gpurun_out/bo_lc_${e}_order.txt 2>/dev/null
  python tools/launch_cost_join.py gpurun_out/bo_lc_$e.csv gpurun_out/bo_lc_${e}_order.txt > gpurun_out/bo_lc_$e.log
done
paste gpurun_out/bo_lc_0.log gpurun_out/bo_lc_384.log | grep ours | awk -F'\t' '{print substr($1,1,90) " || exp384 " substr($2, 76, 12)}'
for rep in 1 2 3; do for e in 0 384; do
  HGEMM_EXP=$e python tools/headline_ab.py --blocks 3 --block 100 --variants ours,cublas | grep TOTAL | sed "s/^/exp$e rep$rep /"
done; done
