# Traffic that costs energy under the power cap (DRAM, L2 reads, die-to-die fabric, instructions),
# ours per raster grouping vs cuBLAS, on one workload (cold launch under ncu, serialised):
#   bash tools/ncu_energy.sh <workload> -> gpurun_out/energy_<workload>_<variant>.csv, summary on stdout
w=${1:-sq_16384}
M="gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_ltcfabric.sum,smsp__inst_executed.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed,gpc__cycles_elapsed.avg.per_second"
B="python bench.py --workload $w --steps 2 --warmup 3 --no-cpu --no-e2e --no-side --no-strong"
for gm in 8 16 32; do
  timeout 300 ncu --metrics $M --clock-control none -k regex:hgemm_tc -s 3 -c 1 --csv --log-file gpurun_out/energy_${w}_gm$gm.csv \
    $B --no-cublas --group-m $gm > /dev/null 2>&1
done
for gn in 8 16; do
  HGEMM_GROUP_N=$gn timeout 300 ncu --metrics $M --clock-control none -k regex:hgemm_tc -s 3 -c 1 --csv \
    --log-file gpurun_out/energy_${w}_gn$gn.csv $B --no-cublas > /dev/null 2>&1
done
timeout 300 ncu --metrics $M --clock-control none -k regex:nvjet -s 2 -c 1 --csv --log-file gpurun_out/energy_${w}_cublas.csv \
  $B > /dev/null 2>&1
python - "$w" <<'PY'
import csv, glob, collections, sys
for f in sorted(glob.glob(f"gpurun_out/energy_{sys.argv[1]}_*.csv")):
    rows = [r for r in csv.reader(open(f)) if r]
    try:
        i = [k for k, r in enumerate(rows) if r[0] == "ID"][0]
    except IndexError:
        print(f, "no data"); continue
    hdr = rows[i]
    d = collections.defaultdict(list)
    for r in rows[i + 1:]:
        x = dict(zip(hdr, r))
        d[x["Metric Name"]].append(float(x["Metric Value"].replace(",", "")))
    print(f.split("/")[-1], {k.split("__")[1][:40]: round(sum(v) / len(v), 3) for k, v in d.items()})
PY
