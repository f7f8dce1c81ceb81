# wave-barrier experiment (HGEMM_WSYNC=1): sustained throughput + DRAM traffic; parity under it
mkdir -p gpurun_out
HGEMM_WSYNC=1 timeout 900 python -m pytest tests/test_gpu_large.py -q -x -k "metric_config or cfg5_full_32768 or half_tile" 2>&1 | tail -3 > gpurun_out/j17_tests.log
for rep in 1 2; do
for v in "0 16" "1 16" "0 32" "1 32"; do set -- $v
  HGEMM_WSYNC=$1 timeout 200 python tools/sustained.py --m 32768 --warm 2 --iters 12 --order ours --group-m $2 | sed "s/^/32768 wsync$1 gm$2 /"
done
for v in "0 16" "1 16"; do set -- $v
  HGEMM_WSYNC=$1 timeout 200 python tools/sustained.py --m 16384 --warm 2 --iters 100 --order ours --group-m $2 | sed "s/^/16384 wsync$1 gm$2 /"
  HGEMM_WSYNC=$1 timeout 200 python tools/sustained.py --m 8192 --warm 2 --iters 300 --order ours --group-m $2 | sed "s/^/8192 wsync$1 gm$2 /"
done
done > gpurun_out/j17_sustained_wsync.log 2>&1
M="gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_ltcfabric.sum"
for v in "0 16" "1 16" "1 32"; do set -- $v
  HGEMM_WSYNC=$1 timeout 300 ncu --metrics $M --clock-control none -k regex:hgemm_tc -s 3 -c 1 --csv \
    --log-file gpurun_out/w_${1}_gm$2.csv python bench.py --workload cfg5_sharded_32768 --steps 1 --warmup 3 --no-cpu \
    --no-e2e --no-side --no-strong --no-cublas --group-m $2 > /dev/null 2>&1
done
python - <<'PY' > gpurun_out/j17_ncu.log
import csv, glob
for f in sorted(glob.glob("gpurun_out/w_*.csv")):
    rows = [r for r in csv.reader(open(f)) if r]
    try:
        i = [k for k, r in enumerate(rows) if r[0] == "ID"][0]
    except IndexError:
        print(f, "no data"); continue
    hdr = rows[i]; d = {}
    for r in rows[i + 1:]:
        x = dict(zip(hdr, r)); d[x["Metric Name"]] = float(x["Metric Value"].replace(",", ""))
    print(f"{f.split('/')[-1]:16s} t {d['gpu__time_duration.sum']/1e3:9.1f} us  dram_rd {d['dram__bytes_read.sum']/1e9:7.2f} GB  "
          f"L2rd {d['lts__t_sectors_srcunit_tex_op_read.sum']*32/1e9:7.2f} GB  fabric {d['lts__t_sectors_srcunit_ltcfabric.sum']*32/1e9:7.2f} GB")
PY
cat gpurun_out/j17_*.log
