# hardware-suspended waits (try_wait + time hint) for the producer's empty waits and the epilogue's
# accumulator polls, vs polling (HGEMM_EXP=64): instructions (ncu), sustained and default bench
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "random_ragged or half_tile or stream_k or alpha_beta" 2>&1 | tail -2 > gpurun_out/j33_tests.log
M="gpu__time_duration.sum,smsp__inst_executed.sum,gpc__cycles_elapsed.avg.per_second,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed"
for e in 0 64; do
  HGEMM_EXP=$e timeout 300 ncu --metrics $M --clock-control none -k regex:hgemm_tc -s 3 -c 1 --csv --log-file gpurun_out/sl_$e.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e --no-side --no-strong --no-cublas > /dev/null 2>&1
done
python - <<'PY' > gpurun_out/j33_ncu.log
import csv
for e in (0, 64):
    rows = [r for r in csv.reader(open(f"gpurun_out/sl_{e}.csv")) if r]
    i = [k for k, r in enumerate(rows) if r[0] == "ID"][0]
    hdr = rows[i]
    print("EXP", e, {dict(zip(hdr, r))["Metric Name"]: dict(zip(hdr, r))["Metric Value"] for r in rows[i + 1:]})
PY
for rep in 1 2; do for e in 0 64; do
  HGEMM_EXP=$e timeout 200 python tools/sustained.py --m 8192 --warm 2 --iters 300 --order ours | sed "s/^/8192 exp$e /"
  HGEMM_EXP=$e timeout 200 python tools/sustained.py --m 16384 --warm 2 --iters 100 --order ours | sed "s/^/16384 exp$e /"
done; done > gpurun_out/j33_sustained.log 2>&1
for rep in 1 2; do for e in 0 64; do
  HGEMM_EXP=$e timeout 600 python bench.py --no-cpu --no-side --no-strong --no-e2e --no-cublas 2>/dev/null | python -c "import json,sys; d=json.loads([l for l in sys.stdin if l.startswith('{')][-1]); print('bench exp$e', round(d['value'],1), round(d['clocks'].get('sm_mhz_in_kernel_median',0)))"
done; done > gpurun_out/j33_bench.log 2>&1
cat gpurun_out/j33_*.log
