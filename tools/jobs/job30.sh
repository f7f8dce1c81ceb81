mkdir -p gpurun_out
python -m paper_conf_ipps_00020c20_b200.build -DHGEMM_ENABLE_MC --out=/tmp/libhgemm_mc.so > /dev/null 2>&1
M="gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_read.sum,l1tex__m_xbar2l1tex_read_bytes_mem_global_op_tma_ld.sum,sm__cycles_active.avg,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active,launch__cluster_dim_x,launch__grid_size"
for mc in 1 2; do
  HGEMM_LIB=/tmp/libhgemm_mc.so HGEMM_MC=$mc timeout 300 ncu --metrics $M --clock-control none -k regex:hgemm_tc -s 3 -c 1 --csv \
    --log-file gpurun_out/mc_$mc.csv python bench.py --workload cfg3_bert_ffn2_4096 --steps 2 --warmup 3 --no-cpu --no-e2e --no-cublas --no-side --no-strong > /dev/null 2>&1
done
python - <<'PY'
import csv
for mc in (1, 2):
    rows = [r for r in csv.reader(open(f"gpurun_out/mc_{mc}.csv")) if r]
    i = [k for k, r in enumerate(rows) if r[0] == "ID"][0]
    hdr = rows[i]
    print("MC", mc, {dict(zip(hdr, r))["Metric Name"]: dict(zip(hdr, r))["Metric Value"] for r in rows[i + 1:]})
PY
