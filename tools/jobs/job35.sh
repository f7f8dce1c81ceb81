# does a cluster launch attribute cost kernel time? tc1 kernels with / without it (HGEMM_EXP=16), ncu durations
mkdir -p gpurun_out
cat > /tmp/tc1.py <<'PY'
import sys, torch
sys.path.insert(0, ".")
from paper_conf_ipps_00020c20_b200 import binding
for (m, n, k) in [(256, 256, 256), (512, 512, 1024), (1024, 1024, 2048)]:
    A = (torch.rand(m, k, device="cuda") * 2 - 1).half(); B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
    C = torch.empty(n, m, dtype=torch.half, device="cuda")
    binding.set_config("tc1", block_n=128)
    for _ in range(5):
        binding.hgemm(m, n, k, 1.0, A, k, B, k, 0.0, C, m, "T", "N", "f16")
    torch.cuda.synchronize()
PY
for e in 0 16; do
  HGEMM_EXP=$e ncu --metrics gpu__time_duration.sum,sm__cycles_active.max,gpc__cycles_elapsed.max --clock-control none --csv \
    --log-file gpurun_out/tc1_e$e.csv python /tmp/tc1.py > /dev/null 2>&1
done
python - <<'PY'
import csv, collections, statistics
for e in (0, 16):
    rows = [r for r in csv.reader(open(f"gpurun_out/tc1_e{e}.csv")) if r]
    i = [k for k, r in enumerate(rows) if r[0] == "ID"][0]
    hdr = rows[i]; d = collections.OrderedDict()
    for r in rows[i + 1:]:
        x = dict(zip(hdr, r))
        if "hgemm" not in x["Kernel Name"]: continue
        d.setdefault(x["ID"], {})[x["Metric Name"]] = float(x["Metric Value"].replace(",", ""))
    vals = list(d.values())
    for s in range(3):
        grp = vals[5 * s + 1: 5 * s + 5]
        print("EXP", e, "shape", s, "dur us", statistics.median(g["gpu__time_duration.sum"] for g in grp) / 1e3,
              "sm_active_max", statistics.median(g["sm__cycles_active.max"] for g in grp),
              "elapsed", statistics.median(g["gpc__cycles_elapsed.max"] for g in grp))
PY
