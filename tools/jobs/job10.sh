mkdir -p gpurun_out
cat > /tmp/mid_sq.py <<'PY'
import sys, torch
sys.path.insert(0, ".")
from paper_conf_ipps_00020c20_b200 import binding
torch.backends.cuda.matmul.allow_fp16_reduced_precision_reduction = False
for W in (1792, 2048, 2304, 2560, 2816, 3328, 3584, 4608, 5120, 6144):
    A = (torch.rand(W, W, device="cuda") * 2 - 1).half()
    B = (torch.rand(W, W, device="cuda") * 2 - 1).half()
    C = torch.empty(W, W, dtype=torch.half, device="cuda")
    for _ in range(2):
        binding.hgemm(W, W, W, 1.0, A, W, B, W, 0.0, C, W, "T", "N", "f16")
        torch.mm(B, A.t(), out=C)
    torch.cuda.synchronize()
PY
ncu --metrics gpu__time_duration.sum,launch__grid_size,launch__cluster_dim_x,launch__cluster_dim_y --clock-control none --csv \
  --log-file gpurun_out/j10_midsq.csv python /tmp/mid_sq.py > /dev/null 2>&1
python - <<'PY'
import csv, collections
rows = [r for r in csv.reader(open("gpurun_out/j10_midsq.csv")) if r]
i = [k for k, r in enumerate(rows) if r[0] == "ID"][0]
hdr = rows[i]; d = collections.OrderedDict()
for r in rows[i + 1:]:
    x = dict(zip(hdr, r))
    d.setdefault(x["ID"], {"name": x["Kernel Name"].split("(")[0][:60]})[x["Metric Name"]] = x["Metric Value"]
for k, v in d.items():
    print(k, v["name"], v.get("gpu__time_duration.sum"), "grid", v.get("launch__grid_size"), "cl", v.get("launch__cluster_dim_x"), v.get("launch__cluster_dim_y"))
PY
