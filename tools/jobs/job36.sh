# bisect the tc1 256^3 kernel-time change (8.4 -> 10.2 us between launch lists)
mkdir -p gpurun_out
cat > /tmp/small3.py <<'PY'
import sys, torch
sys.path.insert(0, ".")
from paper_conf_ipps_00020c20_b200 import binding
m = n = k = 256
A = (torch.rand(m, k, device="cuda") * 2 - 1).half(); B = (torch.rand(k, n, device="cuda") * 2 - 1).half()
C = torch.empty(n, m, dtype=torch.float32, device="cuda")
for _ in range(8):
    binding.hgemm(m, n, k, 1.0, A, m, B, k, 0.0, C, m, "N", "N", "f32")     # cfg1: NN, FP32 out
for (mm, nn, kk) in [(4096, 1024, 4096), (4096, 4096, 1024)]:
    A2 = (torch.rand(mm, kk, device="cuda") * 2 - 1).half(); B2 = (torch.rand(nn, kk, device="cuda") * 2 - 1).half()
    C2 = torch.empty(nn, mm, dtype=torch.half, device="cuda")
    for _ in range(5):
        binding.hgemm(mm, nn, kk, 1.0, A2, kk, B2, kk, 1.0, C2, mm, "T", "N", "f16")
torch.cuda.synchronize()
PY
for L in f4800b0 head2; do
  HGEMM_LIB=bisect/lib_$L.so ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/bis_$L.csv python /tmp/small3.py > /dev/null 2>&1
done
python - <<'PY'
import csv, statistics
for L in ("f4800b0", "head2"):
    rows = [r for r in csv.reader(open(f"gpurun_out/bis_{L}.csv")) if r]
    i = [k for k, r in enumerate(rows) if r[0] == "ID"][0]
    hdr = rows[i]
    v = [float(dict(zip(hdr, r))["Metric Value"].replace(",", "")) / 1e3 for r in rows[i + 1:] if "hgemm" in dict(zip(hdr, r))["Kernel Name"]]
    print(L, "256^3 NN f32:", round(statistics.median(v[1:8]), 2), " FFN2:", round(statistics.median(v[9:13]), 2), " FFN1-4096:", round(statistics.median(v[14:18]), 2))
PY
