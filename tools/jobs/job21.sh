# L2 prefetch distance sweep (HGEMM_L2PF) on mid-size, skinny, LSTM and 8192^3 shapes
mkdir -p gpurun_out
HGEMM_L2PF=8 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "random_ragged or integer_bit_exact" 2>&1 | tail -2 > gpurun_out/j21_tests.log
for pf in 0 4 8 16; do
  HGEMM_L2PF=$pf timeout 300 python tools/mid_variants.py pf$pf
done > gpurun_out/j21_mid.log 2>&1
cat > /tmp/small.py <<'PY'
import sys, os, statistics, torch
sys.path.insert(0, ".")
from paper_conf_ipps_00020c20_b200 import binding
torch.backends.cuda.matmul.allow_fp16_reduced_precision_reduction = False
w_ = torch.empty(64 * 1024 * 1024, device="cuda"); r_ = torch.zeros(64 * 1024 * 1024, device="cuda")
def timed(fn, reps=20):
    for _ in range(3): fn()
    ts = []
    for _ in range(reps):
        w_.zero_(); r_.sum()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); ts.append((e0, e1))
    torch.cuda.synchronize()
    return statistics.median(a.elapsed_time(b) for a, b in ts) * 1e3
tag = sys.argv[1]
for (m, n, k, beta) in [(16384, 64, 4096, 0.0), (16384, 128, 4096, 0.0), (16384, 256, 4096, 0.0),
                        (64, 4096, 2048, 1.0), (256, 4096, 2048, 1.0)]:
    A = (torch.rand(m, k, device="cuda") * 2 - 1).half(); B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
    C = (torch.rand(n, m, device="cuda") * 2 - 1).half()
    t = timed(lambda: binding.hgemm(m, n, k, 1.0, A, k, B, k, beta, C, m, "T", "N", "f16"))
    st = binding.get_stats()
    print(f"{tag} {m}x{n}x{k} b={beta}: {t:6.1f} us ({st['last_kernel']}/{st['block_n']})", flush=True)
PY
for pf in 0 2 4 8 16; do HGEMM_L2PF=$pf timeout 300 python /tmp/small.py pf$pf; done > gpurun_out/j21_small.log 2>&1
cat gpurun_out/j21_*.log
