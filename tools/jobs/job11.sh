mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "flexible" 2>&1 | tail -15 > gpurun_out/j11_flex_tests.log
cat > /tmp/flex_sweep.py <<'PY'
import sys, statistics, torch
sys.path.insert(0, ".")
from paper_conf_ipps_00020c20_b200 import binding
torch.backends.cuda.matmul.allow_fp16_reduced_precision_reduction = False
w_ = torch.empty(64 * 1024 * 1024, device="cuda"); r_ = torch.zeros(64 * 1024 * 1024, device="cuda")
def timed(fn, reps=15):
    for _ in range(3): fn()
    ts = []
    for _ in range(reps):
        w_.zero_(); r_.sum()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); fn(); e1.record(); ts.append((e0, e1))
    torch.cuda.synchronize()
    return statistics.median(a.elapsed_time(b) for a, b in ts) * 1e3
shapes = [(W, W, W, 0.0) for W in (1536, 1792, 2048, 2304, 2560, 2816, 3072, 3328, 3584, 3840, 4352, 4608, 5120)]
shapes += [(4096, 4096, 1024, 1.0), (4096, 1024, 4096, 1.0), (1024, 4096, 2048, 1.0)]
for (m, n, k, beta) in shapes:
    A = (torch.rand(m, k, device="cuda") * 2 - 1).half(); B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
    C = (torch.rand(n, m, device="cuda") * 2 - 1).half()
    f = lambda: binding.hgemm(m, n, k, 1.0, A, k, B, k, beta, C, m, "T", "N", "f16")
    binding.set_config(); ta = timed(f); st = binding.get_stats()
    res = [f"auto {ta:6.1f} ({st['last_kernel']}/{st['block_n']}/{st['tile_n']})"]
    for tn in (256, 240, 224, 208, 192, 176, 160, 144, 128):
        binding.set_config("tc2", block_n=256, tile_n=0 if tn == 256 else tn, stream_k=1)
        res.append(f"{tn}:{timed(f):6.1f}")
    binding.set_config()
    tc = timed(lambda: torch.addmm(C, B, A.t(), beta=beta, out=C) if beta else torch.mm(B, A.t(), out=C))
    print(f"{m}x{n}x{k} b={beta}: " + " ".join(res) + f" | cuBLAS {tc:6.1f}", flush=True)
PY
timeout 900 python /tmp/flex_sweep.py > gpurun_out/j11_flex_sweep.log 2>&1
cat gpurun_out/j11_*.log
