mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "splitk" 2>&1 | tail -3 > gpurun_out/j12_tests.log
timeout 300 python tools/stream_sweep.py > gpurun_out/j12_stream_sweep.log 2>&1
cat > /tmp/sk_sweep.py <<'PY'
import sys, statistics, torch
sys.path.insert(0, ".")
from paper_conf_ipps_00020c20_b200 import binding
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
for (m, n, k) in [(64, 4096, 2048), (256, 4096, 2048), (128, 4096, 2048), (64, 4096, 4096), (32, 8192, 2048)]:
    A = (torch.rand(m, k, device="cuda") * 2 - 1).half(); B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
    C = (torch.rand(n, m, device="cuda") * 2 - 1).half()
    f = lambda: binding.hgemm(m, n, k, 1.0, A, k, B, k, 1.0, C, m, "T", "N", "f16")
    binding.set_config(); res = [f"auto {timed(f):6.1f} {binding.get_stats()['block_n']}x{binding.get_stats()['splits']}"]
    for bn in (64, 128):
        for s in (2, 4, 8):
            try:
                binding.set_config("splitk", block_n=bn, splits=s); res.append(f"{bn}x{s}:{timed(f):6.1f}")
            except Exception as e:
                res.append(f"{bn}x{s}:err")
    binding.set_config()
    tc = timed(lambda: torch.addmm(C, B, A.t(), beta=1.0, out=C))
    print(f"{m}x{n}x{k}: " + " ".join(res) + f" | cuBLAS {tc:6.1f}", flush=True)
PY
timeout 600 python /tmp/sk_sweep.py > gpurun_out/j12_sk_sweep.log 2>&1
python -m paper_conf_ipps_00020c20_b200.build -DHGEMM_TRACE --out=/tmp/libhgemm_trace.so > /dev/null 2>&1
for s in "64 4096 2048" "256 4096 2048"; do HGEMM_LIB=/tmp/libhgemm_trace.so timeout 120 python tools/trace_sk.py $s; done > gpurun_out/j12_trace_sk.log 2>&1
cat gpurun_out/j12_*.log
