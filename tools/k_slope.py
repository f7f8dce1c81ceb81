"""Mainloop rate vs fixed cost: time one cold launch at several K for a fixed
(m, n) tile grid, ours and cuBLAS; the slope over K is the per-k-block rate,
the intercept the fixed cost (launch, prologue, epilogue, teardown).

    python tools/k_slope.py [m n beta]
"""
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402

torch.backends.cuda.matmul.allow_fp16_reduced_precision_reduction = False
m = int(sys.argv[1]) if len(sys.argv) > 1 else 4096
n = int(sys.argv[2]) if len(sys.argv) > 2 else 1024
beta = float(sys.argv[3]) if len(sys.argv) > 3 else 1.0
w = torch.empty(64 * 1024 * 1024, device="cuda")


def single(fn, reps=15):
    ts = []
    for _ in range(reps):
        w.zero_()
        torch.cuda._sleep(100000)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        ts.append((e0, e1))
    torch.cuda.synchronize()
    return statistics.median(a.elapsed_time(b) for a, b in ts) * 1e3


rows = []
for k in (512, 1024, 2048, 4096, 8192, 16384):
    A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
    B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
    C = (torch.rand(n, m, device="cuda") * 2 - 1).half()

    def ours():
        binding.hgemm(m, n, k, 1.0, A, k, B, k, beta, C, m, "T", "N", "f16")

    def cub():
        torch.addmm(C, B, A.t(), beta=beta, out=C)
    to, tc = single(ours), single(cub)
    rows.append((k, to, tc))
    print(f"{m}x{n}x{k} beta={beta}: ours {to:8.2f} us  cublas {tc:8.2f} us  [{binding.get_stats()['last_kernel']}/"
          f"{binding.get_stats()['block_n']}]", flush=True)
for name, idx in (("ours", 1), ("cublas", 2)):
    ks = [r[0] for r in rows]
    ts = [r[idx] for r in rows]
    mk, mt = statistics.mean(ks), statistics.mean(ts)
    slope = sum((a - mk) * (b - mt) for a, b in zip(ks, ts)) / sum((a - mk) ** 2 for a in ks)
    icpt = mt - slope * mk
    print(f"{name}: {slope * 64 * 1e3:.1f} ns per k-block of 64, intercept {icpt:.2f} us")
