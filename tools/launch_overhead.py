"""Fixed per-launch cost: device time of one launch after an L2 flush versus the
average of back-to-back launches, ours and cuBLAS, on a few shapes (experiments)."""
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402

torch.backends.cuda.matmul.allow_fp16_reduced_precision_reduction = False
w = torch.empty(64 * 1024 * 1024, device="cuda")
r = torch.zeros(64 * 1024 * 1024, device="cuda")


def flush():
    w.zero_()
    r.sum()


def single(fn, reps=20):
    ts = []
    for _ in range(reps):
        flush()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        ts.append((e0, e1))
    torch.cuda.synchronize()
    return statistics.median(a.elapsed_time(b) for a, b in ts) * 1e3


def b2b(fn, reps=20):
    fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps * 1e3


for (m, n, k, beta) in [(256, 256, 256, 0.0), (4096, 1024, 4096, 1.0), (1024, 4096, 2048, 1.0), (16384, 64, 4096, 0.0),
                        (8192, 8192, 8192, 0.0)]:
    A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
    B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
    C = (torch.rand(n, m, device="cuda") * 2 - 1).half()

    def ours():
        binding.hgemm(m, n, k, 1.0, A, k, B, k, beta, C, m, "T", "N", "f16")

    def cub():
        if beta != 0:
            torch.addmm(C, B, A.t(), beta=beta, out=C)
        else:
            torch.mm(B, A.t(), out=C)
    print(f"{m}x{n}x{k} beta={beta}: ours single {single(ours):8.1f} us  b2b {b2b(ours):8.1f} us | "
          f"cublas single {single(cub):8.1f} us  b2b {b2b(cub):8.1f} us  [{binding.get_stats()['last_kernel']}]",
          flush=True)
