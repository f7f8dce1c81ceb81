"""Event-timed (L2 flushed) HBM-streaming shapes: automatic choice, the streaming kernel
at several chunk widths (forced), and cuBLAS (experiments).

    python tools/stream_sweep.py
"""
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402

torch.backends.cuda.matmul.allow_fp16_reduced_precision_reduction = False
w = torch.empty(64 * 1024 * 1024, device="cuda")
r = torch.zeros(64 * 1024 * 1024, device="cuda")


def timed(fn, reps=40):
    for _ in range(3):
        fn()
    ts = []
    for _ in range(reps):
        w.zero_()
        r.sum()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        ts.append((e0, e1))
    torch.cuda.synchronize()
    v = [a.elapsed_time(b) * 1e3 for a, b in ts]
    # the event clock ticks in ~2 us steps on this box: the mean over the reps
    # resolves differences below one step, the median does not
    return statistics.mean(v) if "--mean" in sys.argv else statistics.median(v)


shapes = [(16384, 64, 4096, 0.0), (16384, 128, 4096, 0.0), (16384, 256, 4096, 0.0), (16384, 192, 4096, 0.0),
          (16384, 160, 4096, 0.0), (16384, 96, 4096, 0.0),
          (64, 4096, 2048, 1.0), (256, 4096, 2048, 1.0)]
if "--skinny" in sys.argv:
    shapes = shapes[:6]
if "--lstm" in sys.argv:
    shapes = shapes[6:]
for (m, n, k, beta) in shapes:
    A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
    B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
    C = (torch.rand(n, m, device="cuda") * 2 - 1).half()

    def ours():
        binding.hgemm(m, n, k, 1.0, A, k, B, k, beta, C, m, "T", "N", "f16")
    binding.set_config()
    res = [f"auto {timed(ours):6.1f} ({binding.get_stats()['last_kernel']}/{binding.get_stats()['block_n']})"]
    cws = [16, 32, 48, 64, 96, 112, 128] if min(m, n) <= 256 and "--lstm" not in sys.argv else []
    if "--skinny" in sys.argv:
        cws = [112]
        if n > 128:
            for tn in (208, 224, 240, 256):
                binding.set_config("tc2", block_n=256, tile_n=tn)
                t = timed(ours)
                st = binding.get_stats()
                res.append(f"tc2/256 tile_n {tn} {t:6.1f}" + ("" if st["last_kernel"] == "tc2" else f"[{st['last_kernel']}]"))
    for cw in cws:
        try:
            binding.set_config("stream", block_n=cw)
            t = timed(ours)
            st = binding.get_stats()
            res.append(f"cw{cw} {t:6.1f}" + ("" if st["last_kernel"] == "stream" else f"[{st['last_kernel']}]"))
        except Exception as e:  # noqa: BLE001
            res.append(f"cw{cw} err")
    binding.set_config()
    tc = timed(lambda: torch.addmm(C, B, A.t(), beta=beta, out=C) if beta else torch.mm(B, A.t(), out=C))
    print(f"{m}x{n}x{k} beta={beta}: " + "  ".join(res) + f"  | cuBLAS {tc:6.1f} us", flush=True)
