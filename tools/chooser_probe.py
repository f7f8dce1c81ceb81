"""Forced tile configurations on the sweep's weakest shapes (small W, long K), ncu-timed via
launch_cost_join (experiments: calibrating choose_tc's per-tile-shape efficiencies).

    python tools/chooser_probe.py > order.txt
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402

SHAPES = [(1280, 1280, 1280), (1536, 1536, 1536), (1280, 1280, 2560), (1280, 1280, 5120), (1536, 1536, 3072),
          (1536, 1536, 6144), (1024, 2048, 1024), (2560, 1280, 1280), (1792, 1792, 7168), (1024, 1024, 4096)]
CONFIGS = [("auto", {}), ("tc1", dict(block_n=128)), ("tc1", dict(block_n=128, stream_k=2)),
           ("tc1", dict(block_n=256)), ("tc2", dict(block_n=256)), ("tc2", dict(block_n=256, stream_k=2)),
           ("tc2", dict(block_n=256, stream_k=1)), ("tc2", dict(block_n=512))]
w = torch.empty(64 * 1024 * 1024, device="cuda")
for (m, n, k) in SHAPES:
    A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
    B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
    C = torch.zeros(n, m, device="cuda", dtype=torch.half)
    for kern, kw in CONFIGS:
        if kern == "auto":
            binding.set_config()
        else:
            binding.set_config(kern, **kw)
        for _ in range(3):
            w.zero_()
            binding.hgemm(m, n, k, 1.0, A, k, B, k, 0.0, C, m, "T", "N", "f16")
            torch.cuda.synchronize()
            st = binding.get_stats()
            print(f"{m}x{n}x{k} {kern}/{'/'.join(f'{a}{b}' for a, b in kw.items())} -> "
                  f"{st['last_kernel']}/{st['block_n']} sk{st['stream_k']}", flush=True)
    binding.set_config()
    for _ in range(3):
        w.zero_()
        torch.mm(B, A.t(), out=C)
        torch.cuda.synchronize()
        print(f"{m}x{n}x{k} cublas", flush=True)
