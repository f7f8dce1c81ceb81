"""Automatic-choice launches of a list of TN FP16-out shapes, 3 each after an L2 flush, for an
ncu launch list (gpu__time_duration per launch; join with tools/launch_cost_join.py).
Library knobs come from the environment (HGEMM_*), so two runs compare variants.

    python tools/ncu_shapes.py > order.txt
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402

SHAPES = [(4096, 4096, 1024, 1.0), (16384, 4096, 1024, 1.0), (4096, 1024, 4096, 1.0), (1024, 4096, 2048, 1.0),
          (1792, 1792, 1792, 0.0), (2048, 2048, 2048, 0.0), (2304, 2304, 2304, 0.0), (2560, 2560, 2560, 0.0),
          (2816, 2816, 2816, 0.0), (3072, 3072, 3072, 0.0), (3584, 3584, 3584, 0.0), (4608, 4608, 4608, 0.0),
          (16384, 256, 4096, 0.0), (2048, 2048, 8192, 0.0)]
w = torch.empty(64 * 1024 * 1024, device="cuda")
for (m, n, k, beta) in SHAPES:
    A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
    B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
    C = (torch.rand(n, m, device="cuda") * 2 - 1).half()
    for _ in range(3):
        w.zero_()
        binding.hgemm(m, n, k, 1.0, A, k, B, k, beta, C, m, "T", "N", "f16")
        torch.cuda.synchronize()
        st = binding.get_stats()
        print(f"{m}x{n}x{k} b={beta} {st['last_kernel']}/{st['block_n']} sk{st['stream_k']}", flush=True)
