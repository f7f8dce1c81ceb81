"""Run the fused all-gather GEMM (hgemm_allgather_a) with W virtual ranks on one GPU, for ncu.

    python tools/ag_probe.py [--m 8192 --n 8192 --k 8192 --world 8 --reps 3]
"""
import argparse
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402
from paper_conf_ipps_00020c20_b200.sharded import default_chunk_rows, slab_bounds  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--m", type=int, default=8192)
ap.add_argument("--n", type=int, default=8192)
ap.add_argument("--k", type=int, default=8192)
ap.add_argument("--world", type=int, default=8)
ap.add_argument("--reps", type=int, default=3)
a = ap.parse_args()
m, n, k, W = a.m, a.n, a.k, a.world
cr = default_chunk_rows(m, W)
rs = [slab_bounds(m, W, q, align=cr)[0] for q in range(W)] + [m]
g = torch.Generator(device="cuda").manual_seed(1)
full = (torch.rand(m, k, generator=g, device="cuda") * 2 - 1).half()
bufs = [full.clone() for _ in range(W)]
B = (torch.rand(n, k, generator=g, device="cuda") * 2 - 1).half()
C = torch.empty(n, m, dtype=torch.float16, device="cuda")
ws = torch.zeros(1 + -(-m // cr), dtype=torch.int32, device="cuda")
for _ in range(a.reps):
    bufs[0][rs[1]:].zero_()
    binding.hgemm_allgather_a(m, n, k, 1.0, bufs[0], k, bufs, rs, 0, B, k, 0.0, C, m, "N", "f16",
                              workspace=ws, chunk_rows=cr)
torch.cuda.synchronize()
assert torch.equal(bufs[0], full)
print("ok", binding.get_stats())
