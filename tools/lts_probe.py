"""Is the 256-wide mainloop bound per SM or chip-wide?  The same single-wave shape with the
persistent grid capped at fewer CTA pairs (each pair then runs several tiles in sequence):
a chip-wide L2-throughput limit lets the per-tile time fall as fewer SMs load, a per-SM
limit keeps it (experiments; run under ncu for cold per-launch times).

    python tools/lts_probe.py [--warm] > order.txt

--warm: no L2 flush between launches (run ncu with --cache-control none): operands L2-resident.
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402

w = torch.empty(64 * 1024 * 1024, device="cuda")
for (m, n, k) in [(4096, 1024, 4096), (2048, 2048, 8192)]:
    A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
    B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
    C = torch.zeros(n, m, device="cuda", dtype=torch.half)
    for mc in (0, 96, 64, 32, 16):
        binding.set_config("tc2", block_n=256, max_ctas=mc, stream_k=1)
        for _ in range(3):
            if "--warm" not in sys.argv:
                w.zero_()
            binding.hgemm(m, n, k, 1.0, A, k, B, k, 0.0, C, m, "T", "N", "f16")
            torch.cuda.synchronize()
            print(f"{m}x{n}x{k} tc2/256 max_ctas={mc}", flush=True)
    binding.set_config()
