"""Mid-size DL shapes (BJ configs[2]) event-timed after an L2 flush, ours (library knobs from
the environment: HGEMM_LIB, HGEMM_MC, HGEMM_EXP) vs cuBLAS (experiments).

    python tools/mid_variants.py [tag]
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
tag = sys.argv[1] if len(sys.argv) > 1 else ""


def timed(fn, reps=20):
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
    return statistics.median(a.elapsed_time(b) for a, b in ts) * 1e3


for (m, n, k, beta) in [(4096, 4096, 1024, 1.0), (4096, 1024, 4096, 1.0), (1024, 4096, 2048, 1.0),
                        (2304, 2304, 2304, 0.0), (2560, 2560, 2560, 0.0), (8192, 8192, 8192, 0.0)]:
    A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
    B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
    C = (torch.rand(n, m, device="cuda") * 2 - 1).half()
    res = []
    for kern, bn in (("auto", 0), ("tc2", 256), ("tc2", 512)):
        binding.set_config() if kern == "auto" else binding.set_config(kern, block_n=bn)
        t = timed(lambda: binding.hgemm(m, n, k, 1.0, A, k, B, k, beta, C, m, "T", "N", "f16"))
        st = binding.get_stats()
        res.append(f"{kern}/{bn or st['block_n']} {t:7.1f}")
    binding.set_config()
    tc = timed(lambda: torch.addmm(C, B, A.t(), beta=beta, out=C) if beta else torch.mm(B, A.t(), out=C))
    print(f"{tag} {m}x{n}x{k} beta={beta}: " + "  ".join(res) + f"  | cuBLAS {tc:7.1f} us", flush=True)
