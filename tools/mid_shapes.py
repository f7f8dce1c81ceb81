"""Single-wave mid-size shapes (one 256 x 256 pair tile per CTA pair), event-timed after an
L2 flush: the auto choice of the loaded library (HGEMM_LIB and the HGEMM_* knobs from the
environment) vs cuBLAS, median of --reps launches (experiments).

    python tools/mid_shapes.py [tag] [--reps 30]
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
args = [a for a in sys.argv[1:] if not a.startswith("--")]
tag = args[0] if args else ""
reps = int(sys.argv[sys.argv.index("--reps") + 1]) if "--reps" in sys.argv else 30
no_cublas = "--no-cublas" in sys.argv


def timed(fn):
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


SHAPES = [(4096, 1024, 4096, 1.0), (4096, 1024, 4096, 0.0), (1024, 4096, 2048, 1.0), (1024, 4096, 2048, 0.0),
          (2048, 2048, 2048, 0.0), (1792, 1792, 1792, 0.0), (2048, 2048, 8192, 0.0), (4096, 4096, 1024, 1.0),
          (2304, 2304, 2304, 0.0), (2560, 2560, 2560, 0.0)]
for (m, n, k, beta) in SHAPES:
    A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
    B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
    C = (torch.rand(n, m, device="cuda") * 2 - 1).half()
    binding.set_config()
    t = timed(lambda: binding.hgemm(m, n, k, 1.0, A, k, B, k, beta, C, m, "T", "N", "f16"))
    st = binding.get_stats()
    line = f"{tag} {m}x{n}x{k} beta={beta}: ours {t:7.1f} us ({st['last_kernel']}/{st['block_n']})"
    if not no_cublas:
        tc = timed(lambda: torch.addmm(C, B, A.t(), beta=beta, out=C) if beta else torch.mm(B, A.t(), out=C))
        line += f"  | cuBLAS {tc:7.1f} us  ours/cuBLAS {tc / t:.3f}"
    print(line, flush=True)
