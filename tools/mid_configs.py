"""Every forced kernel configuration on the mid-size shapes, event-timed after an L2 flush,
next to the automatic choice and cuBLAS (experiments: does any existing configuration beat
the automatic one?).

    python tools/mid_configs.py [--reps 20]
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
reps = int(sys.argv[sys.argv.index("--reps") + 1]) if "--reps" in sys.argv else 20


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


CONFIGS = [("tc2", dict(block_n=256)), ("tc2", dict(block_n=256, stream_k=2)), ("tc2", dict(block_n=512)),
           ("tc2", dict(block_n=512, stream_k=2)), ("tc2", dict(block_n=128)), ("tc2", dict(block_n=128, stream_k=2)),
           ("tc1", dict(block_n=256)), ("tc1", dict(block_n=128)), ("tc1", dict(block_n=128, stream_k=2)),
           ("splitk", dict(block_n=128, splits=2)), ("splitk", dict(block_n=128, splits=4))]
SHAPES = [(1792, 1792, 1792, 0.0), (2048, 2048, 2048, 0.0), (2304, 2304, 2304, 0.0), (2560, 2560, 2560, 0.0),
          (4096, 1024, 4096, 1.0), (1024, 4096, 2048, 1.0), (4096, 4096, 1024, 1.0)]
for (m, n, k, beta) in SHAPES:
    A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
    B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
    C = (torch.rand(n, m, device="cuda") * 2 - 1).half()
    f = lambda: binding.hgemm(m, n, k, 1.0, A, k, B, k, beta, C, m, "T", "N", "f16")  # noqa: E731
    binding.set_config()
    res = [f"auto {timed(f):6.1f} ({binding.get_stats()['last_kernel']}/{binding.get_stats()['block_n']})"]
    for kern, kw in CONFIGS:
        try:
            binding.set_config(kern, **kw)
            t = timed(f)
            st = binding.get_stats()
            tag = kern + "/" + "/".join(f"{k_}{v}" for k_, v in kw.items())
            res.append(f"{tag}={t:6.1f}" + ("" if st["last_kernel"] == kern else f"[{st['last_kernel']}]"))
        except Exception as e:  # noqa: BLE001
            res.append(f"{kern}{kw}=ERR {e}")
    binding.set_config()
    tc = timed(lambda: torch.addmm(C, B, A.t(), beta=beta, out=C) if beta else torch.mm(B, A.t(), out=C))
    print(f"{m}x{n}x{k} b={beta}: cuBLAS {tc:6.1f} | " + "  ".join(res), flush=True)
