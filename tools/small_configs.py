"""Forced kernel configurations on the launch-bound BJ shapes (config 1, LSTM gates) and small
squares, event-timed after an L2 flush (median), next to the automatic choice and cuBLAS
(experiments).  Operands come from bench.device_operands in the workload's own layout.

    python tools/small_configs.py [--reps 30]
"""
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from paper_conf_ipps_00020c20_b200 import binding, inputs  # noqa: E402

w = torch.empty(64 * 1024 * 1024, device="cuda")
r = torch.zeros(64 * 1024 * 1024, device="cuda")
reps = int(sys.argv[sys.argv.index("--reps") + 1]) if "--reps" in sys.argv else 30


def flush():
    w.zero_()
    r.sum()


def timed(fn):
    return bench.timed(fn, flush, 3, reps)["median"] * 1e3


CONFIGS = [("tc1", dict(block_n=128)), ("tc1", dict(block_n=256)), ("tc2", dict(block_n=256)),
           ("splitk", dict(block_n=64, splits=2)), ("splitk", dict(block_n=64, splits=4)),
           ("splitk", dict(block_n=64, splits=8)), ("splitk", dict(block_n=128, splits=2)),
           ("splitk", dict(block_n=128, splits=4)), ("splitk", dict(block_n=128, splits=8)),
           ("stream", dict())]
CASES = [("cfg1_256_NN_f32", None), ("cfg3_lstm_b64", None), ("cfg3_lstm_b256", None),
         ("sq512", (512, 512, 512, "T", "N", 1.0, 0.0, "f16")), ("sq1024", (1024, 1024, 1024, "T", "N", 1.0, 0.0, "f16")),
         ("sq1536", (1536, 1536, 1536, "T", "N", 1.0, 0.0, "f16")), ("sq1792", (1792, 1792, 1792, "T", "N", 1.0, 0.0, "f16")),
         ("sq2048", (2048, 2048, 2048, "T", "N", 1.0, 0.0, "f16"))]
dev = torch.device("cuda:0")
for name, wl in CASES:
    m, n, k, tA, tB, alpha, beta, out = wl or inputs.WORKLOADS[name]
    A, lda, B, ldb, C = bench.device_operands(dev, m, n, k, tA, tB, beta, out)
    f = lambda: binding.hgemm(m, n, k, alpha, A, lda, B, ldb, beta, C, m, tA, tB, out)  # noqa: E731
    binding.set_config()
    ta = timed(f)
    st = binding.get_stats()
    res = [f"auto {ta:6.1f} ({st['last_kernel']}/{st['block_n']}/s{st['splits']})"]
    for kern, kw in CONFIGS:
        try:
            binding.set_config(kern, **kw)
            t = timed(f)
            st = binding.get_stats()
            tag = kern + "/" + "/".join(f"{v}" for v in kw.values())
            res.append(f"{tag}={t:5.1f}" + ("" if st["last_kernel"] == kern else f"[{st['last_kernel']}]"))
        except Exception as e:  # noqa: BLE001
            res.append(f"{kern}{tuple(kw.values())}=ERR")
    binding.set_config()
    tc = timed(bench.cublas_fn(A, B, C, tA, tB, alpha, beta))
    print(f"{name} {m}x{n}x{k} {tA}{tB} b={beta} {out}: cuBLAS {tc:5.1f} | " + "  ".join(res), flush=True)
