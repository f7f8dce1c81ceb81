"""Run one BJ workload (inputs.WORKLOADS name) a few times with the automatic kernel choice,
each launch after an L2 flush, then the same through cuBLAS: the target of an ncu capture
(experiments).

    python tools/run_workload.py cfg3_lstm_b64 [launches] [--no-cublas]
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from paper_conf_ipps_00020c20_b200 import binding, inputs  # noqa: E402

name = sys.argv[1]
reps = int(sys.argv[2]) if len(sys.argv) > 2 and sys.argv[2].isdigit() else 3
m, n, k, tA, tB, alpha, beta, out = inputs.WORKLOADS[name]
A, lda, B, ldb, C = bench.device_operands(torch.device("cuda:0"), m, n, k, tA, tB, beta, out)
w = torch.empty(64 * 1024 * 1024, device="cuda")
for _ in range(reps):
    w.zero_()
    binding.hgemm(m, n, k, alpha, A, lda, B, ldb, beta, C, m, tA, tB, out)
torch.cuda.synchronize()
print(name, binding.get_stats())
if "--no-cublas" not in sys.argv:
    f = bench.cublas_fn(A, B, C, tA, tB, alpha, beta)
    for _ in range(reps):
        w.zero_()
        f()
    torch.cuda.synchronize()
