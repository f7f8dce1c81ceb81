"""Forced kernel configurations of one BJ workload, 3 launches each after an L2 flush, for an
ncu launch list (gpu__time_duration per launch; join with tools/launch_cost_join.py):

    ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file X.csv \
        python tools/ncu_configs.py cfg1_256_NN_f32 > order.txt
    python tools/launch_cost_join.py X.csv order.txt
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from paper_conf_ipps_00020c20_b200 import binding, inputs  # noqa: E402

CONFIGS = [("auto", {}), ("tc1", dict(block_n=128)), ("tc1", dict(block_n=256)), ("tc2", dict(block_n=256)),
           ("splitk", dict(block_n=64, splits=2)), ("splitk", dict(block_n=64, splits=4)),
           ("splitk", dict(block_n=128, splits=2)), ("splitk", dict(block_n=128, splits=4)),
           ("splitk", dict(block_n=64, splits=8)), ("splitk", dict(block_n=128, splits=8))]
name = sys.argv[1]
if name.startswith("sq"):  # sqW[_NN_f32]: a W^3 square (TN FP16 out unless given)
    parts = name[2:].split("_")
    W = int(parts[0])
    lay = parts[1] if len(parts) > 1 else "TN"
    m, n, k, tA, tB, alpha, beta, out = W, W, W, lay[0], lay[1], 1.0, 0.0, parts[2] if len(parts) > 2 else "f16"
else:
    m, n, k, tA, tB, alpha, beta, out = inputs.WORKLOADS[name]
A, lda, B, ldb, C = bench.device_operands(torch.device("cuda:0"), m, n, k, tA, tB, beta, out)
w = torch.empty(64 * 1024 * 1024, device="cuda")
for kern, kw in CONFIGS:
    if kern == "auto":
        binding.set_config()
    else:
        binding.set_config(kern, **kw)
    for _ in range(3):
        w.zero_()
        binding.hgemm(m, n, k, alpha, A, lda, B, ldb, beta, C, m, tA, tB, out)
        torch.cuda.synchronize()
        st = binding.get_stats()
        print(f"{name} {kern}/{'/'.join(str(v) for v in kw.values())} -> {st['last_kernel']}/{st['block_n']}/s{st['splits']}",
              flush=True)
binding.set_config()
f = bench.cublas_fn(A, B, C, tA, tB, alpha, beta)
for _ in range(3):
    w.zero_()
    f()
    torch.cuda.synchronize()
    print(f"{name} cublas", flush=True)
