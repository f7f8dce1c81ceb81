"""Measure every tensor-core tile configuration on square sizes (calibrates choose_tc)."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402

sizes = [int(x) for x in sys.argv[1].split(",")] if len(sys.argv) > 1 else [1536, 1792, 2048, 2304, 2560, 2816, 3072, 3584, 4096]
cfgs = [("tc2", 512), ("tc2", 256), ("tc1", 256), ("tc1", 128), ("auto", 0)]
res = []
for W in sizes:
    m = n = k = W
    A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
    B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
    C = torch.empty(n, m, dtype=torch.half, device="cuda")
    row = {"W": W}
    for kern, bn in cfgs:
        binding.set_config(kern, block_n=bn) if kern != "auto" else binding.set_config()
        for _ in range(3):
            binding.hgemm(m, n, k, 1.0, A, k, B, k, 0.0, C, m, "T", "N", "f16")
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(20):
            binding.hgemm(m, n, k, 1.0, A, k, B, k, 0.0, C, m, "T", "N", "f16")
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 20
        row[f"{kern}/{bn}"] = round(2.0 * m * n * k / ms / 1e9, 1)
        if kern == "auto":
            row["auto_kernel"] = binding.get_stats()["last_kernel"] + "/" + str(binding.get_stats()["block_n"])
    binding.set_config()
    torch.mm(B, A.t(), out=C)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(20):
        torch.mm(B, A.t(), out=C)
    e1.record()
    torch.cuda.synchronize()
    row["cublas"] = round(2.0 * m * n * k / (e0.elapsed_time(e1) / 20) / 1e9, 1)
    print(json.dumps(row), flush=True)
