"""Measure every tensor-core tile configuration on square sizes (calibrates choose_tc)."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402

# sizes: "W" (square) or "MxNxK" tokens, comma separated
toks = sys.argv[1].split(",") if len(sys.argv) > 1 else ["1536", "1792", "2048", "2304", "2560", "2816", "3072",
                                                          "3584", "4096"]
shapes = [tuple(int(v) for v in t.split("x")) if "x" in t else (int(t),) * 3 for t in toks]
# (kernel, block_n, stream_k): stream_k 1 = whole tiles only, 2 = forced stream-K
cfgs = [("tc2", 512, 1), ("tc2", 256, 1), ("tc2", 256, 2), ("tc1", 256, 1), ("tc1", 256, 2), ("tc1", 128, 1),
        ("tc1", 128, 2), ("auto", 0, 0)]
for m, n, k in shapes:
    W = f"{m}x{n}x{k}"
    A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
    B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
    C = torch.empty(n, m, dtype=torch.half, device="cuda")
    row = {"W": W}
    for kern, bn, sk in cfgs:
        binding.set_config(kern, block_n=bn, stream_k=sk) if kern != "auto" else binding.set_config()
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
        row[f"{kern}/{bn}" + ("sk" if sk == 2 else "")] = round(2.0 * m * n * k / ms / 1e9, 1)
        if kern == "auto":
            st = binding.get_stats()
            row["auto_kernel"] = f"{st['last_kernel']}/{st['block_n']}" + ("sk" if st["stream_k"] == 2 else "")
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
