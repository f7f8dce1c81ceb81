"""Quick multicast (HGEMM_MC=2) correctness check against torch.mm (experiments)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402

torch.backends.cuda.matmul.allow_fp16_reduced_precision_reduction = False
for (m, n, k, bn) in [(1024, 1024, 512, 512), (1024, 1024, 512, 256), (3000, 2000, 700, 512), (3000, 1300, 700, 256),
                      (8192, 8192, 1024, 512)]:
    for tA, tB in (("T", "N"), ("N", "N"), ("N", "T"), ("T", "T")):
        binding.set_config("tc2", block_n=bn)
        A = (torch.rand(m, k, device="cuda") * 2 - 1).half()   # op(A) m x k
        B = (torch.rand(k, n, device="cuda") * 2 - 1).half()   # op(B) k x n
        ref = (A.float() @ B.float())
        # column-major storage: op(A) 'T' -> stored k x m (= row-major A), 'N' -> stored m x k (= A^T row-major)
        sA = A if tA == "T" else A.t().contiguous()
        lda = k if tA == "T" else m
        sB = B.t().contiguous() if tB == "N" else B
        ldb = k if tB == "N" else n
        C = torch.full((n, m), float("nan"), device="cuda", dtype=torch.float32)
        binding.hgemm(m, n, k, 1.0, sA, lda, sB, ldb, 0.0, C, m, tA, tB, "f32")
        torch.cuda.synchronize()
        err = (C.t() - ref).abs().max().item()
        print(m, n, k, bn, tA + tB, binding.get_stats()["last_kernel"], "max err", err, flush=True)
        assert err < 1e-2, err
print("mc_check ok")
