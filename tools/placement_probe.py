"""Where the CTAs of a persistent cluster launch land (experiments): %smid per blockIdx for
the GEMM's launch shape (74 clusters of 2, 227 KB smem), repeated to see if it is stable."""
import ctypes
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import build  # noqa: E402

mb = ctypes.CDLL(build.build_microbench())
mb.mb_smid.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p]
out = torch.zeros(148, dtype=torch.int32, device="cuda")
s = torch.cuda.current_stream().cuda_stream
for cl, grid in ((2, 148), (4, 132), (1, 148)):
    for rep in range(3):
        out.fill_(-1)
        rc = mb.mb_smid(grid, cl, 200 * 1024, out.data_ptr(), s)
        torch.cuda.synchronize()
        v = out.cpu().tolist()[:grid]
        print(f"cluster {cl} grid {grid} rep {rep} rc {rc}: smid by blockIdx = {v}", flush=True)
        if cl == 2:
            pairs = [(v[2 * i], v[2 * i + 1]) for i in range(grid // 2)]
            same_tpc = sum(1 for a, b in pairs if a // 2 == b // 2)
            print(f"   pairs on one TPC (smid//2 equal): {same_tpc}/{len(pairs)}; "
                  f"monotonic blockIdx->smid: {all(v[i] <= v[i + 1] for i in range(grid - 1))}")
