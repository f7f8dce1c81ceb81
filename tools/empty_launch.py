"""Fixed cost of a launch shape: %globaltimer stamps around an empty kernel (experiments).

    python tools/empty_launch.py
"""
import ctypes
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import build  # noqa: E402

mb = ctypes.CDLL(build.build_microbench())
mb.mb_stamp.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
mb.mb_empty.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p]
w = torch.empty(64 * 1024 * 1024, device="cuda")
st = torch.zeros(2, dtype=torch.int64, device="cuda")
s = torch.cuda.current_stream().cuda_stream
for (grid, block, smem, cl) in [(148, 320, 232448, 2), (148, 320, 200 * 1024, 2), (148, 320, 150 * 1024, 2),
                                (148, 320, 100 * 1024, 2), (148, 320, 48 * 1024, 2), (148, 320, 0, 2),
                                (148, 320, 232448, 1), (148, 320, 0, 1), (74, 320, 232448, 2), (148, 192, 232448, 1),
                                (128, 192, 232448, 4), (148, 256, 218400, 4)]:
    res = []
    for flush in (True, False):
        ts = []
        for i in range(6):
            if flush:
                w.zero_()
            else:
                torch.cuda._sleep(200000)          # keep the GPU busy while the host enqueues
            mb.mb_stamp(st.data_ptr(), s)
            rc = mb.mb_empty(grid, block, smem, cl, None, s)
            mb.mb_stamp(st.data_ptr() + 8, s)
            torch.cuda.synchronize()
            pre, post = st.tolist()
            ts.append((post - pre) / 1e3)
        res.append(sorted(ts)[len(ts) // 2])
    print(f"grid {grid:3d} block {block} smem {smem:6d} cluster {cl}: rc {rc} stamp-to-stamp after flush {res[0]:5.2f} us, "
          f"after sleep {res[1]:5.2f} us", flush=True)
for i in range(3):
    mb.mb_stamp(st.data_ptr(), s)
    mb.mb_stamp(st.data_ptr() + 8, s)
torch.cuda.synchronize()
pre, post = st.tolist()
print(f"stamp -> stamp (nothing between): {(post - pre) / 1e3:.2f} us")
