"""Per-launch cost of kernel features (experiments): event-timed single launches after an
L2 flush (median of 40) and back-to-back launches (mean of 300), for the teardown probe
kernel (csrc/microbench.cu mb_teardown) with and without a cluster attribute, TMEM
allocation, bulk stores in flight at exit and the PDL attribute."""
import ctypes
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import build  # noqa: E402

mb = ctypes.CDLL(build.build_microbench())
mb.mb_teardown.argtypes = [ctypes.c_int] * 6 + [ctypes.c_void_p, ctypes.c_void_p]
w = torch.empty(64 * 1024 * 1024, device="cuda")
g = torch.empty(160 * 16 * 4096, dtype=torch.uint8, device="cuda")
s = torch.cuda.current_stream().cuda_stream


def single(fn, reps=40):
    ts = []
    for _ in range(reps):
        w.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        ts.append((e0, e1))
    torch.cuda.synchronize()
    return statistics.median(a.elapsed_time(b) for a, b in ts) * 1e3


def b2b(fn, reps=300):
    fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / reps * 1e3


for grid, block, smem in ((128, 192, 180 * 1024), (148, 320, 200 * 1024), (4, 320, 200 * 1024)):
    for cl in (0, 1, 2, 4):
        if grid % max(cl, 1):
            continue
        for mode in (0, 1, 2, 3):
            if cl == 4 and mode & 1:
                continue
            for pdl in (0, 1):
                f = lambda: mb.mb_teardown(grid, block, smem, cl, mode, pdl, g.data_ptr(), s)  # noqa: E731
                print(f"grid {grid:3d} smem {smem // 1024}K cluster {cl} tmem {mode & 1} store {(mode >> 1) & 1} "
                      f"pdl {pdl}: single {single(f):6.2f} us  b2b {b2b(f):6.2f} us", flush=True)
