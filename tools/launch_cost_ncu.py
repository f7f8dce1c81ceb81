"""Device-side fixed cost of a launch shape, for ncu (experiments).

Launches empty / teardown-probe kernels of several shapes (grid, block, dynamic smem,
cluster, TMEM alloc, bulk stores at exit), each after a 256 MiB L2 flush, then the
small BJ GEMM shapes (ours and cuBLAS).  Run it under
    ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file X.csv \
        python tools/launch_cost_ncu.py > order.txt
and join X.csv (kernel IDs in launch order, flush kernels filtered by name) with the
printed order (tools/launch_cost_join.py).  gpu__time_duration has ns resolution, unlike
the %globaltimer stamps of tools/teardown_probe.py (1-2 us steps on this part).
"""
import ctypes
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding, build  # noqa: E402

mb = ctypes.CDLL(build.build_microbench())
mb.mb_empty.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p]
mb.mb_teardown.argtypes = [ctypes.c_int] * 6 + [ctypes.c_void_p, ctypes.c_void_p]
torch.backends.cuda.matmul.allow_fp16_reduced_precision_reduction = False
w = torch.empty(64 * 1024 * 1024, device="cuda")
gbuf = torch.empty(160 * 16 * 4096, dtype=torch.uint8, device="cuda")
s = torch.cuda.current_stream().cuda_stream
REPS = 3


def run(tag, fn):
    for _ in range(REPS):
        w.zero_()
        fn()
        print(tag, flush=True)
    torch.cuda.synchronize()


GEMM_ONLY = "--gemm-only" in sys.argv
for (grid, block, smem, cl) in [] if GEMM_ONLY else [(4, 128, 0, 1), (4, 320, 0, 1), (4, 320, 48 * 1024, 1), (4, 320, 100 * 1024, 1),
                                (4, 320, 150 * 1024, 1), (4, 320, 232448, 1), (4, 320, 232448, 2),
                                (148, 320, 0, 1), (148, 320, 232448, 1), (148, 320, 0, 2), (148, 320, 232448, 2),
                                (148, 192, 232448, 1), (128, 192, 232448, 4), (128, 192, 100 * 1024, 4)]:
    run(f"empty grid={grid} block={block} smem={smem} cluster={cl}",
        lambda: mb.mb_empty(grid, block, smem, cl, None, s))
for (grid, block, smem, cl) in [] if GEMM_ONLY else [(4, 320, 200 * 1024, 0), (148, 320, 200 * 1024, 2)]:
    for mode in (0, 1, 2, 3):
        for pdl in (0, 1):
            run(f"teardown grid={grid} block={block} smem={smem} cluster={cl} tmem={mode & 1} "
                f"bulkst={(mode >> 1) & 1} pdl={pdl}",
                lambda: mb.mb_teardown(grid, block, smem, cl, mode, pdl, gbuf.data_ptr(), s))
for (m, n, k, beta) in [(256, 256, 256, 0.0), (64, 4096, 2048, 1.0), (256, 4096, 2048, 1.0),
                        (4096, 1024, 4096, 1.0), (1024, 4096, 2048, 1.0), (2048, 2048, 2048, 0.0),
                        (16384, 64, 4096, 0.0), (8192, 8192, 8192, 0.0)]:
    A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
    B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
    C = (torch.rand(n, m, device="cuda") * 2 - 1).half()
    torch.cuda.synchronize()
    run(f"ours {m}x{n}x{k} beta={beta}", lambda: binding.hgemm(m, n, k, 1.0, A, k, B, k, beta, C, m, "T", "N", "f16"))
    run(f"cublas {m}x{n}x{k} beta={beta}",
        lambda: torch.addmm(C, B, A.t(), beta=beta, out=C) if beta else torch.mm(B, A.t(), out=C))
