"""Where the fixed per-launch time goes (experiments): %globaltimer stamp kernels
right before and after one launch (pre -> post), for
  * empty kernels with the GEMM kernels' launch shapes, adding one GEMM feature at a
    time (TMEM alloc/free, bulk stores left in flight at exit, PDL attribute/trigger);
  * hgemm() on small BJ shapes (library knobs from the environment: HGEMM_PDL,
    HGEMM_EXP = 4 wait for store completion / 8 no PDL trigger / 16 no cluster attribute
    for 1-CTA launches);
  * cuBLAS on the same shapes.
Each number is the median of 9 launches, each after a 256 MiB L2 flush.

    python tools/teardown_probe.py [--kernels-only]
"""
import ctypes
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding, build  # noqa: E402

mb = ctypes.CDLL(build.build_microbench())
mb.mb_stamp.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
mb.mb_teardown.argtypes = [ctypes.c_int] * 6 + [ctypes.c_void_p, ctypes.c_void_p]
torch.backends.cuda.matmul.allow_fp16_reduced_precision_reduction = False
w = torch.empty(64 * 1024 * 1024, device="cuda")
st = torch.zeros(2, dtype=torch.int64, device="cuda")
gbuf = torch.empty(160 * 16 * 4096, dtype=torch.uint8, device="cuda")
s = torch.cuda.current_stream().cuda_stream


def stamped(fn, reps=9):
    ts = []
    for _ in range(reps):
        w.zero_()
        mb.mb_stamp(st.data_ptr(), s)
        fn()
        mb.mb_stamp(st.data_ptr() + 8, s)
        torch.cuda.synchronize()
        pre, post = st.tolist()
        ts.append((post - pre) / 1e3)
    return statistics.median(ts)


tag = f"PDL={os.environ.get('HGEMM_PDL', '1')} EXP={os.environ.get('HGEMM_EXP', '0')}"
if "--gemm-only" not in sys.argv:
    for (grid, block, smem, cl) in [(148, 320, 200 * 1024, 2), (4, 320, 200 * 1024, 1), (4, 320, 200 * 1024, 0),
                                    (128, 192, 180 * 1024, 4)]:
        for mode in (0, 1, 2, 3, 7):
            for pdl in (0, 1):
                if cl == 4 and mode & 1:
                    continue
                t = stamped(lambda: mb.mb_teardown(grid, block, smem, cl, mode, pdl, gbuf.data_ptr(), s))
                print(f"empty grid {grid:3d} block {block} smem {smem // 1024}K cluster {cl} mode {mode} "
                      f"(tmem {mode & 1}, bulk store {(mode >> 1) & 1}, trigger {(mode >> 2) & 1}) pdl {pdl}: "
                      f"pre->post {t:6.2f} us", flush=True)
for (m, n, k, beta) in [(256, 256, 256, 0.0), (64, 4096, 2048, 1.0), (4096, 1024, 4096, 1.0), (16384, 64, 4096, 0.0)]:
    A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
    B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
    C = (torch.rand(n, m, device="cuda") * 2 - 1).half()
    t_o = stamped(lambda: binding.hgemm(m, n, k, 1.0, A, k, B, k, beta, C, m, "T", "N", "f16"))
    kern = binding.get_stats()["last_kernel"]
    t_c = stamped(lambda: torch.addmm(C, B, A.t(), beta=beta, out=C) if beta else torch.mm(B, A.t(), out=C))
    print(f"{tag} {m}x{n}x{k} beta={beta}: ours [{kern}] pre->post {t_o:6.2f} us | cuBLAS {t_c:6.2f} us", flush=True)
