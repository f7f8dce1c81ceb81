"""How many thread-block clusters of each size fit on this GPU at once (227 KB smem per CTA, one
CTA per SM), and which SMs a persistent grid of such clusters lands on (experiments)."""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import build  # noqa: E402

mb = ctypes.CDLL(build.build_microbench())
mb.mb_max_clusters.argtypes = [ctypes.c_int] * 3
for cl in (1, 2, 4, 8, 16):
    n = mb.mb_max_clusters(cl, 200 * 1024, 320)
    print(f"cluster {cl:2d}: max active clusters {n:4d} -> {n * cl if n > 0 else n} SMs busy")
