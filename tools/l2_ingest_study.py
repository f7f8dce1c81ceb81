"""Per-SM TMA ingest from L2 (experiments): a 32 MiB FP16 buffer (L2-resident after a warm-up
pass, no flush between passes) streamed by a few CTAs with the microbench TMA stream kernels;
each CTA's clock64 span gives its bytes per SM cycle.  2-D boxes (128 B per row, like the
tile kernel's k-blocks) against 3-D k-group boxes (G x 128 contiguous bytes per row).

    python tools/l2_ingest_study.py
"""
import ctypes
import os
import statistics
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_ipps_00020c20_b200 import build  # noqa: E402

lib = ctypes.CDLL(build.build_microbench())
lib.mb_tma_stream.argtypes = [ctypes.c_void_p] + [ctypes.c_int] * 5 + [ctypes.c_void_p]
lib.mb_tma_stream3d.argtypes = [ctypes.c_void_p] + [ctypes.c_int] * 6 + [ctypes.c_void_p]
ROW_LEN, ROWS = 4096, 4096                      # 32 MiB, 8 KB pitch
buf = torch.empty(ROWS * ROW_LEN, dtype=torch.float16, device="cuda").uniform_(-1, 1)
cyc = torch.zeros(256, dtype=torch.int64, device="cuda")


def measure(label, launch, per_cta_bytes, grid):
    rates = []
    for i in range(4):
        cyc.zero_()
        assert launch() == 0, label
        torch.cuda.synchronize()
        if i:
            c = cyc[:grid].cpu().tolist()
            rates.append(statistics.median(per_cta_bytes / max(x, 1) for x in c))
    print(f"{label:60s} median per-CTA {max(rates):6.1f} B/clk", flush=True)


for grid in (8, 16, 32):
    for box_rows, depth in ((128, 11), (64, 16)):
        bands = ROWS // box_rows
        my = bands // grid
        per = my * (ROW_LEN // 64) * box_rows * 128
        measure(f"2-D box {box_rows} rows x 128 B, depth {depth}, grid {grid}",
                lambda: lib.mb_tma_stream(buf.data_ptr(), ROW_LEN, ROWS, box_rows, depth, grid, cyc.data_ptr()),
                per, grid)
        for g, d in ((2, max(2, depth // 2)), (4, max(2, depth // 4))):
            measure(f"3-D box {box_rows} rows x {g * 128} B (G={g}), depth {d}, grid {grid}",
                    lambda: lib.mb_tma_stream3d(buf.data_ptr(), ROW_LEN, ROWS, box_rows, g, d, grid, cyc.data_ptr()),
                    per, grid)
