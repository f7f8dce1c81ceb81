"""HBM streaming-pattern study for skinny GEMM operands (csrc/microbench.cu
tma_stream_kernel): GB/s of TMA box loads versus row pitch, box rows and
boxes in flight.  128 MiB per run, L2 flushed (write + read) before each."""
import ctypes
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_ipps_00020c20_b200 import build  # noqa: E402

lib = ctypes.CDLL(build.build_microbench())
lib.mb_tma_stream.argtypes = [ctypes.c_void_p] + [ctypes.c_int] * 5 + [ctypes.c_void_p]
SMS = torch.cuda.get_device_properties(0).multi_processor_count
buf = torch.empty(64 * 1024 * 1024, dtype=torch.float16, device="cuda").uniform_(-1, 1)   # 128 MiB
w = torch.empty(64 * 1024 * 1024, device="cuda")
r = torch.zeros(64 * 1024 * 1024, device="cuda")
cyc = torch.zeros(SMS, dtype=torch.int64, device="cuda")


def run(row_len, box_rows, depth, grid=SMS):
    rows = buf.numel() // row_len
    rows -= rows % box_rows
    ts = []
    for i in range(4):
        w.zero_()
        r.sum()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        assert lib.mb_tma_stream(buf.data_ptr(), row_len, rows, box_rows, depth, grid, cyc.data_ptr()) == 0
        e1.record()
        torch.cuda.synchronize()
        if i:
            ts.append(e0.elapsed_time(e1))
    ms = min(ts)
    gbs = rows * row_len * 2 / (ms * 1e-3) / 1e9
    print(f"row_len {row_len:5d} ({row_len * 2:5d} B pitch) box_rows {box_rows:3d} depth {depth:2d} grid {grid:3d}: "
          f"{ms * 1e3:7.1f} us  {gbs:6.0f} GB/s  in flight/SM {depth * box_rows * 128 // 1024} KB", flush=True)


for row_len in (4096, 512, 64):
    for box_rows in (64, 112, 128, 256):
        for depth in (4, 7, 12):
            if depth * box_rows * 128 <= 200 * 1024:
                run(row_len, box_rows, depth)
run(4096, 128, 7, grid=128)
run(4096, 112, 12, grid=74)
