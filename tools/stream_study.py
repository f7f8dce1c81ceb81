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
lib.mb_tma_stream3d.argtypes = [ctypes.c_void_p] + [ctypes.c_int] * 6 + [ctypes.c_void_p]
lib.mb_ldg_read.argtypes = [ctypes.c_void_p, ctypes.c_longlong, ctypes.c_int, ctypes.c_int, ctypes.c_void_p]
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


def timed_launch(launch, nbytes, label):
    ts = []
    for i in range(6):
        w.zero_()
        r.sum()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        assert launch() == 0, label
        e1.record()
        torch.cuda.synchronize()
        if i:
            ts.append(e0.elapsed_time(e1))
    ms = min(ts)
    print(f"{label}: {ms * 1e3:7.1f} us  {nbytes / (ms * 1e-3) / 1e9:6.0f} GB/s", flush=True)


def run3d(row_len, box_rows, g, depth, grid=SMS):
    rows = buf.numel() // row_len
    rows -= rows % box_rows
    timed_launch(lambda: lib.mb_tma_stream3d(buf.data_ptr(), row_len, rows, box_rows, g, depth, grid, cyc.data_ptr()),
                 rows * row_len * 2, f"3-D row_len {row_len:5d} box_rows {box_rows:3d} G {g} depth {depth:2d} grid {grid:3d} "
                 f"(in flight/SM {depth * box_rows * 128 * g // 1024} KB)")


def ldg(grid, block):
    timed_launch(lambda: lib.mb_ldg_read(buf.data_ptr(), buf.numel() * 2, grid, block, cyc.data_ptr()),
                 buf.numel() * 2, f"ldg.v4 x8 grid {grid:4d} block {block}")


def torch_read():
    """End-to-end read rate of a torch reduction over the same 128 MiB (ld.global path)."""
    ts = []
    for i in range(6):
        w.zero_()
        r.sum()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        buf.sum()
        e1.record()
        torch.cuda.synchronize()
        if i:
            ts.append(e0.elapsed_time(e1))
    ms = min(ts)
    print(f"torch buf.sum() over 128 MiB: {ms * 1e3:7.1f} us  {buf.numel() * 2 / (ms * 1e-3) / 1e9:6.0f} GB/s", flush=True)


torch_read()
if "--3d" in sys.argv:
    for grid, block in ((SMS, 512), (2 * SMS, 512), (4 * SMS, 256), (8 * SMS, 256)):
        ldg(grid, block)
    for row_len, box_rows in ((4096, 112), (4096, 128), (2048, 128), (2048, 32), (2048, 64)):
        run(row_len, box_rows, max(2, min(16, 180 * 1024 // (box_rows * 128))))
        for g in (2, 4, 8):
            depth = 180 * 1024 // (box_rows * 128 * g)
            if depth >= 2:
                run3d(row_len, box_rows, g, depth)
    sys.exit(0)
if "--quick" in sys.argv:
    for box_rows, depth, grid in ((112, 12, SMS), (128, 12, SMS), (128, 12, 128), (64, 24, SMS), (256, 6, SMS)):
        run(4096, box_rows, depth, grid)
    sys.exit(0)
for row_len in (4096, 512, 64):
    for box_rows in (64, 112, 128, 256):
        for depth in (4, 7, 12):
            if depth * box_rows * 128 <= 200 * 1024:
                run(row_len, box_rows, depth)
run(4096, 128, 7, grid=128)
run(4096, 112, 12, grid=74)
