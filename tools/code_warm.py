"""Cold instruction fetch probe: how much of a small launch's time is fetching
the kernel's code from DRAM after the L2 flush?

For each shape: event-timed launches after the bench's L2 flush (A), and the
same with a tiny launch of the SAME kernel instantiation between the flush and
the timed launch (B: code in L2, operands still cold).  A - B ~ the cost of
the cold code fetch.  Mean of N launches (the event clock ticks in ~2 us steps).

    python tools/code_warm.py
"""
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402

w = torch.empty(64 * 1024 * 1024, device="cuda")
r = torch.zeros(64 * 1024 * 1024, device="cuda")
REPS = 60


def run(label, m, n, k, tA, tB, beta, out, force=None):
    def mk(rows, cols):
        return (torch.rand(rows, cols, device="cuda") * 2 - 1).half()
    # column-major operands (stored a_rows x a_cols, lda = a_rows) as torch row-major a_cols x a_rows
    a_rows = k if tA == "T" else m
    a_cols = m if tA == "T" else k
    b_rows = n if tB == "T" else k
    b_cols = k if tB == "T" else n
    A = mk(a_cols, a_rows)  # column-major a_rows x a_cols == row-major a_cols x a_rows
    B = mk(b_cols, b_rows)
    C = torch.zeros(n, m, device="cuda", dtype=torch.float32 if out == "f32" else torch.float16)
    small = (128, 128, 64)
    sa_rows = small[2] if tA == "T" else small[0]
    sa_cols = small[0] if tA == "T" else small[2]
    sb_rows = small[1] if tB == "T" else small[2]
    sb_cols = small[2] if tB == "T" else small[1]
    As = mk(sa_cols, sa_rows)
    Bs = mk(sb_cols, sb_rows)
    Cs = torch.zeros(small[1], small[0], device="cuda", dtype=C.dtype)

    def call():
        binding.hgemm(m, n, k, 1.0, A, a_rows, B, b_rows, beta, C, m, tA, tB, out)

    def warm():
        binding.hgemm(small[0], small[1], small[2], 1.0, As, sa_rows, Bs, sb_rows, beta, Cs, small[0], tA, tB, out)

    if force:
        binding.set_config(*force[0], **force[1])
    call()
    st = binding.get_stats()
    kern = (st["last_kernel"], st["block_n"])
    warm()
    st2 = binding.get_stats()
    same = (st2["last_kernel"], st2["block_n"]) == kern
    res = {}
    for mode in ("cold", "warm"):
        ts = []
        for i in range(REPS + 3):
            w.zero_()
            r.sum()
            if mode == "warm":
                warm()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            call()
            e1.record()
            if i >= 3:
                ts.append((e0, e1))
        torch.cuda.synchronize()
        res[mode] = statistics.mean(a.elapsed_time(b) * 1e3 for a, b in ts)
    binding.set_config()
    print(f"{label:28s} kernel {kern[0]}/{kern[1]} (warm-up launch same kernel: {same}): "
          f"cold code {res['cold']:6.2f} us  code in L2 {res['warm']:6.2f} us  diff {res['cold'] - res['warm']:5.2f} us",
          flush=True)


for rep in range(2):
    run("256^3 NN f32", 256, 256, 256, "N", "N", 0.0, "f32", force=(("tc1",), {"block_n": 128}))
    run("BERT FFN2 4096x1024x4096", 4096, 1024, 4096, "T", "N", 1.0, "f16", force=(("tc2",), {"block_n": 256}))
    run("LSTM-1024 1024x4096x2048", 1024, 4096, 2048, "T", "N", 1.0, "f16", force=(("tc2",), {"block_n": 256}))
    run("LSTM b64 64x4096x2048", 64, 4096, 2048, "T", "N", 1.0, "f16", force=(("splitk",), {"block_n": 64, "splits": 4}))
    run("skinny 16384x64x4096", 16384, 64, 4096, "T", "N", 0.0, "f16", force=(("stream",), {"block_n": 112}))
