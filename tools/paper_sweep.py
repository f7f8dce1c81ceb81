"""The paper's evaluation sweep (PAPER.md SVII) on B200: ours vs cuBLAS.

Square W x W x W, W = 1024 ... 16384 step 256, and the six
rectangular shapes [2W x W x W], [W x 2W x W], [W x W x 2W], [4W x W x W],
[W x 4W x W], [W x W x 4W], where [m x n x k] follows the
paper's notation (A m x k row-major, B n x k: the TN layout of the ABI).
FP16 in / FP16 out, alpha = 1, beta = 0.  Each point: 3 warm-up runs, then
the average of 10 runs timed with CUDA events (the paper's method),
ours and cuBLAS (torch.mm, FP32 accumulation) alternating at every point.

    python tools/paper_sweep.py [--square-step 256] [--rect-step 256] [--out gpurun_out/sweep.jsonl]
                                [--md gpurun_out/sweep.md]
"""
import argparse
import json
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--square-step", type=int, default=256)
ap.add_argument("--rect-step", type=int, default=256)
ap.add_argument("--md", default=None, help="also write a markdown summary (per-shape mean / geomean / min)")
ap.add_argument("--wmax", type=int, default=16384)
ap.add_argument("--iters", type=int, default=10)
ap.add_argument("--out", default="gpurun_out/paper_sweep.jsonl")
args = ap.parse_args()
torch.backends.cuda.matmul.allow_fp16_reduced_precision_reduction = False
dev = torch.device("cuda")


def timed(fn, iters):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(iters):
        fn()
    e1.record()
    torch.cuda.synchronize()
    return e0.elapsed_time(e1) / iters


def point(shape, m, n, k):
    g = torch.Generator(device=dev).manual_seed(m * 7 + n * 3 + k)
    A = (torch.rand(m, k, generator=g, device=dev) * 2 - 1).half()   # row-major A (m x k): ABI op(A) via 'T'
    B = (torch.rand(n, k, generator=g, device=dev) * 2 - 1).half()   # B n x k (paper notation)
    C = torch.empty(n, m, dtype=torch.half, device=dev)              # column-major C (m x n)

    def ours():
        binding.hgemm(m, n, k, 1.0, A, k, B, k, 0.0, C, m, "T", "N", "f16")

    def cub():
        torch.mm(B, A.t(), out=C)

    t_o = timed(ours, args.iters)
    t_c = timed(cub, args.iters)
    fl = 2.0 * m * n * k
    rec = {"shape": shape, "m": m, "n": n, "k": k, "ours_tflops": fl / t_o / 1e9, "cublas_tflops": fl / t_c / 1e9,
           "speedup": t_c / t_o, "kernel": binding.get_stats()["last_kernel"] + "/" +
           str(binding.get_stats()["block_n"])}
    del A, B, C
    return rec


def main():
    os.makedirs(os.path.dirname(args.out) or ".", exist_ok=True)
    recs = []
    with open(args.out, "w") as f:
        for W in range(1024, args.wmax + 1, args.square_step):
            r = point("WxWxW", W, W, W)
            recs.append(r)
            f.write(json.dumps(r) + "\n")
            f.flush()
            print(f"{r['shape']:8s} W={W:6d} ours {r['ours_tflops']:8.1f} cublas {r['cublas_tflops']:8.1f} "
                  f"x{r['speedup']:.3f} {r['kernel']}", flush=True)
        shapes = [("2WxWxW", 2, 1, 1), ("Wx2WxW", 1, 2, 1), ("WxWx2W", 1, 1, 2),
                  ("4WxWxW", 4, 1, 1), ("Wx4WxW", 1, 4, 1), ("WxWx4W", 1, 1, 4)]
        for W in range(1024, args.wmax + 1, args.rect_step):
            for name, a, b, c in shapes:
                r = point(name, a * W, b * W, c * W)
                r["W"] = W
                recs.append(r)
                f.write(json.dumps(r) + "\n")
                f.flush()
                print(f"{name:8s} W={W:6d} ours {r['ours_tflops']:8.1f} cublas {r['cublas_tflops']:8.1f} "
                      f"x{r['speedup']:.3f} {r['kernel']}", flush=True)
    sq = [r["speedup"] for r in recs if r["shape"] == "WxWxW"]
    rect = [r["speedup"] for r in recs if r["shape"] != "WxWxW"]
    print(f"square: mean speedup over cuBLAS {statistics.mean(sq):.3f} (min {min(sq):.3f}, max {max(sq):.3f}); "
          f"rectangular: mean {statistics.mean(rect):.3f} (min {min(rect):.3f}, max {max(rect):.3f})")
    if args.md:
        write_md(recs, args.md)


def write_md(recs, path):
    order = ["WxWxW", "2WxWxW", "Wx2WxW", "WxWx2W", "4WxWxW", "Wx4WxW", "WxWx4W"]
    lines = ["| shape | points | mean ours/cuBLAS | geomean | min (W) | max (W) | mean ours TFLOP/s | mean cuBLAS TFLOP/s |",
             "|---|---|---|---|---|---|---|---|"]
    for sh in order:
        rs = [r for r in recs if r["shape"] == sh]
        if not rs:
            continue
        sp = [r["speedup"] for r in rs]
        lo = min(rs, key=lambda r: r["speedup"])
        hi = max(rs, key=lambda r: r["speedup"])
        wkey = lambda r: r.get("W", r["m"])  # noqa: E731
        lines.append(f"| {sh} | {len(rs)} | {statistics.mean(sp):.3f} | {statistics.geometric_mean(sp):.3f} | "
                     f"{lo['speedup']:.3f} ({wkey(lo)}) | {hi['speedup']:.3f} ({wkey(hi)}) | "
                     f"{statistics.mean(r['ours_tflops'] for r in rs):.1f} | "
                     f"{statistics.mean(r['cublas_tflops'] for r in rs):.1f} |")
    allsp = [r["speedup"] for r in recs]
    lines.append(f"| all | {len(allsp)} | {statistics.mean(allsp):.3f} | {statistics.geometric_mean(allsp):.3f} | "
                 f"{min(allsp):.3f} | {max(allsp):.3f} | | |")
    lines += ["", "| shape | W | m | n | k | ours TFLOP/s | cuBLAS TFLOP/s | ours/cuBLAS | our kernel |",
              "|---|---|---|---|---|---|---|---|---|"]
    for r in recs:
        lines.append(f"| {r['shape']} | {r.get('W', r['m'])} | {r['m']} | {r['n']} | {r['k']} | "
                     f"{r['ours_tflops']:.1f} | {r['cublas_tflops']:.1f} | {r['speedup']:.3f} | {r['kernel']} |")
    with open(path, "w") as f:
        f.write("\n".join(lines) + "\n")


if __name__ == "__main__":
    main()
