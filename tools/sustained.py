"""Sustained-regime comparison (power-capped): ours vs cuBLAS on the same operands.

Each implementation runs back-to-back for --warm seconds (reaching the 1 kW
steady state), then --iters launches are timed with CUDA events; NVML power
and the in-kernel SM clock (our clock probe) are sampled.  Prints one line
per implementation: TFLOP/s, power, clock, TFLOP/J.
"""
import argparse
import os
import statistics
import sys
import threading
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--m", type=int, default=8192)
ap.add_argument("--warm", type=float, default=3.0)
ap.add_argument("--iters", type=int, default=200)
ap.add_argument("--order", default="ours,cublas,ours,cublas")
ap.add_argument("--compute", default="f32", help="accumulation type of ours (f16: hgemm_ex FP16 accumulate)")
ap.add_argument("--group-m", type=int, default=0, help="raster group height of ours (0 = library default)")
args = ap.parse_args()
m = n = k = args.m
A = (torch.rand(m, k, device="cuda") * 2 - 1).half()    # op(A) rows, K-major: the paper's TN layout
B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
C = torch.empty(n, m, dtype=torch.half, device="cuda")
torch.backends.cuda.matmul.allow_fp16_reduced_precision_reduction = False
if args.group_m:
    binding.set_config(group_m=args.group_m)


def ours():
    if args.compute == "f16":
        binding.hgemm_ex(m, n, k, 1.0, A, k, B, k, 0.0, C, m, "T", "N", "f16", compute="f16")
    else:
        binding.hgemm(m, n, k, 1.0, A, k, B, k, 0.0, C, m, "T", "N", "f16")


def cublas():
    torch.mm(B, A.t(), out=C)


def power_sampler(stop, out):
    import pynvml
    pynvml.nvmlInit()
    h = pynvml.nvmlDeviceGetHandleByIndex(torch.cuda.current_device())
    while not stop.is_set():
        out.append((pynvml.nvmlDeviceGetPowerUsage(h) / 1000.0, pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)))
        time.sleep(0.02)


for name in args.order.split(","):
    fn = ours if name == "ours" else cublas
    t0 = time.time()
    while time.time() - t0 < args.warm:
        for _ in range(20):
            fn()
        torch.cuda.synchronize()
    samples, stop = [], threading.Event()
    th = threading.Thread(target=power_sampler, args=(stop, samples), daemon=True)
    th.start()
    probe = torch.zeros(4, dtype=torch.int64, device="cuda")
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for i in range(args.iters):
        if name == "ours" and i == args.iters // 2:
            binding.set_probe(probe)
        fn()
        if name == "ours" and i == args.iters // 2:
            binding.set_probe(None)
    e1.record()
    torch.cuda.synchronize()
    stop.set()
    th.join()
    ms = e0.elapsed_time(e1) / args.iters
    tf = 2.0 * m * n * k / (ms * 1e-3) / 1e12
    pw = statistics.median(s[0] for s in samples) if samples else float("nan")
    clk = statistics.median(s[1] for s in samples) if samples else float("nan")
    kclk = binding.probe_clock_ghz(probe) * 1000 if name == "ours" else float("nan")
    print(f"{name:7s} {tf:8.1f} TF/s  {ms:.4f} ms  power {pw:6.1f} W  nvml-clk {clk:6.0f}  kernel-clk {kclk:6.0f}  "
          f"{tf / pw:.3f} TF/J", flush=True)
