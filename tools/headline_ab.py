"""Headline step-time distribution, ours vs cuBLAS interleaved (experiments).

8192^3 TN FP16 out, the bench protocol (256 MiB write + read flush before each step,
outside the CUDA events), in alternating blocks of --block steps (ours, cuBLAS, ours, ...)
so that both see the same thermal / power-cap history.  NVML power and SM clock are
sampled in a thread.  Prints per block: mean / median / max step ms and the number of
slow steps (> 1.1 x the block median), then the totals.

    python tools/headline_ab.py [--blocks 6] [--block 50] [--group-m G] [--variants a,b]
"""
import argparse
import os
import statistics
import sys
import threading
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--blocks", type=int, default=6)
ap.add_argument("--block", type=int, default=50)
ap.add_argument("--m", type=int, default=8192)
ap.add_argument("--variants", default="ours,cublas", help="comma list: ours, cublas, ours:gm=G, ours:bn=256")
args = ap.parse_args()

dev = torch.device("cuda:0")
m = n = k = args.m
A, lda, B, ldb, C = bench.device_operands(dev, m, n, k, "T", "N", 0.0, "f16")
w = torch.empty(64 * 1024 * 1024, device=dev)
r = torch.empty(64 * 1024 * 1024, device=dev)


def flush():
    w.fill_(1.0)
    r.sum()


def ours_fn(gm=0, bn=0):
    def f():
        binding.hgemm(m, n, k, 1.0, A, lda, B, ldb, 0.0, C, m, "T", "N", "f16")
    return f, (gm, bn)


variants = []
for v in args.variants.split(","):
    if v == "cublas":
        variants.append((v, bench.cublas_fn(A, B, C, "T", "N", 1.0, 0.0), None))
    else:
        kv = dict(x.split("=") for x in v.split(":")[1:])
        variants.append((v, ours_fn()[0], (int(kv.get("gm", 0)), int(kv.get("bn", 0)))))

samples = []
stop = False


def sampler():
    try:
        import pynvml
        pynvml.nvmlInit()
        h = pynvml.nvmlDeviceGetHandleByIndex(0)
        while not stop:
            samples.append((time.time(), pynvml.nvmlDeviceGetPowerUsage(h) / 1e3,
                            pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM),
                            pynvml.nvmlDeviceGetTemperature(h, pynvml.NVML_TEMPERATURE_GPU)))
            time.sleep(0.02)
    except Exception as e:  # noqa: BLE001
        print("nvml:", e)


th = threading.Thread(target=sampler, daemon=True)
th.start()
tot = {v[0]: [] for v in variants}
for name, fn, cfg in variants:   # warm-up of every variant
    if cfg is not None:
        binding.set_config("auto" if cfg[1] == 0 else "tc2", block_n=cfg[1], group_m=cfg[0])
    bench.timed(fn, flush, 5, 1)
for b in range(args.blocks):
    for name, fn, cfg in variants:
        if cfg is not None:
            binding.set_config("auto" if cfg[1] == 0 else "tc2", block_n=cfg[1], group_m=cfg[0])
        t0 = time.time()
        evs = []
        for _ in range(args.block):
            flush()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            fn()
            e1.record()
            evs.append((e0, e1))
        torch.cuda.synchronize()
        t1 = time.time()
        ts = [a.elapsed_time(c) for a, c in evs]
        tot[name] += ts
        med = statistics.median(ts)
        slow = sum(t > 1.1 * med for t in ts)
        sm = [s for s in samples if t0 <= s[0] <= t1]
        pw = statistics.median(s[1] for s in sm) if sm else float("nan")
        ck = statistics.median(s[2] for s in sm) if sm else float("nan")
        tp = max(s[3] for s in sm) if sm else float("nan")
        print(f"block {b} {name:14s} mean {statistics.mean(ts):.4f} med {med:.4f} max {max(ts):.4f} ms  "
              f"slow {slow:2d}  TF(mean) {2 * m * n * k / statistics.mean(ts) / 1e9:7.1f}  "
              f"power {pw:6.1f} W  sm {ck:6.0f} MHz  temp {tp} C", flush=True)
stop = True
binding.set_config()
for name, ts in tot.items():
    print(f"TOTAL {name:14s} mean {statistics.mean(ts):.4f} med {statistics.median(ts):.4f} "
          f"TF(mean) {2 * m * n * k / statistics.mean(ts) / 1e9:7.1f} TF(med) "
          f"{2 * m * n * k / statistics.median(ts) / 1e9:7.1f}")
