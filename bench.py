#!/usr/bin/env python
"""Benchmark: HGEMM TFLOP/s at M=N=K=8192 on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload NAME] [--impl ours|reference]

One "step" = one hgemm() call (the whole hot path: TMA staging, tcgen05 MMA
into TMEM, alpha/beta epilogue) over one batch of synthetic input.
  N = 1 : the metric configuration, C(8192x8192) = A^T B, FP16 in, FP32
          accumulate, FP16 out (BASELINE.json configs[1], paper layout TN).
  N > 1 : torchrun, one rank per GPU; weak scaling: each rank owns one
          8192-column slab of C (global n = 8192*N) and A is replicated by
          an NCCL broadcast (timed and reported separately, "collective").
Timing: W untimed warm-up steps, then K steps, each bracketed by CUDA events
on the launching stream; L2 is flushed (a 256 MiB write + a 256 MiB read) between steps,
outside the events; a barrier + synchronize bracket the timed region; the
time is the max over ranks.  Rank 0 prints ONE JSON line.

--impl reference runs the CPU oracle (oracle/, the correctness reference;
there is no runnable reference implementation of the paper) on the host
cores, on a bounded sample of the same workload, and prints the same JSON
line with "impl": "reference".
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "HGEMM TFLOP/s at M=N=K=8192 and % of B200 dense FP16 peak; 1/2/4/8-GPU"
UNIT = "TFLOP/s"


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return {"tflops_burst": d["bf16_tflops"], "tflops_sustained": d.get("bf16_tflops_sustained"),
                "hbm_gbs": d["hbm_gbs"], "source": "measured (MEASURED_PEAKS.json; fp16 = bf16 x 1.0 nominal ratio)"}
    return {"tflops_burst": 1590.0, "tflops_sustained": 1400.0, "hbm_gbs": 6650.0,
            "source": "fallback (B200_PROFILING.md)"}


def load_traffic(workload):
    p = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d.get(workload)
    return None


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """Samples SM clock and throttle reasons during the timed region (NVML).

    NVML is initialised and sampled once in start(), before the timed region
    begins, and once more in stop(), so even a region shorter than the sampling
    period carries samples taken around and inside it."""

    def __init__(self, index=0):
        self.index = index
        self.samples = []
        self._stop = threading.Event()
        self._t = None
        self._h = None

    def _sample(self):
        import pynvml
        h = self._h
        sm = pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)
        try:
            rs = pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)
        except Exception:
            rs = pynvml.nvmlDeviceGetCurrentClocksThrottleReasons(h)
        self.samples.append((sm, self._max, [k for k, v in self._names.items() if rs & v]))

    def _loop(self):
        try:
            while not self._stop.wait(0.005):
                self._sample()
        except Exception as e:  # pragma: no cover
            self.samples.append((None, None, [f"nvml-error:{type(e).__name__}"]))

    def start(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            self._h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            self._max = pynvml.nvmlDeviceGetMaxClockInfo(self._h, pynvml.NVML_CLOCK_SM)
            self._names = {
                "hw_slowdown": getattr(pynvml, "nvmlClocksEventReasonHwSlowdown", 0x8),
                "hw_thermal_slowdown": getattr(pynvml, "nvmlClocksEventReasonHwThermalSlowdown", 0x40),
                "sw_thermal_slowdown": getattr(pynvml, "nvmlClocksEventReasonSwThermalSlowdown", 0x20),
                "sw_power_cap": getattr(pynvml, "nvmlClocksEventReasonSwPowerCap", 0x4),
                "hw_power_brake_slowdown": getattr(pynvml, "nvmlClocksEventReasonHwPowerBrakeSlowdown", 0x80),
            }
            self._sample()
        except Exception as e:  # pragma: no cover
            self.samples.append((None, None, [f"nvml-error:{type(e).__name__}"]))
            return
        self._t = threading.Thread(target=self._loop, daemon=True)
        self._t.start()

    def stop(self):
        self._stop.set()
        if self._t:
            self._t.join(timeout=2)
            try:
                self._sample()
            except Exception:  # pragma: no cover
                pass
        sm = [s[0] for s in self.samples if s[0]]
        reasons = sorted({r for s in self.samples for r in s[2]})
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max((s[1] for s in self.samples if s[1]), default=None),
                "reasons": reasons, "samples": len(self.samples)}


# ------------------------------------------------------------------ distributed
def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return world, rank, local


def max_over_ranks(x, world, op="max"):
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor([x], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX if op == "max" else dist.ReduceOp.MIN)
    return float(t.item())


def min_over_ranks(x, world):
    return max_over_ranks(x, world, op="min")


# ------------------------------------------------------------------ reference arm (oracle)
def _oracle_block(workload, ms, ns):
    """Seeded ms x k op(A) and k x ns op(B) of the workload's shape family, stored with its flags."""
    from paper_conf_ipps_00020c20_b200 import inputs
    m, n, k, tA, tB, alpha, beta, out = inputs.WORKLOADS[workload]
    opA = inputs.uniform_f16(ms, k, 1)
    opB = inputs.uniform_f16(k, ns, 2)
    A, lda = inputs.store_op(opA, tA)
    B, ldb = inputs.store_op(opB, tB)
    C = inputs.uniform_f16(ms, ns, 3).reshape(-1, order="F") if beta != 0 else None
    if C is not None and out == "f32":
        C = C.astype("float32")
    return (ms, ns, k, alpha, A, lda, B, ldb, beta, C, ms, tA, tB, out)


def _time_oracle(workload, ms, ns, threads):
    import oracle
    args = _oracle_block(workload, ms, ns)
    t0 = time.perf_counter()
    oracle.hgemm_ref(*args, nthreads=threads, want_r=False)
    return time.perf_counter() - t0


def _oracle_sample_size(workload, threads, budget_s):
    """Grow an ms x ns block (full k) until one oracle call takes about budget_s."""
    from paper_conf_ipps_00020c20_b200 import inputs
    m, n, k = inputs.WORKLOADS[workload][:3]
    ms, ns = min(m, 64), min(n, 64)
    _time_oracle(workload, ms, ns, threads)                  # warm the threads / page in
    for _ in range(4):
        dt = _time_oracle(workload, ms, ns, threads)
        if dt >= 0.5 * budget_s or (ms == m and ns == n):
            break
        f = min(8.0, (budget_s / max(dt, 1e-3)) ** 0.5)
        ms, ns = max(1, min(m, int(ms * f))), max(1, min(n, int(ns * f)))
    return ms, ns


def run_reference(args, world, rank):
    """The oracle (the only runnable reference here) on the host cores, on a bounded
    block of the workload per step; rank 0 only."""
    if rank != 0:
        return 0
    import oracle
    from paper_conf_ipps_00020c20_b200 import inputs
    oracle.build()
    m, n, k, tA, tB, alpha, beta, out = inputs.WORKLOADS[args.workload]
    threads = oracle.max_threads()
    per_step = max(1.0, args.ref_budget / max(1, args.warmup + args.steps))
    ms, ns = _oracle_sample_size(args.workload, threads, per_step)
    times = []
    for s in range(args.warmup + args.steps):
        dt = _time_oracle(args.workload, ms, ns, threads)
        if s >= args.warmup:
            times.append(dt)
    flops = 2.0 * ms * ns * k
    ms_step = 1e3 * statistics.mean(times)
    val = flops / (ms_step * 1e-3) / 1e12
    sample = (f"{ms} x {ns} block of C (full k = {k}, layout {tA}{tB}, FP64 oracle) of the {m}x{n}x{k} "
              f"workload per step")
    line = {"metric": METRIC, "value": val, "unit": UNIT, "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True,
            "scaling": "strong" if args.workload in inputs.STRONG_SCALING else "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic", "impl": "reference",
            "config": {"workload": args.workload, "m": m, "n": n, "k": k, "layout": tA + tB, "out": out},
            "cpu_baseline": {"value": val, "unit": UNIT, "cores": threads, "kind": "oracle", "sample": sample,
                             "host": host_info()},
            "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def host_info():
    """The host the oracle ran on: nproc, CPUs in this process's affinity mask, CPU model."""
    model = None
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:  # pragma: no cover
        pass
    try:
        aff = len(os.sched_getaffinity(0))
    except AttributeError:  # pragma: no cover
        aff = None
    return {"nproc": os.cpu_count(), "affinity_cpus": aff, "cpu_model": model}


def cpu_baseline(workload, budget_s=12.0):
    """The oracle, as it stands, on the host cores over a bounded block of the workload:
    all cores (OpenMP over output columns; the reported value) and one thread."""
    import oracle
    from paper_conf_ipps_00020c20_b200 import inputs
    oracle.build()
    k = inputs.WORKLOADS[workload][2]
    threads = oracle.max_threads()
    ms, ns = _oracle_sample_size(workload, threads, budget_s)
    dt = _time_oracle(workload, ms, ns, threads)
    ms1, ns1 = _oracle_sample_size(workload, 1, budget_s / 2)
    dt1 = _time_oracle(workload, ms1, ns1, 1)
    return {"value": 2.0 * ms * ns * k / dt / 1e12, "unit": UNIT, "cores": threads, "kind": "oracle",
            "sample": f"{ms} x {ns} block of C with the full k = {k} of {workload} ({dt:.1f} s)",
            "single_thread": {"value": 2.0 * ms1 * ns1 * k / dt1 / 1e12, "unit": UNIT, "cores": 1,
                              "sample": f"{ms1} x {ns1} block of C, full k ({dt1:.1f} s)"},
            "host": host_info()}


# ------------------------------------------------------------------ L2 flush
class L2Flush:
    """Cold-L2 state between timed launches, outside the events: write a 256 MiB buffer
    (2x the 126 MB L2), then read a second 256 MiB buffer so that the dirty lines of the
    write are written back here rather than inside the next timed launch (the L2 is
    left holding clean, unrelated lines)."""

    def __init__(self, dev):
        import torch
        self.w = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
        self.r = torch.zeros(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
        self.sink = torch.empty((), dtype=torch.float32, device=dev)

    def __call__(self):
        import torch
        self.w.zero_()
        torch.sum(self.r, dim=0, out=self.sink)


# ------------------------------------------------------------------ timing helpers
def timed(fn, flush, warmup, steps, stream=None):
    """W warm-up calls, then `steps` calls each bracketed by CUDA events on `stream`
    (default: torch's current stream) with an L2 flush before each, outside the events."""
    import torch
    for _ in range(warmup):
        flush()
        fn()
    torch.cuda.synchronize()
    evs = []
    for _ in range(steps):
        flush()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        fn()
        e1.record(stream)
        evs.append((e0, e1))
    torch.cuda.synchronize()
    ts = [a.elapsed_time(b) for a, b in evs]
    return {"mean": statistics.mean(ts), "median": statistics.median(ts), "min": min(ts), "max": max(ts),
            "n": len(ts)}


def device_operands(dev, m, n, k, tA, tB, beta, out, seed=1234, seed_b=5678):
    """Seeded device operands in column-major storage (a stored R x C matrix is a (C, R)
    row-major tensor): A, B, C and their leading dimensions (bench-only)."""
    import torch
    from paper_conf_ipps_00020c20_b200 import inputs
    sa, sb = inputs.stored_shape(m, k, tA), inputs.stored_shape(k, n, tB)
    g = torch.Generator(device=dev).manual_seed(seed)
    A = (torch.rand(sa[1], sa[0], generator=g, device=dev) * 2 - 1).half()
    gb = torch.Generator(device=dev).manual_seed(seed_b)
    B = (torch.rand(sb[1], sb[0], generator=gb, device=dev) * 2 - 1).half()
    C = torch.zeros(n, m, dtype=torch.float32 if out == "f32" else torch.float16, device=dev)
    if beta != 0:
        C.uniform_(-1, 1)
    return A, max(1, sa[0]), B, max(1, sb[0]), C


def cublas_fn(A, B, C, tA, tB, alpha, beta):
    """cuBLAS (torch.mm / torch.addmm) on the same operands, layout and alpha/beta as
    hgemm(A, B, C): FP32 accumulation (reduced-precision reduction off); beta != 0
    reads and rewrites C in place."""
    import torch
    torch.backends.cuda.matmul.allow_fp16_reduced_precision_reduction = False
    # A.shape == (cols, rows) of the stored A, so op(A) = A ('T') or A.t() ('N'); likewise
    # op(B) = B.t() ('N') or B ('T').  Column-major C (m x n) is the row-major (n x m)
    # tensor C^T = op(B)^T op(A)^T.
    opA = A if tA in ("T", "t") else A.t()
    opB = B.t() if tB in ("N", "n") else B
    X, Y = opB.t(), opA.t()
    f32 = C.dtype == torch.float32

    def fn():
        if beta != 0:
            if not f32:
                return torch.addmm(C, X, Y, beta=beta, alpha=alpha, out=C)
            return torch.addmm(C, X, Y, out_dtype=torch.float32, beta=beta, alpha=alpha, out=C)
        if not f32:
            return torch.mm(X, Y, out=C) if alpha == 1 else torch.mm(X, Y, out=C).mul_(alpha)
        r = torch.mm(X, Y, out_dtype=torch.float32)
        return C.copy_(r) if alpha == 1 else C.copy_(r).mul_(alpha)
    return fn


# BASELINE.json configs reported beside the metric line, each with cuBLAS on the same
# operands (north_star (5)): config 1 (launch-bound: wall time), config 2 in
# the other layouts / FP32 out, config 3 (DL shapes, beta = 1), config 4 (HBM-bound).
SIDE_CONFIGS = ["cfg1_256_NN_f32", "cfg2_8192_NN_f16", "cfg2_8192_NT_f16", "cfg2_8192_TN_f32",
                "cfg3_bert_ffn1_4096", "cfg3_bert_ffn1_16384", "cfg3_bert_ffn2_4096",
                "cfg3_lstm_b64", "cfg3_lstm_b256", "cfg3_lstm_b1024",
                "cfg4_skinny_n64", "cfg4_skinny_n128", "cfg4_skinny_n256"]


def side_config(name, dev, flush, peaks, warmup, steps, compute=None):
    """One BJ config: ours (automatic kernel choice, or hgemm_ex with `compute`) and cuBLAS,
    device-resident inputs, L2 flushed between launches, mean of `steps` event-timed launches."""
    from paper_conf_ipps_00020c20_b200 import binding, inputs
    m, n, k, tA, tB, alpha, beta, out = inputs.WORKLOADS[name]
    A, lda, B, ldb, C = device_operands(dev, m, n, k, tA, tB, beta, out, seed=99, seed_b=98)
    if compute is None:
        def ours():
            binding.hgemm(m, n, k, alpha, A, lda, B, ldb, beta, C, m, tA, tB, out)
    else:
        def ours():
            binding.hgemm_ex(m, n, k, alpha, A, lda, B, ldb, beta, C, m, tA, tB, out, compute=compute)
    t_ours = timed(ours, flush, warmup, steps)
    st = binding.get_stats()
    t_cub = timed(cublas_fn(A, B, C, tA, tB, alpha, beta), flush, warmup, steps)
    flops = 2.0 * m * n * k
    esz = 4 if out == "f32" else 2
    r = roofline_entry(m, n, k, beta, esz, t_ours["mean"], peaks, None)
    rec = {"shape": [m, n, k], "layout": tA + tB, "alpha": alpha, "beta": beta, "out": out,
           "ours_ms": t_ours["mean"], "ours_ms_median": t_ours["median"],
           "ours_TFLOP/s": flops / (t_ours["mean"] * 1e-3) / 1e12,
           "cublas_ms": t_cub["mean"], "cublas_TFLOP/s": flops / (t_cub["mean"] * 1e-3) / 1e12,
           "ours_over_cublas": t_cub["mean"] / t_ours["mean"],
           "bound": r["bound"], "achieved": r["achieved"], "unit": r["unit"], "frac": r["frac"],
           "kernel": f"{st['last_kernel']}/{st['block_n']}" + (f" split {st['splits']}" if st["splits"] else ""),
           "steps": steps}
    if compute is not None:
        rec["compute"] = compute
    if name.startswith("cfg1"):
        rec["note"] = "launch-latency bound (34 MFLOP): wall time per call is the figure of merit"
    return rec


# ------------------------------------------------------------------ roofline
def alg_bytes(m, n, k, beta, esz):
    """Minimum HBM traffic of one launch: read A and B once, write C (and read it if beta != 0)."""
    return 2.0 * (m * k + k * n) + esz * m * n * (2 if beta != 0 else 1)


def roofline_entry(m, n, k, beta, esz, ms, peaks, traffic):
    """Roofline of the launch: tensor-bound when its intensity 2mnk / alg_bytes is above the
    ridge (measured bf16 TFLOP/s / measured HBM GB/s), HBM-bound below it."""
    flops = 2.0 * m * n * k
    byts = alg_bytes(m, n, k, beta, esz)
    ridge = peaks["tflops_burst"] * 1e12 / (peaks["hbm_gbs"] * 1e9)
    tb = traffic.get("bytes_per_launch") if isinstance(traffic, dict) else None
    if flops / byts >= ridge:
        a = flops / (ms * 1e-3) / 1e12
        return {"bound": "tensor", "achieved": a, "peak": peaks["tflops_burst"], "unit": UNIT,
                "frac": a / peaks["tflops_burst"], "traffic": tb, "traffic_detail": traffic,
                "peak_source": peaks["source"] + " burst (kernel timed alone)",
                "algorithmic": f"2*m*n*k = {flops:.4e} FLOP per launch (intensity {flops / byts:.0f} FLOP/B, "
                               f"ridge {ridge:.0f})"}
    a = byts / (ms * 1e-3) / 1e9
    return {"bound": "hbm", "achieved": a, "peak": peaks["hbm_gbs"], "unit": "GB/s",
            "frac": a / peaks["hbm_gbs"], "traffic": tb, "traffic_detail": traffic,
            "peak_source": peaks["source"],
            "algorithmic": f"2(mk+kn) + s_out*mn*(1+[beta!=0]) = {byts:.4e} B per launch "
                           f"(intensity {flops / byts:.0f} FLOP/B, ridge {ridge:.0f})"}


# ------------------------------------------------------------------ config 5: 32768^3, N-sharded (strong)
def strong_32768(args, world, rank, dev, flush, steps=5, warmup=2):
    """BASELINE.json configs[4]: the GLOBAL 32768^3 TN FP16-out problem with the columns of
    B and C split over the ranks (rank g: 32768 x 32768/G x 32768), A replicated.  Reports
    t_gemm (max over ranks of the mean of `steps` event-timed launches), and for N > 1 the
    exchange of A three ways (NCCL broadcast alone, broadcast then GEMM, broadcast
    pipelined in row panels, all-gather fused into the GEMM kernel), each guarded so that a
    failing leg records its error instead of losing the line.  Rank 0 also times the whole
    problem alone (t1) so the record carries t1 / (N * t_gemm)."""
    import torch
    from paper_conf_ipps_00020c20_b200 import binding
    from paper_conf_ipps_00020c20_b200.sharded import slab_bounds
    m = n = k = 32768
    n0, n1 = slab_bounds(n, world, rank)
    ns = n1 - n0
    A, lda, Bs, ldb, C = device_operands(dev, m, ns, k, "T", "N", 0.0, "f16", seed=4321, seed_b=8765 + rank)
    stream = torch.cuda.current_stream()
    rec = {"global_shape": [m, n, k], "layout": "TN", "out": "f16", "n_per_rank": ns, "world": world,
           "steps": steps, "what": "per-rank hgemm on its N-slab; A replicated (reported separately)"}

    def gemm():
        binding.hgemm(m, ns, k, 1.0, A, lda, Bs, ldb, 0.0, C, m, "T", "N", "f16")
    if world > 1:
        torch.distributed.barrier()
    t = timed(gemm, flush, warmup, steps, stream)
    t_gemm = max_over_ranks(t["mean"], world)
    rec["t_gemm_ms"] = t_gemm
    rec["t_gemm_ms_rank_spread"] = [min_over_ranks(t["mean"], world), t_gemm]
    rec["TFLOP/s_aggregate"] = 2.0 * m * n * k / (t_gemm * 1e-3) / 1e12
    st = binding.get_stats()
    rec["kernel"] = f"{st['last_kernel']}/{st['block_n']}"
    if rank == 0 and not args.no_cublas:
        try:
            tc = timed(cublas_fn(A, Bs, C, "T", "N", 1.0, 0.0), flush, warmup, steps, stream)
            rec["cublas_slab_ms"] = tc["mean"]
            rec["cublas_slab_TFLOP/s"] = 2.0 * m * ns * k / (tc["mean"] * 1e-3) / 1e12
        except Exception as e:  # pragma: no cover
            rec["cublas_error"] = f"{type(e).__name__}: {e}"
    if world > 1:
        # t1: the whole problem on rank 0 alone (same kernel path), for t1 / (N * t_gemm)
        t1 = None
        if rank == 0:
            try:
                del C
                B1 = torch.empty(n, k, dtype=torch.float16, device=dev).uniform_(-1, 1)
                C1 = torch.empty(n, m, dtype=torch.float16, device=dev)
                t1 = timed(lambda: binding.hgemm(m, n, k, 1.0, A, lda, B1, k, 0.0, C1, m, "T", "N", "f16"),
                           flush, 1, 3, stream)["mean"]
                del B1, C1
                C = torch.empty(ns, m, dtype=torch.float16, device=dev)
            except Exception as e:  # pragma: no cover
                rec["t1_error"] = f"{type(e).__name__}: {e}"
                C = torch.empty(ns, m, dtype=torch.float16, device=dev)
        else:
            pass
        torch.distributed.barrier()
        if rank == 0 and t1:
            rec["t1_ms"] = t1
            rec["efficiency_t1_over_N_tgemm"] = t1 / (world * t_gemm)
        rec.update(exchange_legs(args, world, rank, m, n, k, A, lda, Bs, ldb, C, "T", "N", "f16", stream))
    return rec


def exchange_legs(args, world, rank, m, n_glob, k, A, lda, Bs, ldb, C, tA, tB, out, stream, reps=3):
    """The replication of A for the N-slab sharded GEMM, timed three ways (north_star (3):
    the exchange is reported separately from the GEMM): NCCL broadcast alone, broadcast
    then GEMM, broadcast pipelined in row panels of op(A), and the all-gather fused into
    the GEMM kernel (hgemm_allgather_a).  Device time, mean of `reps`, max over ranks.
    Every leg is guarded: an error is recorded in place of its number."""
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_00020c20_b200.sharded import broadcast_A, hgemm_sharded, hgemm_sharded_overlapped
    res = {}

    def leg(name, fn, pre=None):
        try:
            fn()
            torch.cuda.synchronize()
            ts = []
            for _ in range(reps):
                if pre is not None:
                    pre()
                torch.cuda.synchronize()
                dist.barrier()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                fn()
                e1.record(stream)
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1))
            res[name] = max_over_ranks(statistics.mean(ts), world)
            res[name + "_spread"] = [min(ts), max(ts)]
        except Exception as e:  # pragma: no cover
            res[name] = None
            res[name + "_error"] = f"{type(e).__name__}: {e}"[:300]
            try:
                torch.cuda.synchronize()
            except Exception:
                pass
    res["a_bytes"] = A.numel() * 2
    leg("ms_bcast", lambda: broadcast_A(A, src=0))
    if res.get("ms_bcast"):
        res["bcast_GB_s"] = A.numel() * 2 / (res["ms_bcast"] * 1e-3) / 1e9
    res["bcast_backend"] = dist.get_backend()
    leg("ms_bcast_then_gemm", lambda: hgemm_sharded(m, n_glob, k, 1.0, A, lda, Bs, ldb, 0.0, C, m, tA, tB, out,
                                                    broadcast=True, local_slabs=True, stream=stream.cuda_stream))
    if tA in ("T", "t"):
        leg("ms_bcast_gemm_pipelined",
            lambda: hgemm_sharded_overlapped(m, n_glob, k, 1.0, A, lda, Bs, ldb, 0.0, C, m, tA, tB, out,
                                             panels=args.panels, local_slabs=True, stream=stream.cuda_stream))
        res["pipeline_panels"] = args.panels
        ag = None
        try:
            from paper_conf_ipps_00020c20_b200.sharded import FusedAllGatherA
            ag = FusedAllGatherA(m, k, lda=lda)
            r0, r1 = ag.own_rows
            ag.own_view().copy_(A[r0:r1, :k])
            torch.cuda.synchronize()
            dist.barrier()
            n_rank = C.shape[0]
            leg("ms_allgather_gemm_fused",
                lambda: ag(n_rank, 1.0, Bs, ldb, 0.0, C, m, tB, out, stream=stream.cuda_stream))
            res["allgather_fused_chunk_rows"] = ag.chunk_rows
            res["allgather_fused_gather_ok"] = bool(torch.equal(ag.A[:, :k], A[:, :k]))
        except Exception as e:  # pragma: no cover
            res["ms_allgather_gemm_fused"] = None
            res["ms_allgather_gemm_fused_error"] = f"{type(e).__name__}: {e}"[:300]
        finally:
            try:
                torch.cuda.synchronize()
                dist.barrier()
                if ag is not None:
                    ag.close()
            except Exception:
                pass
    return res


# ------------------------------------------------------------------ fused all-gather, one GPU
def ag_virtual(args, m, n, k, alpha, beta, tB, out, flush):
    """hgemm_allgather_a for virtual rank 0 of W ranks sharing this GPU (peers = other
    buffers on the same device, so the copy warps read local HBM): the kernel-side
    cost of the fusion (copy warp, chunk waits, chunk-ordered raster, copies competing
    for HBM) against hgemm() of the same shape.  No NVLink is involved; multi-GPU timing is in
    `collective` of an N > 1 run."""
    import torch
    from paper_conf_ipps_00020c20_b200 import binding
    from paper_conf_ipps_00020c20_b200.sharded import default_chunk_rows, slab_bounds
    W = args.ag_virtual
    cr = default_chunk_rows(m, W)
    rs = [slab_bounds(m, W, q, align=cr)[0] for q in range(W)] + [m]
    g = torch.Generator(device="cuda").manual_seed(77)
    full = (torch.rand(m, k, generator=g, device="cuda") * 2 - 1).half()
    bufs = [full.clone() for _ in range(W)]
    B = (torch.rand(n, k, generator=g, device="cuda") * 2 - 1).half()
    C = torch.empty(n, m, dtype=torch.float32 if out == "f32" else torch.float16, device="cuda")
    ws = torch.zeros(1 + -(-m // cr), dtype=torch.int32, device="cuda")

    def fused():
        binding.hgemm_allgather_a(m, n, k, alpha, bufs[0], k, bufs, rs, 0, B, k, beta, C, m, tB, out,
                                  workspace=ws, chunk_rows=cr)

    def plain():
        binding.hgemm(m, n, k, alpha, full, k, B, k, beta, C, m, "T", tB, out)
    res = {"virtual_world": W, "chunk_rows": cr, "copy_bytes": (m - rs[1]) * k * 2}
    for name, fn in (("ms_fused", fused), ("ms_plain", plain)):
        for _ in range(3):
            fn()
        ts = []
        for _ in range(max(3, min(args.steps, 20))):
            flush()
            if fn is fused:
                bufs[0][rs[1]:].fill_(0)              # the peers' rows must really be copied again
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            fn()
            e1.record()
            ts.append((e0, e1))
        torch.cuda.synchronize()
        res[name] = statistics.mean(a.elapsed_time(b) for a, b in ts)
        if fn is fused:
            res["gather_ok"] = bool(torch.equal(bufs[0], full))
    res["TFLOP/s_fused"] = 2.0 * m * n * k / (res["ms_fused"] * 1e-3) / 1e12
    return res


# ------------------------------------------------------------------ our arm
def run_ours(args, world, rank, local):
    import torch
    from paper_conf_ipps_00020c20_b200 import binding, inputs
    from paper_conf_ipps_00020c20_b200.sharded import hgemm_sharded, slab_bounds
    # HGEMM_DIST_BACKEND=gloo lets several ranks share one GPU to exercise the N > 1
    # code path where only one GPU is available (no performance meaning).
    backend = os.environ.get("HGEMM_DIST_BACKEND", "nccl")
    local = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        import torch.distributed as dist
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    lib = binding.load_library()
    m, n_cfg, k, tA, tB, alpha, beta, out = inputs.WORKLOADS[args.workload]
    if args.beta is not None:       # experiments only: override the workload's beta
        beta = args.beta
    strong = args.workload in inputs.STRONG_SCALING
    if args.kernel != "auto" or args.group_m or args.stream_k or args.splits:
        binding.set_config(args.kernel, block_n=args.block_n, group_m=args.group_m, stream_k=args.stream_k,
                           splits=args.splits)
    # weak scaling: every rank owns an n_cfg-wide slab (global n = n_cfg * world);
    # strong scaling (config 5): the global n_cfg columns are split over the ranks.
    n_glob = n_cfg if strong else n_cfg * world
    n0, n1 = slab_bounds(n_glob, world, rank)
    n_rank = n1 - n0
    out_t = torch.float32 if out == "f32" else torch.float16
    esz = 4 if out == "f32" else 2
    # device inputs, seeded on the device (bench-only large configs);
    # A is the replicated operand, Bs / C this rank's slabs
    A, lda, Bs, ldb, C = device_operands(dev, m, n_rank, k, tA, tB, beta, out, seed=1234, seed_b=5678 + rank)
    flush = L2Flush(dev)
    stream = torch.cuda.current_stream()
    compute = args.compute

    def step():
        if compute == "f16":
            binding.hgemm_ex(m, n_rank, k, alpha, A, lda, Bs, ldb, beta, C, m, tA, tB, out, compute="f16")
        else:
            hgemm_sharded(m, n_glob, k, alpha, A, lda, Bs, ldb, beta, C, m, tA, tB, out,
                          broadcast=False, local_slabs=True, stream=stream.cuda_stream)

    for _ in range(args.warmup):
        flush()
        step()
    torch.cuda.synchronize()
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    launches0 = lib.hgemm_launch_count()
    clocks = ClockSampler(local)
    clocks.start()
    evs = []
    probe = torch.zeros(4 * args.steps, dtype=torch.int64, device=dev)   # in-kernel SM clock probe
    for i in range(args.steps):
        flush()                                   # L2 flush, outside the events
        binding.set_probe(probe[4 * i:])
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        step()
        e1.record(stream)
        evs.append((e0, e1))
    binding.set_probe(None)
    torch.cuda.synchronize()
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize()
    clk = clocks.stop()
    pv = probe.view(-1, 4).cpu().tolist()
    ghz = [(c1 - c0) / (n1_ - n0_) for c0, n0_, c1, n1_ in pv if n1_ > n0_]
    if ghz:
        clk["sm_mhz_in_kernel_median"] = 1000.0 * statistics.median(ghz)
        clk["sm_mhz_in_kernel_min"] = 1000.0 * min(ghz)
        clk["in_kernel_how"] = "clock64 / %globaltimer deltas of CTA 0 per timed launch"
    launches = lib.hgemm_launch_count() - launches0
    step_ms = [a.elapsed_time(b) for a, b in evs]
    ms_local = statistics.mean(step_ms)
    ms = max_over_ranks(ms_local, world)
    flops_rank = 2.0 * m * n_rank * k
    flops_total = 2.0 * m * n_glob * k
    value = flops_total / (ms * 1e-3) / 1e12
    peaks = load_peaks()
    stats = binding.get_stats()
    if stats["last_kernel"] == "tc2" and compute == "f16":
        stats["compute"] = "f16 accumulate (hgemm_ex)"

    # cuBLAS on the same box, same tensors and layout (reference point, north_star (5)),
    # right after our timed region so that both see the same power-cap state
    cublas = None
    if not args.no_cublas and rank == 0:
        try:
            Cc = C.clone()
            tc = timed(cublas_fn(A, Bs, Cc, tA, tB, alpha, beta), flush, args.warmup, args.steps, stream)
            diff = (Cc.float() - C.float()).abs().max().item() if beta == 0 else None
            # tripwire: both accumulate in FP32, so they differ by ~1 output ulp at most
            # (|C| <~ 6 sqrt(k/9) for uniform[-1,1) inputs); a larger difference is a bug
            tol = 4.0 * 2.0 ** -10 * 6.0 * (k / 9.0) ** 0.5 if out == "f16" else 1e-4 * (k / 9.0) ** 0.5
            cublas = {"value": flops_rank / (tc["mean"] * 1e-3) / 1e12, "unit": UNIT, "ms": tc["mean"],
                      "ms_median": tc["median"], "max_abs_diff_vs_ours": diff,
                      "agrees_with_ours": None if diff is None else bool(diff <= tol), "agree_tol": tol,
                      "what": ("torch.addmm(C, ..., beta, alpha, out=C)" if beta != 0 else "torch.mm") +
                              " (cuBLAS), same operands, layout and alpha/beta, fp16 reduced-precision reduction off,"
                              " same W warm-up and K flushed steps as ours"}
            del Cc
        except Exception as e:  # pragma: no cover
            cublas = {"error": f"{type(e).__name__}: {e}"}

    # the exchange of A for the default (weak-scaling) workload, reported separately
    coll = None
    if world > 1 and not args.no_exchange:
        coll = exchange_legs(args, world, rank, m, n_glob, k, A, lda, Bs, ldb, C, tA, tB, out, stream)

    # e2e through the public C-ABI host-buffer call (hgemm_host): every step copies this
    # step's A and B from pinned host memory, runs the GEMM and copies C back, all
    # inside the timed region (the library pipelines panels on its own streams)
    e2e = None
    if not args.no_e2e:
        hA = A.cpu().pin_memory()
        hB = Bs.cpu().pin_memory()
        hC = torch.empty_like(C, device="cpu").pin_memory()
        ws = torch.empty(binding.host_workspace_size(m, n_rank, k, tA, tB, out), dtype=torch.uint8, device=dev)
        e2e_steps = max(1, min(args.steps, 10))
        binding.hgemm_host(m, n_rank, k, alpha, hA, lda, hB, ldb, beta, hC, m, tA, tB, out, ws,
                           stream=stream.cuda_stream)
        torch.cuda.synchronize()
        if world > 1:
            torch.distributed.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(e2e_steps):
            binding.hgemm_host(m, n_rank, k, alpha, hA, lda, hB, ldb, beta, hC, m, tA, tB, out, ws,
                               stream=stream.cuda_stream)
        e1.record(stream)
        torch.cuda.synchronize()
        ems = max_over_ranks(e0.elapsed_time(e1) / e2e_steps, world)
        e2e = {"value": flops_total / (ems * 1e-3) / 1e12, "unit": UNIT,
               "h2d_bytes_per_step": (A.numel() + Bs.numel()) * 2 * world + (C.numel() * esz * world if beta else 0),
               "d2h_bytes_per_step": C.numel() * esz * world, "ms_per_step": ems,
               "api": "hgemm_host (C ABI, pinned host buffers, panelled H2D/GEMM/D2H pipeline)"}
        del hA, hB, hC, ws

    # config 5 (32768^3 N-sharded, strong scaling) at every N; guarded
    strong_rec = None
    if not args.no_strong and args.workload != "cfg5_sharded_32768":
        try:
            strong_rec = strong_32768(args, world, rank, dev, flush)
        except Exception as e:  # pragma: no cover
            strong_rec = {"error": f"{type(e).__name__}: {e}"[:300]}
        torch.cuda.empty_cache()

    # every other BJ config with cuBLAS beside it, and the FP16-accumulate compute type (rank 0, N = 1)
    side = None
    if rank == 0 and world == 1 and not args.no_side and args.workload == "cfg2_8192_TN_f16":
        side = {}
        sst = max(5, min(args.steps, 30))
        for name in SIDE_CONFIGS:
            try:
                side[name] = side_config(name, dev, flush, peaks, 5, sst)
            except Exception as e:  # pragma: no cover
                side[name] = {"error": f"{type(e).__name__}: {e}"[:300]}
        try:
            side["cfg2_8192_TN_f16_acc16"] = side_config("cfg2_8192_TN_f16", dev, flush, peaks, 5, sst, compute="f16")
        except Exception as e:  # pragma: no cover
            side["cfg2_8192_TN_f16_acc16"] = {"error": f"{type(e).__name__}: {e}"[:300]}
        torch.cuda.empty_cache()

    agv = None
    if rank == 0 and world == 1 and args.ag_virtual > 0 and tA in ("T", "t"):
        agv = ag_virtual(args, m, n_rank, k, alpha, beta, tB, out, flush)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        cpu = cpu_baseline(args.workload, budget_s=args.cpu_budget)

    if rank == 0:
        peak = peaks["tflops_burst"]
        traffic = load_traffic(args.workload)
        roof = roofline_entry(m, n_rank, k, beta, esz, ms_local, peaks, traffic)
        if roof["bound"] == "tensor" and peaks.get("tflops_sustained"):
            roof["frac_vs_sustained_peak"] = roof["achieved"] / peaks["tflops_sustained"]
            roof["sustained_peak"] = peaks["tflops_sustained"]
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "strong" if strong else "weak",
            "vs_baseline": None,
            "dtype": "f16xf16->" + ("f16 accumulate" if compute == "f16" else "f32") + " (" + out + " out)",
            "data": "synthetic",
            "config": {"workload": args.workload, "m": m, "n": n_glob, "k": k, "n_per_gpu_rank0": n_rank,
                       "layout": tA + tB, "alpha": alpha, "beta": beta, "out": out,
                       "kernel": stats, "l2": "flushed between steps, outside the events: 256 MiB write, then a 256 MiB read so the write's dirty lines are written back before the timed launch",
                       "parallelism": f"n-slab x{world}" if world > 1 else "single GPU"},
            "pct_of_peak": 100.0 * value / world / peak,
            "roofline": roof,
            "gpu_launches": int(launches),
            "clocks": clk,
            "e2e": e2e,
            "cublas": cublas,
            "cpu_baseline": cpu,
            "collective": coll,
            "strong_32768": strong_rec,
            "bj_configs": side,
            "hbm_bound_configs": ({kk: v for kk, v in side.items() if v.get("bound") == "hbm"} if side else None),
            "allgather_fused_virtual": agv,
            "step_ms": {"min": min(step_ms), "median": statistics.median(step_ms), "max": max(step_ms)},
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
        dist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="cfg2_8192_TN_f16")
    ap.add_argument("--kernel", default="auto", choices=["auto", "tc1", "tc2", "simt", "splitk", "stream"])
    ap.add_argument("--stream-k", type=int, default=0, help="0 auto, 1 never, 2 always (experiments)")
    ap.add_argument("--splits", type=int, default=0, help="split-K cluster size (experiments)")
    ap.add_argument("--beta", type=float, default=None, help="override the workload's beta (experiments)")
    ap.add_argument("--block-n", type=int, default=0)
    ap.add_argument("--group-m", type=int, default=0)
    ap.add_argument("--ref-budget", type=float, default=60.0, help="seconds of oracle work for --impl reference")
    ap.add_argument("--cpu-budget", type=float, default=12.0)
    ap.add_argument("--panels", type=int, default=8, help="row panels of the pipelined broadcast (N > 1)")
    ap.add_argument("--ag-virtual", type=int, default=0,
                    help="also time the fused all-gather GEMM with W virtual ranks on this GPU (TN only)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cublas", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-side", action="store_true", help="skip the other BJ configs (bj_configs)")
    ap.add_argument("--no-strong", action="store_true", help="skip the 32768^3 N-sharded record (strong_32768)")
    ap.add_argument("--no-exchange", action="store_true", help="N > 1: skip the exchange-of-A legs")
    ap.add_argument("--compute", default="f32", choices=["f32", "f16"],
                    help="accumulation type of the timed step (f16: hgemm_ex FP16 accumulate, FP16 out)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    world, rank, local = dist_env()
    if args.impl == "reference":
        return run_reference(args, world, rank)
    return run_ours(args, world, rank, local)


if __name__ == "__main__":
    sys.exit(main())
