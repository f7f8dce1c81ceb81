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


def max_over_ranks(x, world):
    if world == 1:
        return x
    import torch
    import torch.distributed as dist
    dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor([x], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


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
            "cpu_baseline": {"value": val, "unit": UNIT, "cores": threads, "kind": "oracle", "sample": sample},
            "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


def cpu_baseline(workload, budget_s=12.0):
    """The oracle, as it stands, on the host cores over a bounded block of the workload."""
    import oracle
    from paper_conf_ipps_00020c20_b200 import inputs
    oracle.build()
    k = inputs.WORKLOADS[workload][2]
    threads = oracle.max_threads()
    ms, ns = _oracle_sample_size(workload, threads, budget_s)
    dt = _time_oracle(workload, ms, ns, threads)
    return {"value": 2.0 * ms * ns * k / dt / 1e12, "unit": UNIT, "cores": threads, "kind": "oracle",
            "sample": f"{ms} x {ns} block of C with the full k = {k} of {workload} ({dt:.1f} s)"}


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


def skinny_roofline(dev, flush, peaks, reps=20):
    """BJ configs[3]: M=16384, N in {64,128,256}, K=4096 (TN, FP16 out), device-resident,
    L2 flushed between launches; achieved GB/s of the algorithmic bytes vs the HBM peak."""
    import torch
    from paper_conf_ipps_00020c20_b200 import binding, inputs
    out = {}
    for name in ("cfg4_skinny_n64", "cfg4_skinny_n128", "cfg4_skinny_n256"):
        m, n, k, tA, tB, alpha, beta, o = inputs.WORKLOADS[name]
        g = torch.Generator(device=dev).manual_seed(99)
        sa, sb = inputs.stored_shape(m, k, tA), inputs.stored_shape(k, n, tB)
        A = (torch.rand(sa[1], sa[0], generator=g, device=dev) * 2 - 1).half()
        B = (torch.rand(sb[1], sb[0], generator=g, device=dev) * 2 - 1).half()
        C = torch.empty(n, m, dtype=torch.float16, device=dev)

        def call():
            binding.hgemm(m, n, k, alpha, A, sa[0], B, sb[0], beta, C, m, tA, tB, o)
        for _ in range(3):
            call()
        ts = []
        for _ in range(reps):
            flush()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            call()
            e1.record()
            ts.append((e0, e1))
        torch.cuda.synchronize()
        ms = statistics.mean(a.elapsed_time(b) for a, b in ts)
        r = roofline_entry(m, n, k, beta, 2, ms, peaks, None)
        st = binding.get_stats()
        out[name] = {"ms": ms, "bound": r["bound"], "achieved": r["achieved"], "unit": r["unit"],
                     "frac": r["frac"], "TFLOP/s": 2.0 * m * n * k / (ms * 1e-3) / 1e12,
                     "kernel": f"{st['last_kernel']}/{st['block_n']}" + (f" split {st['splits']}" if st['splits'] else "")}
    return out


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
    from paper_conf_ipps_00020c20_b200.sharded import broadcast_A, hgemm_sharded, slab_bounds
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
    sa = inputs.stored_shape(m, k, tA)
    sb_rank = inputs.stored_shape(k, n_rank, tB)
    # device inputs, seeded on the device (bench-only large configs).
    # Column-major storage: a stored R x C matrix is a (C, R) row-major tensor.
    g = torch.Generator(device=dev).manual_seed(1234)
    A = (torch.rand(sa[1], sa[0], generator=g, device=dev) * 2 - 1).half()
    gb = torch.Generator(device=dev).manual_seed(5678 + rank)
    Bs = (torch.rand(sb_rank[1], sb_rank[0], generator=gb, device=dev) * 2 - 1).half()   # this rank's slab
    C = torch.zeros(n_rank, m, dtype=out_t, device=dev)                                   # this rank's slab
    if beta != 0:
        C.uniform_(-1, 1)
    lda, ldb = sa[0], sb_rank[0]
    flush = L2Flush(dev)
    stream = torch.cuda.current_stream()

    # the sharded path's one collective: replicate A (rank 0's copy) over NCCL, timed separately
    coll = None
    if world > 1:
        import torch.distributed as dist
        for _ in range(2):
            broadcast_A(A, src=0)
        torch.cuda.synchronize()
        dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        broadcast_A(A, src=0)
        e1.record()
        torch.cuda.synchronize()
        bms = max_over_ranks(e0.elapsed_time(e1), world)
        coll = {"op": f"broadcast(A) over {dist.get_backend()} (torch.distributed)", "bytes": A.numel() * 2, "ms": bms,
                "GB_s": A.numel() * 2 / (bms * 1e-3) / 1e9,
                "note": "reported separately from the GEMM (north_star (3)); not inside value"}
        # broadcast + GEMM as one step: serial, and pipelined in row panels of op(A) (NEXT-2)
        if tA in ("T", "t"):
            from paper_conf_ipps_00020c20_b200.sharded import hgemm_sharded_overlapped

            def serial():
                hgemm_sharded(m, n_glob, k, alpha, A, lda, Bs, ldb, beta, C, m, tA, tB, out,
                              broadcast=True, local_slabs=True, stream=stream.cuda_stream)

            def overlapped():
                hgemm_sharded_overlapped(m, n_glob, k, alpha, A, lda, Bs, ldb, beta, C, m, tA, tB, out,
                                         panels=args.panels, local_slabs=True, stream=stream.cuda_stream)
            for name, fn in (("ms_bcast_then_gemm", serial), ("ms_bcast_gemm_pipelined", overlapped)):
                fn()
                torch.cuda.synchronize()
                dist.barrier()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                fn()
                e1.record()
                torch.cuda.synchronize()
                coll[name] = max_over_ranks(e0.elapsed_time(e1), world)
            coll["pipeline_panels"] = args.panels
            # the all-gather fused with the GEMM (hgemm_allgather_a): A row-sharded over the
            # ranks, peers' rows pulled over NVLink by the copy engines chunk by chunk while
            # the persistent kernel consumes each chunk once its flag is raised
            from paper_conf_ipps_00020c20_b200.sharded import FusedAllGatherA
            ag = FusedAllGatherA(m, k, lda=lda)
            r0, r1 = ag.own_rows
            ag.own_view().copy_(A[r0:r1, :k])

            def fused():
                ag(n_rank, alpha, Bs, ldb, beta, C, m, tB, out, stream=stream.cuda_stream)
            tf = []
            for it in range(3):
                torch.cuda.synchronize()
                dist.barrier()                       # peers' rows are complete and no longer being read
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                fused()
                e1.record(stream)
                torch.cuda.synchronize()
                if it:
                    tf.append(e0.elapsed_time(e1))
            coll["ms_allgather_gemm_fused"] = max_over_ranks(statistics.mean(tf), world)
            coll["allgather_fused_chunk_rows"] = ag.chunk_rows
            coll["allgather_fused_gather_ok"] = bool(torch.equal(ag.A[:, :k], A[:, :k]))
            torch.cuda.synchronize()
            dist.barrier()
            ag.close()

    def step():
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
    ghz = [(c1 - c0) / (n1 - n0) for c0, n0, c1, n1 in pv if n1 > n0]
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
    achieved = flops_rank / (ms_local * 1e-3) / 1e12
    stats = binding.get_stats()

    # cuBLAS on the same box, same tensors and layout (reference point, north_star (5)),
    # right after our timed region so that both see the same power-cap state (the
    # PCIe-bound e2e leg below lets the GPU cool down)
    cublas = None
    if not args.no_cublas and rank == 0:
        try:
            torch.backends.cuda.matmul.allow_fp16_reduced_precision_reduction = False
            # Storage tensors are the transposes of the column-major matrices:
            # A.shape == (cols, rows) of the stored A, so op(A) = A ('T') or A.t() ('N');
            # likewise op(B) = Bs.t() ('N') or Bs ('T').  Column-major C (m x n) is the
            # row-major (n x m) tensor C^T = op(B)^T op(A)^T.
            opA = A if tA in ("T", "t") else A.t()
            opB = Bs.t() if tB in ("N", "n") else Bs
            X, Y = opB.t(), opA.t()

            # same alpha/beta semantics: beta != 0 reads and rewrites C in place (addmm)
            Cc = C.clone() if beta != 0 else None

            def cub():
                if beta != 0:
                    if out_t == torch.float16:
                        return torch.addmm(Cc, X, Y, beta=beta, alpha=alpha, out=Cc)
                    return torch.addmm(Cc, X, Y, out_dtype=torch.float32, beta=beta, alpha=alpha, out=Cc)
                if out_t == torch.float16:
                    return torch.mm(X, Y) if alpha == 1 else torch.mm(X, Y).mul_(alpha)
                return torch.mm(X, Y, out_dtype=torch.float32)
            ref_c = cub()
            # same protocol as our timed region (W warm-up steps, then K flushed steps):
            # under the 1 kW power cap the SM clock falls during a long run, so a shorter
            # cuBLAS run would be timed at a higher clock than ours
            for _ in range(args.warmup):
                flush()
                cub()
            torch.cuda.synchronize()
            ts = []
            for _ in range(args.steps):
                flush()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                cub()
                e1.record()
                ts.append((e0, e1))
            torch.cuda.synchronize()
            # agreement with our C (both FP32-accumulated; loose sanity bound only)
            diff = (ref_c.float() - C.float()).abs().max().item() if beta == 0 else None
            cms = statistics.mean(a.elapsed_time(b) for a, b in ts)
            cublas = {"value": flops_rank / (cms * 1e-3) / 1e12, "unit": UNIT, "ms": cms, "max_abs_diff_vs_ours": diff,
                      "what": ("torch.addmm(C, ..., beta, alpha, out=C)" if beta != 0 else "torch.mm") +
                              " (cuBLAS), same operands, layout and alpha/beta, fp16 reduced-precision reduction off"}
        except Exception as e:  # pragma: no cover
            cublas = {"error": f"{type(e).__name__}: {e}"}

    # e2e through the public C-ABI host-buffer call (hgemm_host): every step copies this
    # step's A and B from pinned host memory, runs the GEMM and copies C back, all
    # inside the timed region (the library pipelines column panels on its own streams)
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

    # the HBM-bound skinny configs (BJ configs[3]) against the HBM roofline (north_star (5))
    side = None
    if rank == 0 and world == 1 and not args.no_side and args.workload == "cfg2_8192_TN_f16":
        side = skinny_roofline(dev, flush, peaks)

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
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "strong" if strong else "weak",
            "vs_baseline": None, "dtype": "f16xf16->f32 (" + out + " out)", "data": "synthetic",
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
            "hbm_bound_configs": side,
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
    ap.add_argument("--no-side", action="store_true", help="skip the skinny-shape HBM roofline report")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    world, rank, local = dist_env()
    if args.impl == "reference":
        return run_reference(args, world, rank)
    return run_ours(args, world, rank, local)


if __name__ == "__main__":
    sys.exit(main())
