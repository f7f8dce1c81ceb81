"""B200 micro-benchmarks (NEXT-4): the paper's SIV-SV characterisation redone
for the sm_100a units the HGEMM is built on.  Needs a GPU; writes a JSON
summary (default gpurun_out/microbench.json).

  tcgen05.mma kind::f16 throughput per SM and latency   (cf. Table I, HMMA.1688 CPI 8.06)
  tcgen05.ld  TMEM -> register bandwidth                 (cf. Table IV/V, LDS/STS)
  TMA loads from L2 and from HBM                          (cf. Table II/III, DRAM/L2/LDG)
"""
import ctypes
import json
import os
import statistics
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_ipps_00020c20_b200 import build  # noqa: E402

lib = ctypes.CDLL(build.build_microbench())
i32, vp = ctypes.c_int, ctypes.c_void_p
lib.mb_mma_rate.argtypes = [i32, i32, i32, i32, i32, vp]
lib.mb_tmem_ld.argtypes = [i32, i32, i32, i32, vp]
lib.mb_tma_load.argtypes = [vp, i32, i32, i32, i32, vp]
SMS = torch.cuda.get_device_properties(0).multi_processor_count
out_path = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "gpurun_out", "microbench.json")
res = {"device": torch.cuda.get_device_name(0), "sms": SMS}


def run(fn, grid):
    cyc = torch.zeros(grid + 1, dtype=torch.int64, device="cuda")
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    fn(cyc, warm=True)
    torch.cuda.synchronize()
    e0.record()
    rc = fn(cyc, warm=False)
    e1.record()
    torch.cuda.synchronize()
    assert rc == 0, rc
    c = [int(x) for x in cyc[:grid].cpu().tolist() if int(x) > 0]
    return c, e0.elapsed_time(e1)


# tcgen05.mma throughput: back-to-back MMAs from one thread, all SMs busy
mma = []
for cg in (1, 2):
    for n in (64, 128, 256):
        iters = 2048
        c, ms = run(lambda cyc, warm: lib.mb_mma_rate(cg, n, 64 if warm else iters, SMS, 0, cyc.data_ptr()), SMS)
        per = statistics.median(c) / (iters * 4)
        M = 128 * cg
        flop = 2.0 * M * n * 16
        rec = {"cta_group": cg, "M": M, "N": n, "K": 16, "cycles_per_mma": per,
               "flop_per_clk_per_sm": flop / per / cg,
               "chip_tflops_at_kernel_time": flop * iters * 4 * (SMS // cg) / (ms * 1e-3) / 1e12,
               "clock_ghz_est": statistics.median(c) / (ms * 1e6)}
        mma.append(rec)
        print(f"mma cg={cg} M={M:3d} N={n:3d}: {per:7.1f} cycles/MMA  {rec['flop_per_clk_per_sm']:7.0f} FLOP/clk/SM  "
              f"chip {rec['chip_tflops_at_kernel_time']:7.1f} TFLOP/s @ {rec['clock_ghz_est']:.2f} GHz", flush=True)
res["mma_throughput"] = mma

# latency: MMA + commit + mbarrier wait round trip
lat = []
for cg in (1, 2):
    for n in (64, 256):
        iters = 256
        c, _ = run(lambda cyc, warm: lib.mb_mma_rate(cg, n, 8 if warm else iters, 2 * cg, 1, cyc.data_ptr()), 2 * cg)
        per = statistics.median(c) / iters
        lat.append({"cta_group": cg, "M": 128 * cg, "N": n, "cycles_issue_to_mbarrier": per})
        print(f"mma latency cg={cg} M={128 * cg} N={n}: {per:.0f} cycles (issue -> commit -> mbarrier)", flush=True)
res["mma_latency"] = lat

# TMEM -> registers
tm = []
for warps in (4, 8):
    for unroll in (1, 4):
        iters = 4096
        c, ms = run(lambda cyc, warm: lib.mb_tmem_ld(64 if warm else iters, warps, unroll, SMS, cyc.data_ptr()), SMS)
        bpc = warps * 4096.0 * iters / statistics.median(c)
        tm.append({"warps": warps, "loads_per_wait": unroll, "bytes_per_clk_per_sm": bpc})
        print(f"tcgen05.ld 32x32b.x32, {warps} warps, {unroll} load(s) per wait: {bpc:.1f} B/clk/SM", flush=True)
res["tmem_ld"] = tm

# TMA loads
tma = []
big_rows = 2 * 1024 * 1024  # 2 Mi rows x 1 KB = 2 GiB
buf = torch.empty(big_rows * 512, dtype=torch.float16, device="cuda").uniform_(-1, 1)
for streaming, label in ((0, "L2-resident 16 KB tile"), (1, "HBM streaming (each CTA its own 8 MiB)")):
    iters = 4096 if not streaming else 512   # streaming: 148 x 512 x 16 KB = 1.2 GiB, no re-reads
    c, ms = run(lambda cyc, warm: lib.mb_tma_load(buf.data_ptr(), big_rows, 64 if warm else iters, SMS, streaming,
                                                  cyc.data_ptr()), SMS)
    bpc = 16384.0 * iters / statistics.median(c)
    gbs = 16384.0 * iters * SMS / (ms * 1e-3) / 1e9
    tma.append({"source": label, "bytes_per_clk_per_sm": bpc, "chip_GB_s": gbs})
    print(f"TMA 128x128B boxes, {label}: {bpc:.1f} B/clk/SM, chip {gbs:.0f} GB/s", flush=True)
res["tma_load"] = tma
os.makedirs(os.path.dirname(out_path), exist_ok=True)
with open(out_path, "w") as f:
    json.dump(res, f, indent=1)
print("wrote", out_path)
