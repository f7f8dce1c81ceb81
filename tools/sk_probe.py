"""Stream-K experiments: throughput per cluster count and the CTA-0 item timeline (trace build)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402

m, n, k = (int(v) for v in (sys.argv[1] if len(sys.argv) > 1 else "4096x1024x4096").split("x"))
A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
C = torch.empty(n, m, dtype=torch.half, device="cuda")


def run(kern, bn, sk, max_ctas, iters=20):
    binding.set_config(kern, block_n=bn, stream_k=sk, max_ctas=max_ctas)
    for _ in range(3):
        binding.hgemm(m, n, k, 1.0, A, k, B, k, 0.0, C, m, "T", "N", "f16")
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(iters):
        binding.hgemm(m, n, k, 1.0, A, k, B, k, 0.0, C, m, "T", "N", "f16")
    e1.record()
    torch.cuda.synchronize()
    st = binding.get_stats()
    return 2.0 * m * n * k / (e0.elapsed_time(e1) / iters) / 1e9, st["stream_k"]


for kern, bn in ([("tc2", 256), ("tc1", 256)] if not os.environ.get("HGEMM_LIB", "").endswith("trace.so") else []):
    for sk, mc in [(1, 0), (2, 0), (2, 146), (2, 140), (2, 132), (2, 130), (1, 128)]:
        tf, used = run(kern, bn, sk, mc)
        print(f"{kern}/{bn} sk={sk} max_ctas={mc}: {tf:7.1f} TF (stream_k used: {used == 2})", flush=True)

if os.environ.get("HGEMM_LIB", "").endswith("trace.so"):
    for sk, mc in [(1, 0), (2, 0), (2, 130)]:
        binding.set_config("tc2", block_n=256, stream_k=sk, max_ctas=mc)
        probe = torch.zeros(264 + 2 * 8 * 160, dtype=torch.int64, device="cuda")
        for i in range(4):
            binding.set_probe(probe if i == 3 else None)
            binding.hgemm(m, n, k, 1.0, A, k, B, k, 0.0, C, m, "T", "N", "f16")
        torch.cuda.synchronize()
        binding.set_probe(None)
        v = probe.cpu().tolist()
        t0 = v[0]
        print(f"stream_k={sk}: kernel {v[2]-v[0]} cycles, {v[3]-v[1]} ns, {(v[2]-v[0])/max(v[3]-v[1],1):.3f} GHz")
        names = {0: "mma_done", 1: "epi_wake", 2: "drain0", 4: "tempty0", 6: "full0", 12: "flags_ok", 13: "epi_end"}
        for it in range(16):
            row = v[8 + 16 * it: 8 + 16 * it + 16]
            if not any(row):
                break
            d = {nm: (row[f] - t0 if row[f] else 0) for f, nm in names.items()}
            d["full_wait"] = row[7]
            print(it, d)
        ct = {b: v[264 + 8 * b: 272 + 8 * b] for b in range(160) if v[264 + 8 * b]}
        g0 = min(r[0] for r in ct.values())
        ends = sorted(r[1] - g0 for r in ct.values())
        print(f"  {len(ct)} CTAs; end ns: min {ends[0]} med {ends[len(ends)//2]} max {ends[-1]}")
        nkb = (k + 63) // 64
        G = len(ct) // 2
        tiles = ((n + 255) // 256) * ((m + 255) // 256)
        for b in sorted(ct, key=lambda b: ct[b][1])[-6:] + sorted(ct, key=lambda b: ct[b][1])[:3]:
            r = [x - g0 if x else 0 for x in ct[b]]
            c = b // 2
            u0, u1 = tiles * nkb * c // G, tiles * nkb * (c + 1) // G
            print(f"  cta {b:3d} range [{u0},{u1}) tile {u0 // nkb}:{u0 % nkb}..{u1 // nkb}:{u1 % nkb} end {r[1]} "
                  f"item0 mma {r[2]} flags {r[3]} epi {r[4]} | item1 mma {r[5]} flags {r[6]} epi {r[7]}")
