"""Per-CTA phase timeline of one cold launch (library built with -DHGEMM_TRACE).

    HGEMM_LIB=.../libhgemm_trace.so python tools/trace_cta2.py M N K [--beta B] [--warm]

Slots (globaltimer ns, relative to the earliest CTA entry): entry, prologue done
(after griddepcontrol.wait), first TMA issued, first full stage at the MMA warp,
first item MMA done, epilogue wake, epilogue done, end.  min / median / max over CTAs.
"""
import argparse
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("m", type=int)
ap.add_argument("n", type=int)
ap.add_argument("k", type=int)
ap.add_argument("--beta", type=float, default=0.0)
ap.add_argument("--warm", action="store_true")
a = ap.parse_args()
m, n, k = a.m, a.n, a.k
A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
C = (torch.rand(n, m, device="cuda") * 2 - 1).half()
w = torch.empty(64 * 1024 * 1024, device="cuda")
probe = torch.zeros(264 + 8 * 160 * 2, dtype=torch.int64, device="cuda")
for i in range(5):
    if not a.warm:
        w.zero_()
    torch.cuda._sleep(100000)
    binding.set_probe(probe if i == 4 else None)
    binding.hgemm(m, n, k, 1.0, A, k, B, k, a.beta, C, m, "T", "N", "f16")
torch.cuda.synchronize()
binding.set_probe(None)
v = probe.view(-1).tolist()
rows = [v[264 + 8 * b: 272 + 8 * b] for b in range(160) if v[264 + 8 * b]]
t0 = min(r[0] for r in rows)
st = binding.get_stats()
print(f"{m}x{n}x{k} beta={a.beta} {'warm' if a.warm else 'cold'} {st['last_kernel']}/{st['block_n']}: {len(rows)} CTAs")
names = [(0, "entry"), (2, "prologue"), (3, "tma0"), (4, "full0"), (5, "mma_done"), (6, "epi_wake"), (7, "epi_done"),
         (1, "end")]
for f, nm in names:
    xs = [r[f] - t0 for r in rows if r[f]]
    if xs:
        print(f"  {nm:9s} n={len(xs):3d} min {min(xs) / 1e3:7.2f} med {statistics.median(xs) / 1e3:7.2f} "
              f"max {max(xs) / 1e3:7.2f} us")
rows2 = [v[264 + 1280 + 8 * b: 264 + 1280 + 8 * b + 8] for b in range(160) if v[264 + 8 * b]]
for f, nm in [(0, "prod_start"), (1, "item0"), (2, "empty0"), (3, "expect_tx"), (4, "tmaA0"),
              (5, "epi_tmem"), (6, "epi_stores"), (7, "epi_wait")]:
    xs = [r[f] - t0 for r in rows2 if r[f]]
    if xs:
        print(f"  {nm:10s} n={len(xs):3d} min {min(xs) / 1e3:7.2f} med {statistics.median(xs) / 1e3:7.2f} "
              f"max {max(xs) / 1e3:7.2f} us")
