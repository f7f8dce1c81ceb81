"""Per-CTA timeline (globaltimer ns) of the tile kernel (build with -DHGEMM_TRACE and
run with HGEMM_LIB pointing at that build).

    python tools/trace_cta.py M N K [--beta B] [--kernel tc2] [--bn 256]

Fields (first two work items of every CTA): start, item0 MMA done, item0 epilogue
wake, item0 epilogue done, item1 ..., end.  Printed as min / median / max over CTAs.
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
ap.add_argument("--beta", type=float, default=1.0)
ap.add_argument("--kernel", default="auto")
ap.add_argument("--bn", type=int, default=0)
ap.add_argument("--sk", type=int, default=0)
ap.add_argument("--warm", action="store_true", help="no L2 flush between launches")
a = ap.parse_args()
if a.kernel != "auto":
    binding.set_config(a.kernel, block_n=a.bn, stream_k=a.sk)
m, n, k = a.m, a.n, a.k
A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
C = (torch.rand(n, m, device="cuda") * 2 - 1).half()
flush = torch.empty(64 * 1024 * 1024, device="cuda")
probe = torch.zeros(264 + 2 * 8 * 160, dtype=torch.int64, device="cuda")
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for i in range(6):
    if not a.warm:
        flush.zero_()
    binding.set_probe(probe if i == 5 else None)
    if i == 5:
        e0.record()
    binding.hgemm(m, n, k, 1.0, A, k, B, k, a.beta, C, m, "T", "N", "f16")
    if i == 5:
        e1.record()
torch.cuda.synchronize()
print(f"event time of the probed launch: {e0.elapsed_time(e1) * 1e3:.1f} us")
print(binding.get_stats())
v = probe.cpu().view(-1).tolist()
rows = [v[264 + 8 * b: 272 + 8 * b] for b in range(160) if v[264 + 8 * b]]
t0 = min(r[0] for r in rows)
names = ["start", "end", "i0_mma", "i0_wake", "i0_done", "i1_mma", "i1_wake", "i1_done"]
print(f"{len(rows)} CTAs; kernel span {max(r[1] for r in rows) - t0} ns")
for b, r in enumerate(rows[:6]):
    print(f"cta {b:3d} " + " ".join(f"{nm}={(x - t0) if x else -1}" for nm, x in zip(names, r)))
for f, nm in enumerate(names):
    xs = [r[f] - t0 for r in rows if r[f]]
    if xs:
        print(f"{nm:8s} n={len(xs):3d} min {min(xs):7d} med {statistics.median(xs):9.0f} max {max(xs):7d}")
