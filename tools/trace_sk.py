"""Per-CTA timeline (globaltimer ns) of the split-K kernel (build with -DHGEMM_TRACE).

    python tools/trace_sk.py [m n k] [--warm]

--warm: no L2 flush before the probed launch (code, tensor maps and operands L2-resident).
Also prints the producer's prologue detail (second probe region)."""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402

_a = [x for x in sys.argv[1:] if not x.startswith('--')]
m, n, k = (int(x) for x in _a[:3]) if len(_a) >= 3 else (64, 4096, 2048)
A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
C = (torch.rand(n, m, device="cuda") * 2 - 1).half()
flush = torch.empty(64 * 1024 * 1024, device="cuda")
probe = torch.zeros(8 + 3 * 256 * 8, dtype=torch.int64, device="cuda")
warm = "--warm" in sys.argv
for i in range(5):
    if not (warm and i == 4):
        flush.zero_()
    binding.set_probe(probe if i == 4 else None)
    binding.hgemm(m, n, k, 1.0, A, k, B, k, 1.0, C, m, "T", "N", "f16")
torch.cuda.synchronize()
print(binding.get_stats())
v = probe.cpu().view(-1).tolist()
rows = [v[8 + 8 * b: 16 + 8 * b] for b in range(256) if v[8 + 8 * b]]
t0 = min(r[0] for r in rows)
names = ["start", "setup", "data0", "mma_issued", "tfull", "sent", "epi_done", "end"]
print("cta " + " ".join(f"{x:>10s}" for x in names))
for b, r in enumerate(rows[:12]):
    print(f"{b:3d} " + " ".join(f"{(x - t0) if x else -1:10d}" for x in r))
import statistics
for f in range(8):
    xs = [r[f] - t0 for r in rows if r[f]]
    print(f"{names[f]:10s} min {min(xs):7d} med {statistics.median(xs):9.0f} max {max(xs):7d}")
names2 = ["p_entry", "p_init", "p_gdwait", "p_ring", "w1_alloc0", "w1_alloc1", "p_tma0"]
rows2 = [v[8 + 2048 + 8 * b: 8 + 2048 + 8 * b + 8] for b in range(256) if v[8 + 8 * b]]
for f in range(7):
    xs = [r[f] - t0 for r in rows2 if r[f]]
    if xs:
        print(f"{names2[f]:10s} min {min(xs):7d} med {statistics.median(xs):9.0f} max {max(xs):7d}")
names3 = ["w2_presync", "w5_presync", "t0_postsync", "w2_cpre", "w2_tmld0", "w2_staged", "w2_rbar", "w2_summed"]
rows3 = [v[8 + 4096 + 8 * b: 8 + 4096 + 8 * b + 8] for b in range(256) if v[8 + 8 * b]]
for f in range(8):
    xs = [r[f] - t0 for r in rows3 if r[f]]
    if xs:
        print(f"{names3[f]:10s} min {min(xs):7d} med {statistics.median(xs):9.0f} max {max(xs):7d}")
