"""Print the accumulator hand-off timeline of CTA 0 (build with -DHGEMM_TRACE).

Fields per tile (clock64 cycles, relative to the kernel start):
 0 MMA: last MMA issued + tfull committed   1 EPI: tfull observed
 2 EPI: half 0 drained (tempty[0] arrive)   3 EPI: half 1 drained
 4 MMA: tempty[0] acquired                  5 MMA: tempty[1] acquired
 6 MMA: first full stage acquired
"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402

import argparse  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("m", type=int, nargs="?", default=8192)
ap.add_argument("--n", type=int, default=0)
ap.add_argument("--k", type=int, default=0)
ap.add_argument("--bn", type=int, default=0)
ap.add_argument("--beta", type=float, default=0.0)
a = ap.parse_args()
m = a.m
n = a.n or m
k = a.k or m
if a.bn:
    binding.set_config("tc2", block_n=a.bn)
A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
C = (torch.rand(n, m, device="cuda") * 2 - 1).half()
probe = torch.zeros(8 + 16 * 16, dtype=torch.int64, device="cuda")
for i in range(6):
    binding.set_probe(probe if i == 5 else None)
    binding.hgemm(m, n, k, 1.0, A, k, B, k, a.beta, C, m, "T", "N", "f16")
torch.cuda.synchronize()
v = probe.cpu().tolist()
t0 = v[0]
print(f"kernel: {v[2]-v[0]} cycles, {v[3]-v[1]} ns, {(v[2]-v[0])/(v[3]-v[1]):.3f} GHz")
names = ["mma_done", "epi_wake", "drain0", "drain1", "tempty0", "tempty1", "full0", "fullwait", "bar_pass", "ld0_done"]
print("tile " + " ".join(f"{x:>10s}" for x in names))
for it in range(16):
    row = v[8 + 16 * it: 8 + 16 * it + 10]
    if not any(row):
        break
    print(f"{it:4d} " + " ".join(f"{(x - t0 if x else 0):10d}" for x in row[:7]) + f" {row[7]:10d}"
          + " ".join(f"{(x - t0 if x else 0):10d}" for x in row[8:10]))
for it in range(15):
    a = v[8 + 16 * it: 8 + 16 * it + 12]
    b = v[8 + 16 * (it + 1): 8 + 16 * (it + 1) + 12]
    if not any(b):
        break
    print(f"tile {it}->{it+1}: commit->wake {a[1]-a[0]}, wake->bar {a[8]-a[1]}, bar->ld0 {a[9]-a[8]}, "
          f"ld0->packed0 {a[10]-a[9]}, packed0->arrived0 {a[2]-a[10]}, arrived0->packed1 {a[11]-a[2]}, "
          f"wake->drain0 {a[2]-a[1]}, drain0->drain1 {a[3]-a[2]}, "
          f"drain0->mma_tempty0 {b[4]-a[2]}, commit->next_tempty0 {b[4]-a[0]}, next tile MMA span {b[0]-b[4]}")
