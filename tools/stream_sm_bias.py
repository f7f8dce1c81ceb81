"""Is the streaming kernel's tail systematic per SM?  Runs the skinny config several times with
the HGEMM_TRACE build (HGEMM_LIB) and correlates each SM's mainloop finish time across runs
(experiments).

    HGEMM_LIB=.../trace.so python tools/stream_sm_bias.py [n]
"""
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 64
m, k = 16384, 4096
A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
C = torch.empty(n, m, device="cuda", dtype=torch.half)
w = torch.empty(64 * 1024 * 1024, device="cuda")
probe = torch.zeros(8 * 160, dtype=torch.int64, device="cuda")
runs = []
for rep in range(6):
    w.zero_()
    probe.zero_()
    binding.set_probe(probe)
    binding.hgemm(m, n, k, 1.0, A, k, B, k, 0.0, C, m, "T", "N", "f16")
    torch.cuda.synchronize()
    binding.set_probe(None)
    v = probe.view(-1, 8).cpu().tolist()
    rows = [r for r in v if r[0]]
    t0 = min(r[0] for r in rows)
    runs.append({int(r[7]): (r[3] - t0) / 1e3 for r in rows})  # smid -> mma_done (us)
sms = sorted(set.intersection(*[set(r) for r in runs[1:]]))
def ranks(d):
    order = sorted(sms, key=lambda s: d[s])
    return {s: i for i, s in enumerate(order)}
rk = [ranks(r) for r in runs[1:]]
def corr(a, b):
    xs = [a[s] for s in sms]; ys = [b[s] for s in sms]
    mx, my = statistics.mean(xs), statistics.mean(ys)
    num = sum((x - mx) * (y - my) for x, y in zip(xs, ys))
    den = (sum((x - mx) ** 2 for x in xs) * sum((y - my) ** 2 for y in ys)) ** 0.5
    return num / den
print(f"n={n}: {len(sms)} SMs; finish spread per run (us):",
      [f"{min(r[s] for s in sms):.1f}-{max(r[s] for s in sms):.1f}" for r in runs[1:]])
print("rank correlation of per-SM finish times between consecutive runs:",
      [round(corr(rk[i], rk[i + 1]), 2) for i in range(len(rk) - 1)])
avg = {s: statistics.mean(r[s] for r in runs[1:]) for s in sms}
slow = sorted(sms, key=lambda s: -avg[s])[:12]
print("slowest SMs (mean finish us):", [(s, round(avg[s], 1)) for s in slow])
print("fastest SMs:", [(s, round(avg[s], 1)) for s in sorted(sms, key=lambda s: avg[s])[:8]])
