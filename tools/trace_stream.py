"""Per-CTA timeline (globaltimer ns) of the HBM-streaming kernel (build with
-DHGEMM_TRACE; HGEMM_LIB pointing at that build).  python tools/trace_stream.py M N K"""
import os
import statistics
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding, build  # noqa: E402
import ctypes  # noqa: E402

mb = ctypes.CDLL(build.build_microbench())
mb.mb_stamp.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
st = torch.zeros(2, dtype=torch.int64, device="cuda")

m, n, k = (int(x) for x in sys.argv[1:4]) if len(sys.argv) > 3 else (16384, 64, 4096)
beta = float(sys.argv[4]) if len(sys.argv) > 4 else 0.0
cw = int(sys.argv[5]) if len(sys.argv) > 5 else 0
if "--force" in sys.argv or cw:
    binding.set_config("stream", block_n=cw)
A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
C = torch.empty(n, m, device="cuda", dtype=torch.half)
w = torch.empty(64 * 1024 * 1024, device="cuda")
r = torch.zeros(64 * 1024 * 1024, device="cuda")
probe = torch.zeros(8 * 160, dtype=torch.int64, device="cuda")
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
for i in range(6):
    w.zero_()
    r.sum()
    binding.set_probe(probe if i == 5 else None)
    if i == 5:
        e0.record()
        mb.mb_stamp(st.data_ptr(), torch.cuda.current_stream().cuda_stream)
    binding.hgemm(m, n, k, 1.0, A, k, B, k, beta, C, m, "T", "N", "f16")
    if i == 5:
        mb.mb_stamp(st.data_ptr() + 8, torch.cuda.current_stream().cuda_stream)
        e1.record()
torch.cuda.synchronize()
print(f"event time of the probed launch {e0.elapsed_time(e1) * 1e3:.1f} us")
print(binding.get_stats())
v = probe.cpu().view(-1).tolist()
rows = [v[8 * b: 8 * b + 8] for b in range(160) if v[8 * b]]
t0 = min(x[0] for x in rows)
names = ["start", "setup", "data0", "mma_done", "epi_wake", "epi_done", "end"]
print(f"{m}x{n}x{k} beta={beta}: {len(rows)} CTAs; span {max(x[6] for x in rows) - t0} ns")
for f, nm in enumerate(names):
    xs = [x[f] - t0 for x in rows if x[f]]
    if xs:
        print(f"{nm:9s} n={len(xs):3d} min {min(xs):7d} med {statistics.median(xs):9.0f} max {max(xs):7d}")
pre, post = st.tolist()
print(f"pre stamp -> first CTA start {(t0 - pre) / 1e3:.2f} us; last epilogue done -> post stamp "
      f"{(post - max(x[5] for x in rows)) / 1e3:.2f} us; pre -> post {(post - pre) / 1e3:.2f} us")
