"""Where the fixed time of a launch goes (experiments; library built with -DHGEMM_TRACE).

One-thread stamp kernels write %globaltimer right before and right after the
hgemm launch; the traced kernel records every CTA's entry and end.  Prints
entry - pre (launch latency), the CTA span, and post - last end (teardown).

    HGEMM_LIB=.../libhgemm_trace.so python tools/launch_gap.py
"""
import ctypes
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding, build  # noqa: E402

mb = ctypes.CDLL(build.build_microbench())
mb.mb_stamp.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
w = torch.empty(64 * 1024 * 1024, device="cuda")
for (m, n, k, beta) in [(256, 256, 256, 0.0), (4096, 1024, 4096, 1.0), (1024, 4096, 2048, 1.0),
                        (4096, 4096, 1024, 1.0), (16384, 64, 4096, 0.0)]:
    A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
    B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
    C = (torch.rand(n, m, device="cuda") * 2 - 1).half()
    st = torch.zeros(2, dtype=torch.int64, device="cuda")
    probe = torch.zeros(264 + 2 * 8 * 160, dtype=torch.int64, device="cuda")
    s = torch.cuda.current_stream().cuda_stream
    for warm in (False, True):
        for i in range(4):
            if not warm:
                w.zero_()
            binding.set_probe(probe if i == 3 else None)
            mb.mb_stamp(st.data_ptr(), s)
            binding.hgemm(m, n, k, 1.0, A, k, B, k, beta, C, m, "T", "N", "f16")
            mb.mb_stamp(st.data_ptr() + 8, s)
        torch.cuda.synchronize()
        binding.set_probe(None)
        pre, post = st.tolist()
        v = probe.view(-1).tolist()
        rows = [v[264 + 8 * b: 266 + 8 * b] for b in range(160) if v[264 + 8 * b]]
        if not rows:
            print(f"{m}x{n}x{k}: no CTA trace ({binding.get_stats()['last_kernel']} kernel)")
            break
        e0 = min(r[0] for r in rows)
        e1 = max(r[1] for r in rows)
        print(f"{m}x{n}x{k} beta={beta} {'warm' if warm else 'cold'} [{binding.get_stats()['last_kernel']}]: "
              f"pre->first entry {(e0 - pre) / 1e3:6.2f} us, last entry {(max(r[0] for r in rows) - pre) / 1e3:6.2f}, "
              f"CTA span {(e1 - e0) / 1e3:7.2f} us, last end->post {(post - e1) / 1e3:6.2f} us, "
              f"pre->post {(post - pre) / 1e3:7.2f} us", flush=True)

# the same stamps around cuBLAS and around an empty kernel of our launch shape
mb.mb_empty.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p]
st = torch.zeros(2, dtype=torch.int64, device="cuda")
s = torch.cuda.current_stream().cuda_stream
for (m, n, k, beta) in [(256, 256, 256, 0.0), (4096, 1024, 4096, 1.0), (4096, 4096, 1024, 1.0)]:
    A = (torch.rand(m, k, device="cuda") * 2 - 1).half()
    B = (torch.rand(n, k, device="cuda") * 2 - 1).half()
    C = (torch.rand(n, m, device="cuda") * 2 - 1).half()
    for i in range(4):
        w.zero_()
        mb.mb_stamp(st.data_ptr(), s)
        torch.addmm(C, B, A.t(), beta=beta, out=C)
        mb.mb_stamp(st.data_ptr() + 8, s)
    torch.cuda.synchronize()
    pre, post = st.tolist()
    print(f"cuBLAS {m}x{n}x{k} beta={beta} cold: pre->post {(post - pre) / 1e3:7.2f} us", flush=True)
for (grid, block, smem, cl) in [(148, 320, 236992 - 4544, 2), (148, 320, 0, 2), (148, 320, 0, 1), (148, 256, 213 * 1024, 4)]:
    for i in range(4):
        w.zero_()
        mb.mb_stamp(st.data_ptr(), s)
        rc = mb.mb_empty(grid, block, smem, cl, None, s)
        mb.mb_stamp(st.data_ptr() + 8, s)
    torch.cuda.synchronize()
    pre, post = st.tolist()
    print(f"empty kernel grid {grid} block {block} smem {smem} cluster {cl} (rc {rc}): pre->post {(post - pre) / 1e3:7.2f} us",
          flush=True)
