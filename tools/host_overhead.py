"""Host cost of one hgemm() call (enqueue only) and the device time of tiny GEMMs,
eagerly and replayed from a CUDA graph (the launch-bound regime of BASELINE config 1)."""
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_00020c20_b200 import binding  # noqa: E402

lib = binding.load_library()
for (m, n, k) in [(256, 256, 256), (1024, 1024, 1024)]:
    A = torch.randn(m, k, device="cuda").half()
    B = torch.randn(n, k, device="cuda").half()
    C = torch.empty(n, m, device="cuda", dtype=torch.float32)
    s = torch.cuda.current_stream()
    h = s.cuda_stream
    pa, pb, pc = A.data_ptr(), B.data_ptr(), C.data_ptr()
    for _ in range(50):
        lib.hgemm(m, n, k, 1.0, pa, k, pb, k, 0.0, pc, m, b"T", b"N", 1, h)
    torch.cuda.synchronize()
    N = 2000
    t0 = time.perf_counter()
    for _ in range(N):
        lib.hgemm(m, n, k, 1.0, pa, k, pb, k, 0.0, pc, m, b"T", b"N", 1, h)
    t1 = time.perf_counter()
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    host_us = (t1 - t0) / N * 1e6
    eager_us = (t2 - t0) / N * 1e6
    # CUDA graph of 20 calls
    g = torch.cuda.CUDAGraph()
    cap = torch.cuda.Stream()
    with torch.cuda.stream(cap):
        with torch.cuda.graph(g, stream=cap):
            for _ in range(20):
                lib.hgemm(m, n, k, 1.0, pa, k, pb, k, 0.0, pc, m, b"T", b"N", 1, cap.cuda_stream)
    g.replay()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(50):
        g.replay()
    e1.record()
    torch.cuda.synchronize()
    graph_us = e0.elapsed_time(e1) * 1e3 / (50 * 20)
    print(f"{m}x{n}x{k}: host enqueue {host_us:.1f} us/call (ctypes), eager throughput {eager_us:.1f} us/call, "
          f"graph replay {graph_us:.1f} us/GEMM ({2.0*m*n*k/graph_us/1e6:.1f} TFLOP/s), kernel {binding.get_stats()['last_kernel']}")
