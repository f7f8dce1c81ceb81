import sys, numpy as np
sys.path.insert(0, ".")
from paper_conf_ipps_00020c20_b200 import binding, inputs
from tests.gpu_util import GpuCase
m, n, mc = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
beta = float(sys.argv[4]); out = sys.argv[5]
k = 520
C = inputs.uniform_f16(m, n, 27).astype(np.float32 if out == "f32" else np.float16)
opA, opB = inputs.uniform_f16(m, k, 25), inputs.uniform_f16(k, n, 26)
binding.set_config("tc2", block_n=512, max_ctas=mc, stream_k=1)
case = GpuCase(opA, opB, "T", "N", 1.0, beta, C=C, out=out, pad=(8, 16, 8))
got = case.run_gpu()
print("ok", case.stats)
