"""B200-native (sm_100a) half-precision GEMM: C = alpha*op(A)*op(B) + beta*C.

Public API (thin ctypes binding over the C ABI in include/hgemm.h):
  hgemm(...)          -- same arguments as the C call, device pointers
  hgemm_ex(...)       -- hgemm with an explicit accumulation type (FP32, or the paper's FP16)
  hgemm_torch(...)    -- row-major torch tensors (operand swap to the column-major ABI)
  hgemm_sharded(...)  -- N-slab sharded multi-GPU path (torch.distributed / NCCL)
The shared library is loaded on first use; a missing library raises.
"""
from .binding import (HGEMM_OUT_F16, HGEMM_OUT_F32, HgemmError, hgemm, hgemm_ex, hgemm_host, hgemm_torch,  # noqa: F401
                      host_workspace_size,
                      lib_path, load_library, status_string, set_config, get_stats,
                      set_probe, probe_clock_ghz)
from .sharded import hgemm_sharded, hgemm_sharded_overlapped, slab_bounds  # noqa: F401
