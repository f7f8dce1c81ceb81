"""Thin ctypes binding over the C ABI of include/hgemm.h (argument marshalling only).

Every arithmetic step of the GEMM runs in the CUDA kernels of libhgemm.so;
this module only converts Python/torch arguments to pointers and sizes and
raises on a non-success status.  There is no CPU fallback: if the library
is missing, ``load_library()`` raises ``HgemmError``.
"""
from __future__ import annotations

import ctypes
import os
import re

_PKG = os.path.dirname(os.path.abspath(__file__))
_ROOT = os.path.dirname(_PKG)
HEADER = os.path.join(_ROOT, "include", "hgemm.h")

HGEMM_OUT_F16 = 0
HGEMM_OUT_F32 = 1
HGEMM_KERNEL = {"auto": 0, "simt": 1, "tc1": 2, "tc2": 3, "splitk": 4, "stream": 5}
HGEMM_COMPUTE = {"f32": 0, "f16": 1}

_lib = None


class HgemmError(RuntimeError):
    pass


class _Config(ctypes.Structure):
    _fields_ = [("kernel", ctypes.c_int32), ("block_n", ctypes.c_int32),
                ("group_m", ctypes.c_int32), ("max_ctas", ctypes.c_int32), ("splits", ctypes.c_int32),
                ("stream_k", ctypes.c_int32), ("half_tail", ctypes.c_int32), ("tile_n", ctypes.c_int32)]


class IpcHandle(ctypes.Structure):
    """hgemm_ipc_handle_t: cudaIpcMemHandle_t bytes + offset from the allocation base."""
    _fields_ = [("handle", ctypes.c_ubyte * 64), ("offset", ctypes.c_int64)]


def lib_path() -> str:
    return os.environ.get("HGEMM_LIB", os.path.join(_PKG, "libhgemm.so"))


def header_functions() -> list[str]:
    """Names of the functions include/hgemm.h declares."""
    txt = open(HEADER).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return re.findall(r"^\s*(?:const\s+)?[A-Za-z_][A-Za-z0-9_]*\s*\*?\s*(hgemm[A-Za-z0-9_]*)\s*\(",
                      txt, flags=re.M)


def load_library():
    """Load libhgemm.so (built by ``python -m paper_conf_ipps_00020c20_b200.build``)."""
    global _lib
    if _lib is not None:
        return _lib
    path = lib_path()
    if not os.path.exists(path):
        raise HgemmError(f"{path} is missing: build it with `python -m paper_conf_ipps_00020c20_b200.build` "
                         "(there is no CPU fallback)")
    lib = ctypes.CDLL(path)
    i64, f32, vp = ctypes.c_int64, ctypes.c_float, ctypes.c_void_p
    lib.hgemm.argtypes = [i64, i64, i64, f32, vp, i64, vp, i64, f32, vp, i64,
                          ctypes.c_char, ctypes.c_char, ctypes.c_int, vp]
    lib.hgemm.restype = ctypes.c_int
    lib.hgemm_ex.argtypes = [i64, i64, i64, f32, vp, i64, vp, i64, f32, vp, i64,
                             ctypes.c_char, ctypes.c_char, ctypes.c_int, ctypes.c_int, vp]
    lib.hgemm_ex.restype = ctypes.c_int
    lib.hgemm_status_string.argtypes = [ctypes.c_int]
    lib.hgemm_status_string.restype = ctypes.c_char_p
    lib.hgemm_set_config.argtypes = [ctypes.POINTER(_Config)]
    lib.hgemm_set_config.restype = ctypes.c_int
    lib.hgemm_get_last_config.argtypes = [ctypes.POINTER(_Config)]
    lib.hgemm_get_last_config.restype = ctypes.c_int
    lib.hgemm_host.argtypes = [i64, i64, i64, f32, vp, i64, vp, i64, f32, vp, i64,
                               ctypes.c_char, ctypes.c_char, ctypes.c_int, vp, ctypes.c_size_t, vp]
    lib.hgemm_host.restype = ctypes.c_int
    lib.hgemm_host_workspace_size.argtypes = [i64, i64, i64, ctypes.c_char, ctypes.c_char, ctypes.c_int]
    lib.hgemm_host_workspace_size.restype = ctypes.c_size_t
    lib.hgemm_set_probe.argtypes = [vp]
    lib.hgemm_set_probe.restype = ctypes.c_int
    lib.hgemm_launch_count.argtypes = []
    lib.hgemm_launch_count.restype = ctypes.c_int64
    i32, pi64 = ctypes.c_int32, ctypes.POINTER(ctypes.c_int64)
    lib.hgemm_allgather_a.argtypes = [i64, i64, i64, f32, vp, i64, ctypes.POINTER(vp), pi64, i32, i32,
                                      vp, i64, f32, vp, i64, ctypes.c_char, ctypes.c_int,
                                      vp, i64, i64, vp]
    lib.hgemm_allgather_a.restype = ctypes.c_int
    lib.hgemm_allgather_plan.argtypes = [i64, pi64, i32, i32, i64, pi64, i64, pi64]
    lib.hgemm_allgather_plan.restype = ctypes.c_int
    lib.hgemm_ipc_get_handle.argtypes = [vp, ctypes.POINTER(IpcHandle)]
    lib.hgemm_ipc_get_handle.restype = ctypes.c_int
    lib.hgemm_ipc_open.argtypes = [ctypes.POINTER(IpcHandle), ctypes.POINTER(vp)]
    lib.hgemm_ipc_open.restype = ctypes.c_int
    lib.hgemm_ipc_close.argtypes = [vp]
    lib.hgemm_ipc_close.restype = ctypes.c_int
    _lib = lib
    return lib


def status_string(code: int) -> str:
    return load_library().hgemm_status_string(int(code)).decode()


def _check(code: int):
    if code != 0:
        raise HgemmError(status_string(code))


def set_config(kernel: str | int = "auto", block_n: int = 0, group_m: int = 0, max_ctas: int = 0,
               splits: int = 0, stream_k: int = 0, half_tail: int = 0, tile_n: int = 0):
    """Force a kernel choice (tests / bench).  ``set_config()`` restores automatic selection."""
    lib = load_library()
    kern = HGEMM_KERNEL[kernel] if isinstance(kernel, str) else int(kernel)
    if (kern == 0 and not block_n and not group_m and not max_ctas and not splits and not stream_k
            and not half_tail and not tile_n):
        _check(lib.hgemm_set_config(None))
    else:
        _check(lib.hgemm_set_config(ctypes.byref(_Config(kern, block_n, group_m, max_ctas, splits,
                                                                  stream_k, half_tail, tile_n))))


def set_probe(buf=None):
    """Enable (a >= 4-element int64 CUDA tensor) or disable (None) the kernel clock probe."""
    _check(load_library().hgemm_set_probe(_ptr(buf) or None))


def probe_clock_ghz(buf) -> float:
    """SM clock of the last probed launch, from {clk0, ns0, clk1, ns1}."""
    v = [int(x) for x in buf[:4].cpu().tolist()]
    return (v[2] - v[0]) / max(v[3] - v[1], 1)


def get_stats() -> dict:
    lib = load_library()
    c = _Config()
    _check(lib.hgemm_get_last_config(ctypes.byref(c)))
    inv = {v: k for k, v in HGEMM_KERNEL.items()}
    return {"last_kernel": inv.get(c.kernel, c.kernel), "block_n": c.block_n, "group_m": c.group_m,
            "max_ctas": c.max_ctas, "splits": c.splits, "stream_k": c.stream_k, "half_tail": c.half_tail,
            "tile_n": c.tile_n, "launches": int(lib.hgemm_launch_count())}


def _ptr(x) -> int:
    if x is None:
        return 0
    if isinstance(x, int):
        return x
    return int(x.data_ptr())


def _stream(stream) -> int:
    if stream is None:
        import torch
        return int(torch.cuda.current_stream().cuda_stream)
    if isinstance(stream, int):
        return stream
    return int(stream.cuda_stream)


def _out_code(out_dtype) -> int:
    if out_dtype in (HGEMM_OUT_F16, HGEMM_OUT_F32):
        return int(out_dtype)
    s = str(out_dtype)
    if s in ("f16", "float16", "torch.float16", "half"):
        return HGEMM_OUT_F16
    if s in ("f32", "float32", "torch.float32", "float"):
        return HGEMM_OUT_F32
    raise HgemmError(f"unsupported out_dtype {out_dtype!r}")


def hgemm(m, n, k, alpha, A, lda, B, ldb, beta, C, ldc, transA="N", transB="N",
          out_dtype=HGEMM_OUT_F16, stream=None):
    """C <- alpha*op(A)*op(B) + beta*C, column-major (include/hgemm.h).

    A, B, C: device pointers (int) or tensors (their data_ptr() is used).
    stream: None (torch's current stream), an int handle, or a torch.cuda.Stream."""
    lib = load_library()
    code = lib.hgemm(int(m), int(n), int(k), float(alpha), _ptr(A), int(lda), _ptr(B), int(ldb),
                     float(beta), _ptr(C), int(ldc), transA.encode()[:1], transB.encode()[:1],
                     _out_code(out_dtype), _stream(stream))
    _check(code)


def hgemm_ex(m, n, k, alpha, A, lda, B, ldb, beta, C, ldc, transA="N", transB="N",
             out_dtype=HGEMM_OUT_F16, compute="f32", stream=None):
    """hgemm() with an explicit accumulation type (include/hgemm.h hgemm_ex):
    compute "f32" (FP32 accumulation, as hgemm) or "f16" (FP16 accumulation on the
    tensor cores, the paper's HMMA.1688.F16 mode; FP16 output only)."""
    lib = load_library()
    comp = HGEMM_COMPUTE[compute] if isinstance(compute, str) else int(compute)
    code = lib.hgemm_ex(int(m), int(n), int(k), float(alpha), _ptr(A), int(lda), _ptr(B), int(ldb),
                        float(beta), _ptr(C), int(ldc), transA.encode()[:1], transB.encode()[:1],
                        _out_code(out_dtype), comp, _stream(stream))
    _check(code)


def host_workspace_size(m, n, k, transA="N", transB="N", out_dtype=HGEMM_OUT_F16) -> int:
    return int(load_library().hgemm_host_workspace_size(int(m), int(n), int(k), transA.encode()[:1],
                                                        transB.encode()[:1], _out_code(out_dtype)))


def hgemm_host(m, n, k, alpha, A, lda, B, ldb, beta, C, ldc, transA="N", transB="N",
               out_dtype=HGEMM_OUT_F16, workspace=None, workspace_bytes=None, stream=None):
    """Host-buffer variant (include/hgemm.h): A, B, C are HOST pointers / CPU tensors
    (pinned for copy-compute overlap); `workspace` is device memory of at least
    host_workspace_size(...) bytes.  Synchronous."""
    lib = load_library()
    if workspace_bytes is None:
        workspace_bytes = int(workspace.numel() * workspace.element_size()) if workspace is not None else 0
    code = lib.hgemm_host(int(m), int(n), int(k), float(alpha), _ptr(A), int(lda), _ptr(B), int(ldb), float(beta),
                          _ptr(C), int(ldc), transA.encode()[:1], transB.encode()[:1], _out_code(out_dtype),
                          _ptr(workspace), int(workspace_bytes), _stream(stream))
    _check(code)


def _as_colmajor_op_of_transpose(X):
    """(trans, ld, tensor) such that op(buffer) == X^T in the column-major ABI."""
    r, c = X.shape
    s0, s1 = X.stride()
    if (s1 == 1 or c <= 1) and (s0 >= max(c, 1) or r <= 1):
        return "N", max(s0 if r > 1 else c, c, 1), X
    if (s0 == 1 or r <= 1) and (s1 >= max(r, 1) or c <= 1):
        return "T", max(s1 if c > 1 else r, r, 1), X
    Xc = X.contiguous()
    return "N", max(c, 1), Xc


def hgemm_torch(A, B, C=None, *, alpha=1.0, beta=0.0, out_dtype=None, stream=None):
    """Row-major torch front end: returns C = alpha * A @ B + beta * C.

    A: (M, K) float16 CUDA tensor, B: (K, N) float16 CUDA tensor (any strides;
    a transposed view such as ``W.t()`` is consumed without a copy).  C: (M, N)
    float16/float32, row-major contiguous rows, updated in place when given.
    The row-major product is the column-major ABI call C^T = B^T A^T:
    hgemm(m=N, n=M, k=K, A=B, B=A, C=C)."""
    import torch
    if A.dim() != 2 or B.dim() != 2 or A.shape[1] != B.shape[0]:
        raise HgemmError(f"shape mismatch {tuple(A.shape)} @ {tuple(B.shape)}")
    if A.dtype != torch.float16 or B.dtype != torch.float16:
        raise HgemmError("A and B must be torch.float16")
    M, K = A.shape
    N = B.shape[1]
    if C is None:
        if beta != 0.0:
            raise HgemmError("beta != 0 needs C")
        C = torch.empty((M, N), dtype=out_dtype or torch.float16, device=A.device)
    if C.shape != (M, N) or C.dtype not in (torch.float16, torch.float32):
        raise HgemmError("C must be (M, N) float16 or float32")
    if N > 1 and C.stride(1) != 1:
        raise HgemmError("C rows must be contiguous")
    ldc = max(C.stride(0) if M > 1 else N, N, 1)
    tA, lda, Bt = _as_colmajor_op_of_transpose(B)   # op(A_abi) = B^T  (N x K)
    tB, ldb, At = _as_colmajor_op_of_transpose(A)   # op(B_abi) = A^T  (K x M)
    out = HGEMM_OUT_F32 if C.dtype == torch.float32 else HGEMM_OUT_F16
    hgemm(N, M, K, alpha, Bt, lda, At, ldb, beta, C, ldc, tA, tB, out, stream)
    return C


def _i64_array(vals):
    return (ctypes.c_int64 * len(vals))(*[int(v) for v in vals])


def allgather_plan(m, row_splits, rank, chunk_rows):
    """Chunk order of hgemm_allgather_a (host only): list of (chunk, src_rank, row0, row1)."""
    lib = load_library()
    world = len(row_splits) - 1
    rs = _i64_array(row_splits)
    cnt = ctypes.c_int64(0)
    _check(lib.hgemm_allgather_plan(int(m), rs, int(world), int(rank), int(chunk_rows), None, 0, ctypes.byref(cnt)))
    ops = (ctypes.c_int64 * (4 * max(cnt.value, 1)))()
    _check(lib.hgemm_allgather_plan(int(m), rs, int(world), int(rank), int(chunk_rows), ops, cnt.value,
                                    ctypes.byref(cnt)))
    return [tuple(ops[4 * i:4 * i + 4]) for i in range(cnt.value)]


def hgemm_allgather_a(m, n, k, alpha, A, lda, A_peers, row_splits, rank, B, ldb, beta, C, ldc,
                      transB="N", out_dtype=HGEMM_OUT_F16, *, workspace, chunk_rows, stream=None):
    """All-gather of op(A) rows fused with the GEMM in one kernel (include/hgemm.h hgemm_allgather_a).

    A: this rank's full-size gather buffer (transA = 'T' layout); A_peers: the
    other ranks' gather buffers as device pointers/tensors (entry `rank` ignored);
    workspace: int32 CUDA tensor of >= 1 + ceil(m/chunk_rows) entries."""
    lib = load_library()
    world = len(row_splits) - 1
    if len(A_peers) != world:
        raise HgemmError("A_peers needs one entry per rank")
    peers = (ctypes.c_void_p * world)(*[_ptr(x) or None for x in A_peers])
    nws = int(workspace.numel()) if hasattr(workspace, "numel") else 0
    code = lib.hgemm_allgather_a(int(m), int(n), int(k), float(alpha), _ptr(A), int(lda), peers,
                                 _i64_array(row_splits), int(world), int(rank), _ptr(B), int(ldb), float(beta),
                                 _ptr(C), int(ldc), transB.encode()[:1], _out_code(out_dtype), _ptr(workspace), nws,
                                 int(chunk_rows), _stream(stream))
    _check(code)


def ipc_get_handle(buf) -> bytes:
    """72 bytes (hgemm_ipc_handle_t) naming the device buffer `buf` for other processes."""
    h = IpcHandle()
    _check(load_library().hgemm_ipc_get_handle(_ptr(buf), ctypes.byref(h)))
    return bytes(ctypes.string_at(ctypes.addressof(h), ctypes.sizeof(h)))


def ipc_open(handle: bytes) -> int:
    """Map a peer's buffer (from ipc_get_handle) into this process; returns its device pointer."""
    if len(handle) != ctypes.sizeof(IpcHandle):
        raise HgemmError("bad IPC handle size")
    h = IpcHandle.from_buffer_copy(handle)
    out = ctypes.c_void_p()
    _check(load_library().hgemm_ipc_open(ctypes.byref(h), ctypes.byref(out)))
    return int(out.value)


def ipc_close(ptr: int):
    _check(load_library().hgemm_ipc_close(ctypes.c_void_p(int(ptr))))
