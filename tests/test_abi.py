"""CPU checks of the C-ABI boundary: the library loads (no GPU needed) and
exports every function include/hgemm.h declares; argument errors are
reported synchronously without touching the device."""
import ctypes
import os

import pytest

from paper_conf_ipps_00020c20_b200 import binding


def test_library_exports_every_header_symbol():
    names = binding.header_functions()
    assert set(names) >= {"hgemm", "hgemm_status_string", "hgemm_set_config", "hgemm_get_last_config",
                          "hgemm_launch_count"}
    lib = binding.load_library()
    for nm in names:
        assert hasattr(lib, nm), nm
        assert ctypes.cast(getattr(lib, nm), ctypes.c_void_p).value


def test_status_strings():
    for code in range(4):
        s = binding.status_string(code)
        assert s.startswith("HGEMM")
    assert "unknown" in binding.status_string(99)


@pytest.mark.parametrize("args", [
    dict(m=-1), dict(n=-1), dict(k=-1), dict(transA="X"), dict(transB="q"), dict(out_dtype=7),
    dict(lda=1), dict(ldb=1), dict(ldc=1),
])
def test_invalid_arguments_rejected_synchronously(args):
    """Invalid values return HGEMM_ERR_INVALID_VALUE before any CUDA call (works without a GPU)."""
    lib = binding.load_library()
    a = dict(m=4, n=4, k=4, alpha=1.0, A=16, lda=4, B=16, ldb=4, beta=0.0, C=16, ldc=4, transA="N",
             transB="N", out_dtype=0)
    a.update(args)
    code = lib.hgemm(a["m"], a["n"], a["k"], a["alpha"], a["A"], a["lda"], a["B"], a["ldb"], a["beta"], a["C"],
                     a["ldc"], a["transA"].encode(), a["transB"].encode(), a["out_dtype"], None)
    assert code == 1


def test_null_pointers_rejected():
    lib = binding.load_library()
    assert lib.hgemm(4, 4, 4, 1.0, None, 4, 16, 4, 0.0, 16, 4, b"N", b"N", 0, None) == 1
    assert lib.hgemm(4, 4, 4, 1.0, 16, 4, 16, 4, 0.0, None, 4, b"N", b"N", 0, None) == 1
    # m == 0: no-op success even with NULL pointers
    assert lib.hgemm(0, 4, 4, 1.0, None, 1, None, 4, 0.0, None, 1, b"N", b"N", 0, None) == 0


def test_set_config_validation():
    lib = binding.load_library()
    assert lib.hgemm_set_config(ctypes.byref(binding._Config(9, 0, 0, 0))) == 1
    assert lib.hgemm_set_config(ctypes.byref(binding._Config(2, 96, 0, 0))) == 1
    assert lib.hgemm_set_config(ctypes.byref(binding._Config(2, 128, 8, 0))) == 0
    assert lib.hgemm_set_config(ctypes.byref(binding._Config(2, 128, 0, 0, 0, 3))) == 1   # stream_k 0..2
    assert lib.hgemm_set_config(ctypes.byref(binding._Config(3, 256, 0, 0, 0, 2))) == 0
    assert lib.hgemm_set_config(ctypes.byref(binding._Config(3, 512, 0, 0, 0, 1, 2))) == 0   # half_tail 0..2
    assert lib.hgemm_set_config(ctypes.byref(binding._Config(3, 512, 0, 0, 0, 1, 3))) == 1
    # flexible tile width: CTA pair, block_n 256, a multiple of 16 in [128, 256]
    assert lib.hgemm_set_config(ctypes.byref(binding._Config(3, 256, 0, 0, 0, 0, 0, 144))) == 0
    assert lib.hgemm_set_config(ctypes.byref(binding._Config(3, 256, 0, 0, 0, 0, 0, 136))) == 1
    assert lib.hgemm_set_config(ctypes.byref(binding._Config(3, 512, 0, 0, 0, 0, 0, 144))) == 1
    assert lib.hgemm_set_config(ctypes.byref(binding._Config(2, 256, 0, 0, 0, 0, 0, 144))) == 1
    assert lib.hgemm_set_config(ctypes.byref(binding._Config(3, 256, 0, 0, 0, 0, 0, 112))) == 1
    # HBM-streaming kernel: chunk width a multiple of 16 in [16, 256] (0 = auto)
    assert lib.hgemm_set_config(ctypes.byref(binding._Config(5, 112, 0, 0))) == 0
    assert lib.hgemm_set_config(ctypes.byref(binding._Config(5, 0, 0, 0))) == 0
    assert lib.hgemm_set_config(ctypes.byref(binding._Config(5, 100, 0, 0))) == 1
    assert lib.hgemm_set_config(ctypes.byref(binding._Config(5, 272, 0, 0))) == 1
    assert lib.hgemm_set_config(ctypes.byref(binding._Config(6, 0, 0, 0))) == 1
    assert lib.hgemm_set_config(None) == 0


def test_missing_library_raises(monkeypatch, tmp_path):
    monkeypatch.setattr(binding, "_lib", None)
    monkeypatch.setenv("HGEMM_LIB", os.path.join(str(tmp_path), "nope.so"))
    with pytest.raises(binding.HgemmError):
        binding.load_library()
    monkeypatch.setattr(binding, "_lib", None)


def test_kernel_sass_is_blackwell_native():
    """The fast path is tcgen05 + TMA (UTCHMMA / UTMALDG / LDTM in SASS), not legacy HMMA."""
    import shutil
    import subprocess
    exe = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"
    if not os.path.exists(exe):
        pytest.skip("cuobjdump not available")
    sass = subprocess.run([exe, "-sass", binding.lib_path()], capture_output=True, text=True).stdout
    assert "UTCHMMA" in sass and "UTMALDG" in sass and "LDTM" in sass
    assert "UTCHMMA.2CTA" in sass
    assert " HMMA" not in sass


def test_host_entry_validation():
    lib = binding.load_library()
    need = binding.host_workspace_size(100, 200, 300, "T", "N", "f16")
    # A (300 x 100 -> pitch 304), B (300 x 200 -> 304), C (100 x 200 -> 104), 256-byte aligned segments
    up = lambda x: (x + 255) // 256 * 256
    assert need == up(304 * 100 * 2) + up(304 * 200 * 2) + up(104 * 200 * 2)
    assert binding.host_workspace_size(-1, 2, 3, "N", "N", "f16") == 0
    # too small a workspace is an argument error (checked before any CUDA call)
    assert lib.hgemm_host(100, 200, 300, 1.0, 16, 300, 16, 300, 0.0, 16, 100, b"T", b"N", 0, 16, need - 1,
                          None) == 1
    assert lib.hgemm_host(100, 200, 300, 1.0, 16, 300, 16, 300, 0.0, 16, 100, b"T", b"N", 0, None, need,
                          None) == 1
    assert lib.hgemm_host(100, 200, 300, 1.0, 16, 10, 16, 300, 0.0, 16, 100, b"T", b"N", 0, 16, need, None) == 1
