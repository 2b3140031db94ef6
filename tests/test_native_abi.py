"""CPU tests of the native comparator library (benchmarks/native/libuc_nccl_dev.so):
it loads, exports every function its header declares, and rejects bad arguments before touching
NCCL or the GPU.  Its numerics are GPU tests (tests/test_gpu_native.py)."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "benchmarks", "native", "nccl_dev_jacobi.h")


def _lib():
    from benchmarks import nccl_dev_bench
    try:
        return nccl_dev_bench.load()
    except ImportError as e:
        pytest.fail(str(e))


def test_exports_every_declared_function():
    lib = _lib()
    names = re.findall(r"^\s*(?:int|const char\*)\s+(ucn_\w+)\s*\(", open(HDR).read(), re.M)
    assert len(names) == 7
    for n in names:
        assert hasattr(lib, n), n


def test_argument_errors_without_gpu():
    lib = _lib()
    h = ctypes.c_void_p()
    uid = ctypes.create_string_buffer(128)
    for args in [(0, 1, uid, 6, 4, -1, -1), (0, 1, uid, 16, 0, -1, -1), (1, 1, uid, 16, 4, -1, -1),
                 (0, 2, uid, 16, 4, 2, -1), (0, 1, None, 16, 4, -1, -1)]:
        assert lib.ucn_create(*args, ctypes.byref(h)) == 1
        assert b"ucn_create" in lib.ucn_last_error()
    assert lib.ucn_run(None, 1, None) == 1
    assert lib.ucn_destroy(None) == 0
