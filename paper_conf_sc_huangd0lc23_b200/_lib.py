"""ctypes loader of libcuszp.so (the C ABI of include/cuszp.h).

Fails loudly: there is no CPU fallback anywhere in this package.  If the
shared library is missing it is built in-tree with nvcc; if that is not
possible an ImportError-like RuntimeError is raised.
"""
from __future__ import annotations

import ctypes as C
import os
import threading

from . import build as _build

LIB_PATH = _build.LIB

OK, EINVAL, ECUDA, ERANGE, ECORRUPT, ENOSPACE = 0, 1, 2, 3, 4, 5
STATUS_NAMES = {0: "OK", 1: "EINVAL", 2: "ECUDA", 3: "ERANGE", 4: "ECORRUPT", 5: "ENOSPACE"}

# every symbol include/cuszp.h declares (checked by tests/test_abi_symbols.py)
SYMBOLS = (
    "cuszp_max_compressed_bytes", "cuszp_compressed_bytes_from_F", "cuszp_workspace_bytes",
    "cuszp_range", "cuszp_compress", "cuszp_compress_minmax", "cuszp_decompress",
    "cuszp_last_status", "cuszp_read_header", "cuszp_compress_host", "cuszp_decompress_host",
    "cuszp_status_string", "cuszp_version", "cuszp_quality_workspace_bytes", "cuszp_quality",
    "cuszp_compress_host_async", "cuszp_decompress_host_async",
    "cuszp_compress_L", "cuszp_compress_minmax_L", "cuszp_decompress_L", "cuszp_max_compressed_bytes_L",
    "cuszp_compress_ex", "cuszp_decompress_ex",
    "cuszp_num_blocks_md", "cuszp_max_compressed_bytes_md", "cuszp_workspace_bytes_md", "cuszp_compress_md",
    "cuszp_decompress_md", "cuszp_container_put",
)

_lock = threading.Lock()
_lib = None


class CuszpError(RuntimeError):
    def __init__(self, status: int, where: str):
        super().__init__(f"{where}: {STATUS_NAMES.get(status, status)}")
        self.status = status


def _declare(h):
    sz, vp, i32, f32 = C.c_size_t, C.c_void_p, C.c_int, C.c_float
    h.cuszp_max_compressed_bytes.argtypes = [sz]
    h.cuszp_max_compressed_bytes.restype = sz
    h.cuszp_compressed_bytes_from_F.argtypes = [vp, sz]
    h.cuszp_compressed_bytes_from_F.restype = sz
    h.cuszp_workspace_bytes.argtypes = [sz]
    h.cuszp_workspace_bytes.restype = sz
    h.cuszp_range.argtypes = [vp, sz, vp, vp, sz, vp]
    h.cuszp_range.restype = i32
    h.cuszp_compress.argtypes = [vp, sz, f32, i32, vp, sz, vp, vp, sz, vp]
    h.cuszp_compress.restype = i32
    h.cuszp_compress_minmax.argtypes = [vp, sz, f32, vp, i32, vp, sz, vp, vp, sz, vp]
    h.cuszp_compress_minmax.restype = i32
    h.cuszp_decompress.argtypes = [vp, sz, vp, sz, vp, sz, vp]
    h.cuszp_decompress.restype = i32
    h.cuszp_last_status.argtypes = [vp, vp]
    h.cuszp_last_status.restype = i32
    h.cuszp_read_header.argtypes = [vp, vp, vp]
    h.cuszp_read_header.restype = i32
    h.cuszp_compress_host.argtypes = [vp, sz, f32, i32, vp, sz, vp, vp, vp, vp, sz, vp]
    h.cuszp_compress_host.restype = i32
    h.cuszp_decompress_host.argtypes = [vp, sz, vp, sz, vp, vp, vp, sz, vp]
    h.cuszp_decompress_host.restype = i32
    h.cuszp_status_string.argtypes = [i32]
    h.cuszp_status_string.restype = C.c_char_p
    h.cuszp_quality_workspace_bytes.argtypes = []
    h.cuszp_quality_workspace_bytes.restype = sz
    h.cuszp_quality.argtypes = [vp, vp, sz, C.c_double, vp, vp, sz, vp]
    h.cuszp_quality.restype = i32
    h.cuszp_compress_host_async.argtypes = [vp, sz, f32, i32, vp, sz, vp, vp, vp, vp, sz, vp]
    h.cuszp_compress_host_async.restype = i32
    h.cuszp_decompress_host_async.argtypes = [vp, sz, vp, sz, vp, vp, vp, sz, vp]
    h.cuszp_decompress_host_async.restype = i32
    h.cuszp_compress_ex.argtypes = [vp, sz, f32, i32, i32, i32, vp, sz, vp, vp, sz, vp]
    h.cuszp_compress_ex.restype = i32
    h.cuszp_decompress_ex.argtypes = [vp, sz, vp, sz, i32, i32, vp, sz, vp]
    h.cuszp_decompress_ex.restype = i32
    h.cuszp_max_compressed_bytes_L.argtypes = [sz, i32]
    h.cuszp_max_compressed_bytes_L.restype = sz
    h.cuszp_compress_L.argtypes = [vp, sz, f32, i32, i32, vp, sz, vp, vp, sz, vp]
    h.cuszp_compress_L.restype = i32
    h.cuszp_compress_minmax_L.argtypes = [vp, sz, f32, vp, i32, i32, vp, sz, vp, vp, sz, vp]
    h.cuszp_compress_minmax_L.restype = i32
    h.cuszp_decompress_L.argtypes = [vp, sz, vp, sz, i32, vp, sz, vp]
    h.cuszp_decompress_L.restype = i32
    for f in ("cuszp_num_blocks_md", "cuszp_max_compressed_bytes_md", "cuszp_workspace_bytes_md"):
        getattr(h, f).argtypes = [sz, sz, sz, i32]
        getattr(h, f).restype = sz
    h.cuszp_compress_md.argtypes = [vp, sz, sz, sz, i32, f32, i32, vp, sz, vp, vp, sz, vp]
    h.cuszp_compress_md.restype = i32
    h.cuszp_decompress_md.argtypes = [vp, sz, vp, sz, sz, sz, i32, vp, sz, vp]
    h.cuszp_decompress_md.restype = i32
    h.cuszp_container_put.argtypes = [vp, vp, C.c_uint, C.c_uint, vp, i32, vp]
    h.cuszp_container_put.restype = i32
    h.cuszp_version.argtypes = []
    h.cuszp_version.restype = i32


def lib():
    """The loaded library (built in-tree first if absent or stale)."""
    global _lib
    with _lock:
        if _lib is None:
            if _build.needs_build():
                try:
                    _build.build()
                except Exception as e:  # no silent fallback
                    if not os.path.exists(LIB_PATH):
                        raise RuntimeError(f"libcuszp.so is missing and cannot be built: {e}") from e
            h = C.CDLL(LIB_PATH)
            _declare(h)
            _lib = h
    return _lib


def check(status: int, where: str) -> None:
    if status != OK:
        raise CuszpError(status, where)
