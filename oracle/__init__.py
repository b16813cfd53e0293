"""ctypes front end of the C++ oracle (oracle/cuszp_oracle.cpp).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and
bench.py's cpu_baseline / ``--impl reference`` legs -- never by the product
package.  It shares no code with paper_conf_sc_huangd0lc23_b200/.

Every function is a thin marshalling layer over the C++ function of the
same name (numpy arrays in, numpy arrays out); all arithmetic is in C++.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "cuszp_oracle.cpp")
LIB = os.path.join(HERE, "libcuszp_oracle.so")

OK, EINVAL, ERANGE, ECORRUPT, ENOSPACE = 0, 1, 3, 4, 5
ABS, REL = 0, 1
HEADER_BYTES = 32
L = 32

_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile the oracle with plain IEEE settings (no contraction, no fast math)."""
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < max(
        os.path.getmtime(SRC), os.path.getmtime(os.path.join(HERE, "cuszp_oracle.h"))
    ):
        cmd = [
            "g++", "-std=c++17", "-O2", "-ffp-contract=off", "-fno-fast-math",
            "-fno-finite-math-only", "-shared", "-fPIC", "-o", LIB + ".tmp", SRC,
        ]
        subprocess.run(cmd, check=True)
        os.replace(LIB + ".tmp", LIB)
    return LIB


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            h = C.CDLL(LIB)
            u64, f32, i32, vp = C.c_uint64, C.c_float, C.c_int, C.c_void_p
            h.oracle_value_range.argtypes = [vp, C.c_size_t, vp, vp]
            h.oracle_prequantize.argtypes = [vp, C.c_size_t, f32, vp]
            h.oracle_prequantize.restype = i32
            h.oracle_block_lorenzo.argtypes = [vp, C.c_size_t, vp]
            h.oracle_bit_length.argtypes = [C.c_uint32]
            h.oracle_bit_length.restype = i32
            h.oracle_block_bytes.argtypes = [i32, i32]
            h.oracle_block_bytes.restype = u64
            h.oracle_exclusive_scan.argtypes = [vp, C.c_size_t, vp]
            h.oracle_encode_block.argtypes = [vp, vp]
            h.oracle_encode_block.restype = i32
            h.oracle_decode_block.argtypes = [vp, i32, vp]
            h.oracle_max_compressed_bytes.argtypes = [u64]
            h.oracle_max_compressed_bytes.restype = u64
            h.oracle_compress.argtypes = [vp, u64, f32, i32, vp, u64, vp]
            h.oracle_compress.restype = i32
            h.oracle_compress_minmax.argtypes = [vp, u64, f32, vp, i32, vp, u64, vp]
            h.oracle_compress_minmax.restype = i32
            h.oracle_decompress.argtypes = [vp, u64, vp, u64]
            h.oracle_decompress.restype = i32
            h.oracle_quality.argtypes = [vp, vp, u64, C.c_double, vp, vp]
            h.oracle_num_blocks_md.argtypes = [u64, u64, u64, i32]
            h.oracle_num_blocks_md.restype = u64
            h.oracle_max_compressed_bytes_md.argtypes = [u64, u64, u64, i32]
            h.oracle_max_compressed_bytes_md.restype = u64
            h.oracle_block_lorenzo_md.argtypes = [vp, i32, vp]
            h.oracle_compress_md.argtypes = [vp, u64, u64, u64, i32, f32, i32, vp, u64, vp]
            h.oracle_compress_md.restype = i32
            h.oracle_decompress_md.argtypes = [vp, u64, vp, u64, u64, u64, i32]
            h.oracle_decompress_md.restype = i32
            h.oracle_block_lorenzo_L.argtypes = [vp, C.c_size_t, i32, vp]
            h.oracle_encode_block_L.argtypes = [vp, i32, vp]
            h.oracle_encode_block_L.restype = i32
            h.oracle_decode_block_L.argtypes = [vp, i32, i32, vp]
            h.oracle_max_compressed_bytes_L.argtypes = [u64, i32]
            h.oracle_max_compressed_bytes_L.restype = u64
            h.oracle_compress_L.argtypes = [vp, u64, f32, i32, i32, vp, u64, vp]
            h.oracle_compress_L.restype = i32
            h.oracle_compress_minmax_L.argtypes = [vp, u64, f32, vp, i32, i32, vp, u64, vp]
            h.oracle_compress_minmax_L.restype = i32
            h.oracle_compress_ex.argtypes = [vp, u64, f32, i32, i32, i32, vp, u64, vp]
            h.oracle_compress_ex.restype = i32
            _lib = h
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(C.c_void_p)


def _f32(x) -> np.ndarray:
    return np.ascontiguousarray(x, dtype=np.float32)


def value_range(x) -> tuple[float, float]:
    x = _f32(x)
    mn, mx = np.zeros(1, np.float32), np.zeros(1, np.float32)
    lib().oracle_value_range(_ptr(x), x.size, _ptr(mn), _ptr(mx))
    return float(mn[0]), float(mx[0])


def prequantize(x, eb_abs: float):
    x = _f32(x)
    q = np.zeros(x.size, np.int32)
    st = lib().oracle_prequantize(_ptr(x), x.size, np.float32(eb_abs), _ptr(q))
    return st, q


def block_lorenzo(q) -> np.ndarray:
    q = np.ascontiguousarray(q, dtype=np.int32)
    assert q.size % L == 0
    out = np.zeros_like(q)
    lib().oracle_block_lorenzo(_ptr(q), q.size // L, _ptr(out))
    return out


def bit_length(m: int) -> int:
    return lib().oracle_bit_length(int(m))


def block_bytes(F: int, Lb: int = L) -> int:
    return int(lib().oracle_block_bytes(F, Lb))


def exclusive_scan(cmpl) -> np.ndarray:
    a = np.ascontiguousarray(cmpl, dtype=np.uint64)
    out = np.zeros_like(a)
    lib().oracle_exclusive_scan(_ptr(a), a.size, _ptr(out))
    return out


def encode_block(l) -> tuple[int, bytes]:
    l = np.ascontiguousarray(l, dtype=np.int32)
    assert l.size == L
    buf = np.zeros(100, np.uint8)
    F = lib().oracle_encode_block(_ptr(l), _ptr(buf))
    return F, bytes(buf[: block_bytes(F)])


def decode_block(payload: bytes, F: int) -> np.ndarray:
    buf = np.zeros(100, np.uint8)
    buf[: len(payload)] = np.frombuffer(payload, np.uint8)
    out = np.zeros(L, np.int32)
    lib().oracle_decode_block(_ptr(buf), int(F), _ptr(out))
    return out


def max_compressed_bytes(n: int) -> int:
    return int(lib().oracle_max_compressed_bytes(int(n)))


def compress(x, eb: float, mode: int = REL) -> tuple[int, np.ndarray]:
    """Returns (status, stream bytes as uint8 array)."""
    x = _f32(x).ravel()
    cap = max_compressed_bytes(x.size)
    out = np.zeros(cap, np.uint8)
    nbytes = np.zeros(1, np.uint64)
    st = lib().oracle_compress(_ptr(x), x.size, np.float32(eb), int(mode), _ptr(out), cap, _ptr(nbytes))
    return st, out[: int(nbytes[0])].copy() if st in (OK, ERANGE) else out[:0]


def compress_minmax(x, lam: float, minmax) -> tuple[int, np.ndarray]:
    x = _f32(x).ravel()
    mm = _f32(minmax).ravel()
    cap = max_compressed_bytes(x.size)
    out = np.zeros(cap, np.uint8)
    nbytes = np.zeros(1, np.uint64)
    st = lib().oracle_compress_minmax(
        _ptr(x), x.size, np.float32(lam), _ptr(mm), mm.size // 2, _ptr(out), cap, _ptr(nbytes)
    )
    return st, out[: int(nbytes[0])].copy() if st in (OK, ERANGE) else out[:0]


def decompress(stream, n: int) -> tuple[int, np.ndarray]:
    s = np.ascontiguousarray(np.frombuffer(bytes(stream), np.uint8) if isinstance(stream, (bytes, bytearray)) else stream, dtype=np.uint8)
    out = np.zeros(int(n), np.float32)
    st = lib().oracle_decompress(_ptr(s), s.size, _ptr(out), int(n))
    return st, out


# ---- block-length variants: L in {8, 16, 32, 64, 128}

def block_lorenzo_L(q, Lb: int) -> np.ndarray:
    q = np.ascontiguousarray(q, dtype=np.int32)
    assert q.size % Lb == 0
    out = np.zeros_like(q)
    lib().oracle_block_lorenzo_L(_ptr(q), q.size // Lb, int(Lb), _ptr(out))
    return out


def encode_block_L(l, Lb: int) -> tuple[int, bytes]:
    l = np.ascontiguousarray(l, dtype=np.int32)
    assert l.size == Lb
    buf = np.zeros(25 * 16, np.uint8)
    F = lib().oracle_encode_block_L(_ptr(l), int(Lb), _ptr(buf))
    return F, bytes(buf[: block_bytes(F, Lb)])


def decode_block_L(payload: bytes, F: int, Lb: int) -> np.ndarray:
    buf = np.zeros(25 * 16, np.uint8)
    buf[: len(payload)] = np.frombuffer(payload, np.uint8)
    out = np.zeros(Lb, np.int32)
    lib().oracle_decode_block_L(_ptr(buf), int(F), int(Lb), _ptr(out))
    return out


def max_compressed_bytes_L(n: int, Lb: int) -> int:
    return int(lib().oracle_max_compressed_bytes_L(int(n), int(Lb)))


def compress_L(x, eb: float, mode: int, Lb: int) -> tuple[int, np.ndarray]:
    x = _f32(x).ravel()
    cap = max_compressed_bytes_L(x.size, Lb)
    out = np.zeros(cap, np.uint8)
    nbytes = np.zeros(1, np.uint64)
    st = lib().oracle_compress_L(_ptr(x), x.size, np.float32(eb), int(mode), int(Lb), _ptr(out), cap, _ptr(nbytes))
    return st, out[: int(nbytes[0])].copy() if st in (OK, ERANGE) else out[:0]


def compress_ex(x, eb: float, mode: int, Lb: int = L, order: int = 1) -> tuple[int, np.ndarray]:
    """Block length Lb and Lorenzo order (1, or 2 = the 2-layer predictor)."""
    x = _f32(x).ravel()
    cap = max_compressed_bytes_L(x.size, Lb)
    out = np.zeros(cap, np.uint8)
    nbytes = np.zeros(1, np.uint64)
    st = lib().oracle_compress_ex(_ptr(x), x.size, np.float32(eb), int(mode), int(Lb), int(order), _ptr(out), cap,
                                  _ptr(nbytes))
    return st, out[: int(nbytes[0])].copy() if st in (OK, ERANGE) else out[:0]


def compress_minmax_L(x, lam: float, minmax, Lb: int) -> tuple[int, np.ndarray]:
    x = _f32(x).ravel()
    mm = _f32(minmax).ravel()
    cap = max_compressed_bytes_L(x.size, Lb)
    out = np.zeros(cap, np.uint8)
    nbytes = np.zeros(1, np.uint64)
    st = lib().oracle_compress_minmax_L(_ptr(x), x.size, np.float32(lam), _ptr(mm), mm.size // 2, int(Lb), _ptr(out),
                                        cap, _ptr(nbytes))
    return st, out[: int(nbytes[0])].copy() if st in (OK, ERANGE) else out[:0]


# ---- multi-dimensional Lorenzo (DESIGN R18)

def num_blocks_md(shape, dims: int) -> int:
    nz, ny, nx = _shape3(shape)
    return int(lib().oracle_num_blocks_md(nz, ny, nx, int(dims)))


def _shape3(shape):
    shape = tuple(int(v) for v in shape)
    return (1,) * (3 - len(shape)) + shape


def block_lorenzo_md(r, dims: int) -> np.ndarray:
    """Block-local Lorenzo of ONE block (32 integers in block order)."""
    r = np.ascontiguousarray(r, dtype=np.int32)
    assert r.size == 32
    out = np.zeros(32, np.int32)
    lib().oracle_block_lorenzo_md(_ptr(r), int(dims), _ptr(out))
    return out


def compress_md(x, shape, dims: int, eb: float, mode: int = REL) -> tuple[int, np.ndarray]:
    """x: the field (any array of prod(shape) float32, C order), shape
    (ny, nx) or (nz, ny, nx); dims 2 or 3."""
    x = _f32(x).ravel()
    nz, ny, nx = _shape3(shape)
    assert x.size == nz * ny * nx
    cap = int(lib().oracle_max_compressed_bytes_md(nz, ny, nx, int(dims)))
    out = np.zeros(cap, np.uint8)
    nbytes = np.zeros(1, np.uint64)
    st = lib().oracle_compress_md(_ptr(x), nz, ny, nx, int(dims), np.float32(eb), int(mode), _ptr(out), cap,
                                  _ptr(nbytes))
    return st, out[: int(nbytes[0])].copy() if st in (OK, ERANGE) else out[:0]


def decompress_md(stream, shape, dims: int) -> tuple[int, np.ndarray]:
    s = np.ascontiguousarray(stream, dtype=np.uint8)
    nz, ny, nx = _shape3(shape)
    out = np.zeros(nz * ny * nx, np.float32)
    st = lib().oracle_decompress_md(_ptr(s), s.size, _ptr(out), nz, ny, nx, int(dims))
    return st, out


QUALITY_KEYS = ("min", "max", "range", "max_abs_err", "max_rel_err", "max_pw_rel_err", "mse", "psnr", "nrmse",
                "norm_err", "norm_err_norm", "pearson")


def quality(x, y, bound: float = -1.0) -> dict:
    """Reconstruction statistics of QCAT compareData in fp64."""
    xa, ya = _f32(x), _f32(y)
    assert xa.size == ya.size and xa.size > 0
    out = np.zeros(12, np.float64)
    cnt = np.zeros(2, np.uint64)
    lib().oracle_quality(_ptr(xa), _ptr(ya), xa.size, float(bound), _ptr(out), _ptr(cnt))
    d = dict(zip(QUALITY_KEYS, (float(v) for v in out)))
    d["n"], d["n_over_bound"] = int(cnt[0]), int(cnt[1])
    return d
