"""paper_conf_sc_huangd0lc23_b200 -- B200-native cuSZp (Huang et al., SC'23).

Thin Python binding over the C ABI in include/cuszp.h (libcuszp.so):
argument marshalling only.  Every step of compression and decompression
runs in the CUDA kernels of csrc/; torch supplies device memory, streams
and (in .dist) process groups.  Tensors must be CUDA tensors: there is no
CPU path.

    import paper_conf_sc_huangd0lc23_b200 as cz
    stream, nbytes = cz.compress(x, 1e-3, "rel")     # x: float32 CUDA tensor
    y = cz.decompress(stream, x.numel())
"""
from __future__ import annotations

import ctypes as C
import struct

import torch

from ._lib import (  # noqa: F401
    ECORRUPT, ECUDA, EINVAL, ENOSPACE, ERANGE, OK, STATUS_NAMES, CuszpError, check, lib,
)

ABS, REL = 0, 1
HEADER_BYTES = 32
BLOCK_LEN = 32

__all__ = [
    "ABS", "REL", "Workspace", "compress", "compress_minmax", "decompress", "value_range",
    "max_compressed_bytes", "workspace_bytes", "last_status", "read_header", "compress_host",
    "decompress_host", "CuszpError", "exact_bytes_from_F", "quality", "QUALITY_KEYS",
    "compress_host_async", "decompress_host_async", "compress_md", "decompress_md", "WorkspaceMD",
]


def _mode(mode) -> int:
    if isinstance(mode, str):
        return {"abs": ABS, "rel": REL}[mode.lower()]
    return int(mode)


def _stream_ptr(stream) -> int:
    s = stream if stream is not None else torch.cuda.current_stream()
    return int(s.cuda_stream)


def _check_out_bytes(t: torch.Tensor):
    _require_cuda(t, "out_bytes", torch.int64)
    if t.numel() < 1:
        raise ValueError("out_bytes must hold one int64")


def _require_cuda(t: torch.Tensor, name: str, dtype=None):
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError(f"{name} must be a CUDA tensor (no CPU path exists)")
    if dtype is not None and t.dtype != dtype:
        raise TypeError(f"{name} must be {dtype}, got {t.dtype}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")


def max_compressed_bytes(n: int, block_len: int = BLOCK_LEN) -> int:
    return int(lib().cuszp_max_compressed_bytes_L(int(n), int(block_len)))


def workspace_bytes(n: int) -> int:
    return int(lib().cuszp_workspace_bytes(int(n)))


def exact_bytes_from_F(F) -> int:
    import numpy as np

    a = np.ascontiguousarray(F, dtype=np.uint8)
    return int(lib().cuszp_compressed_bytes_from_F(a.ctypes.data_as(C.c_void_p), a.size))


class Workspace:
    """Zero-initialised device workspace for calls with up to ``n`` elements.
    Calls sharing a workspace must be stream-ordered."""

    def __init__(self, n: int, device=None):
        device = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
        self.n = int(n)
        self.nbytes = workspace_bytes(max(1, self.n))
        self.buf = torch.zeros(self.nbytes, dtype=torch.uint8, device=device)

    def ptr(self) -> int:
        return self.buf.data_ptr()

    def fits(self, n: int) -> bool:
        return workspace_bytes(max(1, int(n))) <= self.nbytes


_ws_cache: dict = {}


def _workspace(n: int, device, ws: Workspace | None, stream=None) -> Workspace:
    """The caller's workspace, or a cached one per (device, stream the call
    is launched on): calls on different streams never share a workspace."""
    if ws is not None:
        if not ws.fits(n):
            raise CuszpError(ENOSPACE, "workspace too small")
        return ws
    dev_index = device.index if device.index is not None else torch.cuda.current_device()
    s = stream if stream is not None else torch.cuda.current_stream(torch.device("cuda", dev_index))
    key = (dev_index, int(s.cuda_stream))
    w = _ws_cache.get(key)
    if w is None or not w.fits(n):
        cur = torch.cuda.current_stream(torch.device("cuda", dev_index))
        if w is not None:
            # calls already queued on s may still use the old buffer: the
            # caching allocator must not hand it out before s reaches this point
            w.buf.record_stream(s)
        w = Workspace(max(int(n), 1 << 20), device)
        _ws_cache[key] = w
        s.wait_stream(cur)                                   # zeroed (on cur) before first use on s
        if s != cur:
            w.buf.record_stream(s)
    return w


def value_range(x: torch.Tensor, ws: Workspace | None = None, out: torch.Tensor | None = None, stream=None):
    """(min, max) of x on the device as a float32 tensor of 2 (Eq 1's r)."""
    _require_cuda(x, "x", torch.float32)
    ws = _workspace(x.numel(), x.device, ws, stream)
    if out is None:
        out = torch.empty(2, dtype=torch.float32, device=x.device)
    _require_cuda(out, "out", torch.float32)
    if out.numel() < 2:
        raise ValueError("out must hold 2 float32 values (min, max)")
    check(lib().cuszp_range(x.data_ptr(), x.numel(), out.data_ptr(), ws.ptr(), ws.nbytes, _stream_ptr(stream)),
          "cuszp_range")
    return out


def compress(x: torch.Tensor, eb: float, mode="rel", out: torch.Tensor | None = None,
             out_bytes: torch.Tensor | None = None, ws: Workspace | None = None, stream=None,
             block_len: int = BLOCK_LEN, order: int = 1):
    """Compress a float32 CUDA tensor.  Returns (stream buffer uint8 tensor of
    capacity max_compressed_bytes(n), device int64 tensor [1] holding the
    exact stream length).  Asynchronous; data errors land in the header."""
    _require_cuda(x, "x", torch.float32)
    n = x.numel()
    cap = max_compressed_bytes(n, block_len)
    if out is None:
        out = torch.empty(cap, dtype=torch.uint8, device=x.device)
    _require_cuda(out, "out", torch.uint8)
    if out_bytes is None:
        out_bytes = torch.zeros(1, dtype=torch.int64, device=x.device)
    _check_out_bytes(out_bytes)
    ws = _workspace(n, x.device, ws, stream)
    check(lib().cuszp_compress_ex(x.data_ptr(), n, float(eb), _mode(mode), int(block_len), int(order),
                                  out.data_ptr(), out.numel(), out_bytes.data_ptr(), ws.ptr(), ws.nbytes,
                                  _stream_ptr(stream)), "cuszp_compress")
    return out, out_bytes


def compress_minmax(x: torch.Tensor, lam: float, minmax: torch.Tensor, out: torch.Tensor | None = None,
                    out_bytes: torch.Tensor | None = None, ws: Workspace | None = None, stream=None,
                    block_len: int = BLOCK_LEN):
    """REL compression against a global range given as (min, max) pairs on the device."""
    _require_cuda(x, "x", torch.float32)
    _require_cuda(minmax, "minmax", torch.float32)
    n = x.numel()
    if out is None:
        out = torch.empty(max_compressed_bytes(n, block_len), dtype=torch.uint8, device=x.device)
    _require_cuda(out, "out", torch.uint8)
    if out_bytes is None:
        out_bytes = torch.zeros(1, dtype=torch.int64, device=x.device)
    _check_out_bytes(out_bytes)
    if minmax.numel() < 2:
        raise ValueError("minmax must hold at least one (min, max) pair")
    ws = _workspace(n, x.device, ws, stream)
    check(lib().cuszp_compress_minmax_L(x.data_ptr(), n, float(lam), minmax.data_ptr(), minmax.numel() // 2,
                                        int(block_len), out.data_ptr(), out.numel(), out_bytes.data_ptr(), ws.ptr(),
                                        ws.nbytes, _stream_ptr(stream)), "cuszp_compress_minmax")
    return out, out_bytes


def decompress(stream_buf: torch.Tensor, n: int, out: torch.Tensor | None = None, in_bytes: int | None = None,
               ws: Workspace | None = None, stream=None, block_len: int = BLOCK_LEN, order: int = 1) -> torch.Tensor:
    """Decompress a device stream into n float32 values (asynchronous)."""
    _require_cuda(stream_buf, "stream_buf", torch.uint8)
    if out is None:
        out = torch.empty(int(n), dtype=torch.float32, device=stream_buf.device)
    _require_cuda(out, "out", torch.float32)
    if out.numel() < int(n):
        raise ValueError(f"out holds {out.numel()} floats, {int(n)} needed")
    ws = _workspace(n, stream_buf.device, ws, stream)
    nbytes = stream_buf.numel() if in_bytes is None else int(in_bytes)
    if nbytes > stream_buf.numel() or nbytes < 0:
        raise ValueError(f"in_bytes={nbytes} exceeds the stream buffer ({stream_buf.numel()} bytes)")
    check(lib().cuszp_decompress_ex(stream_buf.data_ptr(), nbytes, out.data_ptr(), int(n), int(block_len),
                                    int(order), ws.ptr(), ws.nbytes, _stream_ptr(stream)), "cuszp_decompress")
    return out


def _shape3(shape) -> tuple[int, int, int]:
    shape = tuple(int(v) for v in shape)
    if not 1 <= len(shape) <= 3:
        raise ValueError("shape must have 1 to 3 dimensions")
    return (1,) * (3 - len(shape)) + shape


class WorkspaceMD(Workspace):
    """Zeroed workspace for the multi-dimensional calls on a given shape."""

    def __init__(self, shape, dims: int, device=None):
        device = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
        nz, ny, nx = _shape3(shape)
        self.n = nz * ny * nx
        self.nbytes = int(lib().cuszp_workspace_bytes_md(nz, ny, nx, int(dims)))
        if self.nbytes == 0:
            raise ValueError("unsupported shape / dims")
        self.buf = torch.zeros(self.nbytes, dtype=torch.uint8, device=device)


def compress_md(x: torch.Tensor, eb: float, mode="rel", dims: int | None = None, shape=None,
                out: torch.Tensor | None = None, out_bytes: torch.Tensor | None = None, ws: Workspace | None = None,
                stream=None):
    """Compress a 2D/3D float32 CUDA field with the multi-dimensional Lorenzo
    predictor (dims 2: 1x4x8 blocks, 3: 2x4x4 blocks; DESIGN R18).  shape
    defaults to x.shape, dims to len(shape).  Returns (stream buffer, device
    int64[1] stream length)."""
    _require_cuda(x, "x", torch.float32)
    shape = tuple(x.shape) if shape is None else tuple(shape)
    nz, ny, nx = _shape3(shape)
    if nz * ny * nx != x.numel():
        raise ValueError("shape does not match x")
    dims = len(shape) if dims is None else int(dims)
    cap = int(lib().cuszp_max_compressed_bytes_md(nz, ny, nx, dims))
    if cap == 0:
        raise ValueError("unsupported shape / dims")
    if out is None:
        out = torch.empty(cap, dtype=torch.uint8, device=x.device)
    _require_cuda(out, "out", torch.uint8)
    if out_bytes is None:
        out_bytes = torch.zeros(1, dtype=torch.int64, device=x.device)
    _check_out_bytes(out_bytes)
    if ws is None:
        ws = WorkspaceMD(shape, dims, x.device)
    check(lib().cuszp_compress_md(x.data_ptr(), nz, ny, nx, dims, float(eb), _mode(mode), out.data_ptr(), out.numel(),
                                  out_bytes.data_ptr(), ws.ptr(), ws.nbytes, _stream_ptr(stream)), "cuszp_compress_md")
    return out, out_bytes


def decompress_md(stream_buf: torch.Tensor, shape, dims: int | None = None, out: torch.Tensor | None = None,
                  in_bytes: int | None = None, ws: Workspace | None = None, stream=None) -> torch.Tensor:
    """Decompress a multi-dimensional-Lorenzo stream into a field of the given shape."""
    _require_cuda(stream_buf, "stream_buf", torch.uint8)
    shape = tuple(int(v) for v in shape)
    nz, ny, nx = _shape3(shape)
    dims = len(shape) if dims is None else int(dims)
    if out is None:
        out = torch.empty(shape, dtype=torch.float32, device=stream_buf.device)
    _require_cuda(out, "out", torch.float32)
    if out.numel() < nz * ny * nx:
        raise ValueError("out is smaller than the field")
    nbytes = stream_buf.numel() if in_bytes is None else int(in_bytes)
    if nbytes > stream_buf.numel() or nbytes < 0:
        raise ValueError("in_bytes exceeds the stream buffer")
    if ws is None:
        ws = WorkspaceMD(shape, dims, stream_buf.device)
    check(lib().cuszp_decompress_md(stream_buf.data_ptr(), nbytes, out.data_ptr(), nz, ny, nx, dims, ws.ptr(),
                                    ws.nbytes, _stream_ptr(stream)), "cuszp_decompress_md")
    return out


def last_status(ws: Workspace | None = None, device=None, stream=None) -> int:
    """Status of the last call on ``ws`` (synchronises the stream)."""
    if ws is None:
        device = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
        ws = _workspace(1, device, None, stream)
    return int(lib().cuszp_last_status(ws.ptr(), _stream_ptr(stream)))


def read_header(stream_buf: torch.Tensor, stream=None) -> dict:
    _require_cuda(stream_buf, "stream_buf", torch.uint8)
    raw = (C.c_uint8 * 32)()
    check(lib().cuszp_read_header(stream_buf.data_ptr(), C.cast(raw, C.c_void_p), _stream_ptr(stream)),
          "cuszp_read_header")
    b = bytes(raw)
    n, = struct.unpack_from("<Q", b, 8)
    eb_abs, eb_in = struct.unpack_from("<ff", b, 16)
    payload, = struct.unpack_from("<Q", b, 24)
    return dict(magic=b[:4], version=b[4], mode=b[5], status=b[6], log2l=b[7], n=n, eb_abs=eb_abs,
                eb_in=eb_in, payload_bytes=payload)


def compress_host(h_in, eb: float, mode, h_out, d_in_scratch: torch.Tensor, d_out_scratch: torch.Tensor,
                  ws: Workspace, stream=None) -> int:
    """End-to-end compression from a host float32 buffer (numpy or pinned
    CPU tensor) into a host uint8 buffer; returns the stream length."""
    n = h_in.numel() if isinstance(h_in, torch.Tensor) else h_in.size
    pin = h_in.data_ptr() if isinstance(h_in, torch.Tensor) else h_in.ctypes.data
    pout = h_out.data_ptr() if isinstance(h_out, torch.Tensor) else h_out.ctypes.data
    cap = h_out.numel() if isinstance(h_out, torch.Tensor) else h_out.size
    nbytes = C.c_size_t(0)
    check(lib().cuszp_compress_host(pin, n, float(eb), _mode(mode), pout, cap, C.byref(nbytes),
                                    d_in_scratch.data_ptr(), d_out_scratch.data_ptr(), ws.ptr(), ws.nbytes,
                                    _stream_ptr(stream)), "cuszp_compress_host")
    return int(nbytes.value)


def decompress_host(h_in, in_bytes: int, h_out, d_in_scratch: torch.Tensor, d_out_scratch: torch.Tensor,
                    ws: Workspace, stream=None) -> None:
    n = h_out.numel() if isinstance(h_out, torch.Tensor) else h_out.size
    pin = h_in.data_ptr() if isinstance(h_in, torch.Tensor) else h_in.ctypes.data
    pout = h_out.data_ptr() if isinstance(h_out, torch.Tensor) else h_out.ctypes.data
    check(lib().cuszp_decompress_host(pin, int(in_bytes), pout, n, d_in_scratch.data_ptr(),
                                      d_out_scratch.data_ptr(), ws.ptr(), ws.nbytes, _stream_ptr(stream)),
          "cuszp_decompress_host")


QUALITY_KEYS = ("min", "max", "range", "max_abs_err", "max_rel_err", "max_pw_rel_err", "mse", "psnr", "nrmse",
                "norm_err", "norm_err_norm", "pearson")
_qws_cache: dict = {}


def quality(x: torch.Tensor, y: torch.Tensor, bound: float = -1.0, out: torch.Tensor | None = None,
            stream=None, sync: bool = True):
    """Reconstruction statistics (QCAT compareData's) of y
    against x in one fused device pass (cuszp_quality).  ``out`` (float64
    CUDA tensor of 14) receives the raw cuszp_quality_stats; with sync=True
    the statistics are returned as a dict (one 112-byte device->host copy)."""
    _require_cuda(x, "x", torch.float32)
    _require_cuda(y, "y", torch.float32)
    if x.numel() != y.numel():
        raise ValueError("x and y must have the same number of elements")
    key = (x.device.index, _stream_ptr(stream))            # one quality workspace per stream
    qws = _qws_cache.get(key)
    if qws is None:
        qws = torch.zeros(int(lib().cuszp_quality_workspace_bytes()), dtype=torch.uint8, device=x.device)
        _qws_cache[key] = qws
        if stream is not None:
            cur = torch.cuda.current_stream(x.device)
            stream.wait_stream(cur)                          # the zeroing (on cur) precedes the first use
            if stream != cur:
                qws.record_stream(stream)
    if out is None:
        out = torch.empty(14, dtype=torch.float64, device=x.device)
    _require_cuda(out, "out", torch.float64)
    if out.numel() < 14:
        raise ValueError("out must hold 14 float64 values (cuszp_quality_stats)")
    check(lib().cuszp_quality(x.data_ptr(), y.data_ptr(), x.numel(), float(bound), out.data_ptr(), qws.data_ptr(),
                              qws.numel(), _stream_ptr(stream)), "cuszp_quality")
    if not sync:
        return out
    raw = out.cpu()
    d = dict(zip(QUALITY_KEYS, (float(v) for v in raw[:12])))
    cnt = raw[12:].view(torch.int64)
    d["n"], d["n_over_bound"] = int(cnt[0]), int(cnt[1])
    return d


def _hptr(t) -> int:
    return t.data_ptr() if isinstance(t, torch.Tensor) else t.ctypes.data


def compress_host_async(h_in: torch.Tensor, eb: float, mode, h_out: torch.Tensor, h_len: torch.Tensor,
                        d_in_scratch: torch.Tensor, d_out_scratch: torch.Tensor, ws: Workspace, stream=None) -> None:
    """Asynchronous end-to-end compression (cuszp_compress_host_async):
    pinned h_in -> device -> stream into the pinned, mapped h_out; its length
    into h_len (pinned int64[1]) once ``stream`` reaches this point."""
    n_out = h_out.numel() if isinstance(h_out, torch.Tensor) else h_out.size
    check(lib().cuszp_compress_host_async(_hptr(h_in), h_in.numel(), float(eb), _mode(mode), _hptr(h_out),
                                          n_out, _hptr(h_len), d_in_scratch.data_ptr(),
                                          d_out_scratch.data_ptr(), ws.ptr(), ws.nbytes, _stream_ptr(stream)),
          "cuszp_compress_host_async")


def decompress_host_async(h_in: torch.Tensor, h_out: torch.Tensor, d_in_scratch: torch.Tensor,
                          d_out_scratch: torch.Tensor, ws: Workspace, stream=None, in_capacity: int | None = None) -> None:
    """Asynchronous end-to-end decompression (cuszp_decompress_host_async)
    of the stream in the pinned, mapped h_in (length from its header) into
    the pinned h_out (n = h_out.numel())."""
    cap = min(h_in.numel(), d_in_scratch.numel()) if in_capacity is None else int(in_capacity)
    check(lib().cuszp_decompress_host_async(_hptr(h_in), cap, _hptr(h_out), h_out.numel(), d_in_scratch.data_ptr(),
                                            d_out_scratch.data_ptr(), ws.ptr(), ws.nbytes, _stream_ptr(stream)),
          "cuszp_decompress_host_async")
