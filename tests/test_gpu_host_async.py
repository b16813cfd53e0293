"""The asynchronous host-buffer calls (cuszp_compress_host_async /
cuszp_decompress_host_async): the stream that lands in pinned host memory
is the oracle's byte for byte, its length is reported exactly, and the
reconstruction that lands back in host memory is the oracle's bit for bit
-- also with two streams in flight at once (the e2e pipeline of bench.py)."""
from __future__ import annotations

import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_huangd0lc23_b200 as cz
import synth

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("n", [0, 1, 33, 4096, 100_003, 1 << 20])
def test_async_round_trip_matches_oracle(n):
    x = synth.smooth1d(max(n, 1), seed=n % 7 + 1, device="cpu")[:n].contiguous()
    x_np = x.numpy()
    cap = cz.max_compressed_bytes(n)
    h_in = x.pin_memory()
    h_out = torch.zeros(cap, dtype=torch.uint8).pin_memory()
    h_len = torch.zeros(1, dtype=torch.int64).pin_memory()
    h_y = torch.full((n,), float("nan"), dtype=torch.float32).pin_memory()
    d_in = torch.empty(max(n, 4), dtype=torch.float32, device="cuda")
    d_out = torch.empty(cap, dtype=torch.uint8, device="cuda")
    d_y = torch.empty(max(n, 4), dtype=torch.float32, device="cuda")
    ws = cz.Workspace(max(n, 1), "cuda")
    s = torch.cuda.Stream()
    cz.compress_host_async(h_in, 1e-4, "rel", h_out, h_len, d_in, d_out, ws, stream=s)
    cz.decompress_host_async(h_out, h_y, d_out, d_y, ws, stream=s)
    s.synchronize()
    st, s_o = oracle.compress(x_np, 1e-4, oracle.REL)
    assert int(h_out[6].item()) == st                  # header status byte (n = 1: constant field -> ERANGE, R5)
    assert int(h_len.item()) == s_o.size
    if st != oracle.OK:
        return
    assert np.array_equal(h_out[: s_o.size].numpy(), s_o)
    st, y_o = oracle.decompress(s_o, n)
    assert np.array_equal(h_y.numpy().view(np.uint32), y_o.view(np.uint32))


def test_two_streams_in_flight():
    fields = ["U", "QCLOUD", "TC"]
    xs = [synth.hurricane_like(f, shape=(20, 100, 100), device="cpu") for f in fields]
    n = xs[0].numel()
    cap = cz.max_compressed_bytes(n)
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    bufs = []
    for _ in streams:
        bufs.append(dict(h_out=torch.zeros(cap, dtype=torch.uint8).pin_memory(),
                         h_len=torch.zeros(1, dtype=torch.int64).pin_memory(),
                         d_in=torch.empty(n, device="cuda"), d_out=torch.empty(cap, dtype=torch.uint8, device="cuda"),
                         d_y=torch.empty(n, device="cuda"), ws=cz.Workspace(n, "cuda")))
    h_in = [x.pin_memory() for x in xs]
    h_y = [torch.empty(n).pin_memory() for _ in xs]
    for j, (x, hy) in enumerate(zip(h_in, h_y)):
        b, s = bufs[j % 2], streams[j % 2]
        cz.compress_host_async(x, 1e-3, "rel", b["h_out"], b["h_len"], b["d_in"], b["d_out"], b["ws"], stream=s)
        cz.decompress_host_async(b["h_out"], hy, b["d_out"], b["d_y"], b["ws"], stream=s)
    torch.cuda.synchronize()
    for x, hy in zip(xs, h_y):
        st, s_o = oracle.compress(x.numpy(), 1e-3, oracle.REL)
        st, y_o = oracle.decompress(s_o, n)
        assert np.array_equal(hy.numpy().view(np.uint32), y_o.view(np.uint32))


def test_async_rejects_unmapped_or_small():
    n = 1000
    x = torch.zeros(n).pin_memory()
    d = torch.empty(n, device="cuda")
    ws = cz.Workspace(n, "cuda")
    small = torch.zeros(16, dtype=torch.uint8).pin_memory()
    with pytest.raises(cz.CuszpError):
        cz.compress_host_async(x, 1e-3, "rel", small, torch.zeros(1, dtype=torch.int64).pin_memory(), d,
                               torch.empty(cz.max_compressed_bytes(n), dtype=torch.uint8, device="cuda"), ws)
    unpinned = np.zeros(cz.max_compressed_bytes(n), np.uint8)
    with pytest.raises(cz.CuszpError):
        cz.compress_host_async(x, 1e-3, "rel", unpinned, torch.zeros(1, dtype=torch.int64).pin_memory(), d,
                               torch.empty(cz.max_compressed_bytes(n), dtype=torch.uint8, device="cuda"), ws)


def test_async_rejects_misaligned_before_any_launch():
    """misaligned mapped/scratch buffers are rejected with EINVAL
    before anything is launched (no sticky misaligned-address error), and the
    context keeps working afterwards."""
    n = 4096
    cap = cz.max_compressed_bytes(n)
    x = synth.smooth1d(n, seed=2, device="cpu").pin_memory()
    h_out = torch.zeros(cap + 64, dtype=torch.uint8).pin_memory()
    h_len = torch.zeros(4, dtype=torch.int64).pin_memory()
    d_in = torch.empty(n + 16, dtype=torch.float32, device="cuda")
    d_out = torch.empty(cap + 64, dtype=torch.uint8, device="cuda")
    d_y = torch.empty(n + 16, dtype=torch.float32, device="cuda")
    ws = cz.Workspace(n, "cuda")
    L = cz.lib()
    sp = int(torch.cuda.current_stream().cuda_stream)
    bad_calls = [
        (h_out.data_ptr() + 1, h_len.data_ptr(), d_in.data_ptr(), d_out.data_ptr()),
        (h_out.data_ptr(), h_len.data_ptr() + 4, d_in.data_ptr(), d_out.data_ptr()),
        (h_out.data_ptr(), h_len.data_ptr(), d_in.data_ptr() + 4, d_out.data_ptr()),
        (h_out.data_ptr(), h_len.data_ptr(), d_in.data_ptr(), d_out.data_ptr() + 8),
    ]
    for ho, hl, di, do in bad_calls:
        st = L.cuszp_compress_host_async(x.data_ptr(), n, 1e-3, cz.REL, ho, cap, hl, di, do, ws.ptr(), ws.nbytes, sp)
        assert st == cz.EINVAL
    st = L.cuszp_decompress_host_async(h_out.data_ptr() + 4, cap, torch.empty(n).pin_memory().data_ptr(), n,
                                       d_out.data_ptr(), d_y.data_ptr(), ws.ptr(), ws.nbytes, sp)
    assert st == cz.EINVAL
    st = L.cuszp_decompress_host_async(h_out.data_ptr(), cap, torch.empty(n).pin_memory().data_ptr(), n,
                                       d_out.data_ptr() + 4, d_y.data_ptr(), ws.ptr(), ws.nbytes, sp)
    assert st == cz.EINVAL
    torch.cuda.synchronize()                    # no sticky error
    cz.compress_host_async(x, 1e-3, "rel", h_out[:cap], h_len[:1], d_in[:n], d_out[:cap], ws)
    torch.cuda.synchronize()
    st, s_o = oracle.compress(x.numpy(), 1e-3, oracle.REL)
    assert int(h_len[0].item()) == s_o.size and np.array_equal(h_out[: s_o.size].numpy(), s_o)


def test_binding_rejects_short_buffers():
    """the binding is the only guard of the output capacity."""
    x = torch.randn(1000, device="cuda")
    out, nb = cz.compress(x, 1e-3, "rel")
    with pytest.raises(ValueError):
        cz.decompress(out, 1000, out=torch.empty(999, device="cuda"))
    with pytest.raises(ValueError):
        cz.decompress(out, 1000, in_bytes=out.numel() + 1)
    with pytest.raises(ValueError):
        cz.compress(x, 1e-3, "rel", out_bytes=torch.zeros(0, dtype=torch.int64, device="cuda"))
    with pytest.raises(ValueError):
        cz.value_range(x, out=torch.empty(1, device="cuda"))
    y = cz.decompress(out, 1000)
    torch.cuda.synchronize()
    assert cz.last_status() == cz.OK and float((x - y).abs().max()) <= float(cz.read_header(out)["eb_abs"]) * 1.001


def test_workspace_replaced_while_in_use_on_side_stream():
    """a cached workspace that grows while calls are queued on a
    side stream is not recycled under them (record_stream)."""
    s = torch.cuda.Stream()
    small = torch.randn(1000, device="cuda")
    big = synth.smooth1d(3 << 20, seed=5, device="cuda")
    torch.cuda.synchronize()
    for _ in range(3):
        o1, n1 = cz.compress(small, 1e-3, "rel", stream=s)
        o2, n2 = cz.compress(big, 1e-3, "rel", stream=s)     # replaces the cached (1 Mi-element) workspace
        junk = torch.ones(cz.workspace_bytes(1 << 20) // 4 + 64, dtype=torch.int32, device="cuda")   # would reuse it
        s.synchronize()
        st, s_o = oracle.compress(big.cpu().numpy(), 1e-3, oracle.REL)
        assert np.array_equal(o2[: int(n2.item())].cpu().numpy(), s_o)
        del junk
