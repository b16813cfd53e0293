"""GPU parity of the block-length variants L in {8, 16, 64, 128} (SURVEY 8(f) NEXT
rank 3) against oracle.compress_L / oracle.decompress: compressed bytes
identical, decompressed floats bit-identical, on sizes spanning many tiles
with ragged tails and on fields that exercise all three packing modes of
the kernels (F <= 7, F <= 15, F up to 24)."""
from __future__ import annotations

import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_huangd0lc23_b200 as cz
import synth

pytestmark = pytest.mark.gpu
DEV = "cuda"


def parity(x_np: np.ndarray, eb: float, mode: int, Lb: int, label=""):
    x = torch.from_numpy(x_np).to(DEV)
    st_o, s_o = oracle.compress_L(x_np, eb, mode, Lb)
    out, nb = cz.compress(x, eb, mode, block_len=Lb)
    torch.cuda.synchronize()
    s_g = out[: int(nb.item())].cpu().numpy()
    assert s_g[6] == st_o, (label, s_g[6], st_o)
    if st_o != oracle.OK:
        return
    assert s_g.size == s_o.size, (label, s_g.size, s_o.size)
    if not np.array_equal(s_g, s_o):
        bad = np.nonzero(s_g != s_o)[0]
        raise AssertionError(f"{label}: {bad.size} bytes differ, first at {bad[0]} of {s_o.size}")
    st, y_o = oracle.decompress(s_o, x_np.size)
    y = cz.decompress(out, x_np.size, in_bytes=s_o.size, block_len=Lb)
    torch.cuda.synchronize()
    assert np.array_equal(y.cpu().numpy().view(np.uint32), y_o.view(np.uint32)), label


@pytest.mark.parametrize("Lb", [8, 16, 64, 128])
@pytest.mark.parametrize("n", [2, 31, 64, 65, 129, 4096, 4097, 100_003, 1 << 20])
def test_sizes(Lb, n):
    rng = np.random.default_rng(n)
    x = np.cumsum(rng.standard_normal(n)).astype(np.float32)
    x[n // 3: n // 2] = 0.0
    parity(x, 1e-3, oracle.REL, Lb, f"L={Lb} n={n}")


@pytest.mark.parametrize("Lb", [8, 16, 64, 128])
@pytest.mark.parametrize("field,rel", [("U", 1e-2), ("QCLOUD", 1e-3), ("TC", 1e-4)])
def test_hurricane_fields(Lb, field, rel):
    x = synth.hurricane_like(field, shape=(20, 100, 100), device="cpu").numpy()
    parity(x, rel, oracle.REL, Lb, f"L={Lb} {field}@{rel}")


@pytest.mark.parametrize("Lb", [8, 16, 64, 128])
def test_wide_fixed_lengths(Lb):
    # ABS with a tiny bound: F up to the guard's 24 bits (one block per transpose)
    rng = np.random.default_rng(Lb)
    x = (rng.standard_normal(300_000) * 1e3).astype(np.float32)
    for eb in (1e-3, 1.0, 30.0):
        parity(x, eb, oracle.ABS, Lb, f"L={Lb} abs eb={eb}")


@pytest.mark.parametrize("Lb", [8, 16, 64, 128])
def test_minmax_and_wrong_L(Lb):
    x_np = synth.smooth1d(200_000, seed=3, device="cpu").numpy()
    x = torch.from_numpy(x_np).to(DEV)
    mm = torch.tensor([-5.0, 7.0], device=DEV)
    st, s_o = oracle.compress_minmax_L(x_np, 1e-4, mm.cpu().numpy(), Lb)
    out, nb = cz.compress_minmax(x, 1e-4, mm, block_len=Lb)
    torch.cuda.synchronize()
    assert np.array_equal(out[: int(nb.item())].cpu().numpy(), s_o)
    cz.decompress(out, x.numel(), block_len=32)          # header says another L
    assert cz.last_status() == cz.ECORRUPT
    with pytest.raises(cz.CuszpError):
        cz.compress(x, 1e-3, "rel", block_len=48)


@pytest.mark.parametrize("Lb,order", [(8, 1), (16, 1), (64, 1), (128, 1), (32, 2)])
def test_empty_tiny_and_nonfinite(Lb, order):
    for x_np in (np.zeros(0, np.float32), np.array([1.5], np.float32), np.array([1.0, -2.0], np.float32),
                 np.array([1.0, np.nan, 2.0], np.float32), np.array([np.inf, 0.0], np.float32)):
        for mode, eb in ((oracle.REL, 1e-3), (oracle.ABS, 1e-2)):
            st_o, s_o = oracle.compress_ex(x_np, eb, mode, Lb, order)
            x = torch.from_numpy(x_np).to(DEV)
            out, nb = cz.compress(x, eb, mode, block_len=Lb, order=order)
            torch.cuda.synchronize()
            s_g = out[: int(nb.item())].cpu().numpy()
            assert s_g[6] == st_o, (Lb, order, x_np, mode, s_g[6], st_o)
            if st_o == oracle.OK:
                assert np.array_equal(s_g, s_o), (Lb, order, x_np, mode)
                y = cz.decompress(out, x_np.size, in_bytes=s_o.size, block_len=Lb, order=order)
                st, y_o = oracle.decompress(s_o, x_np.size)
                torch.cuda.synchronize()
                assert np.array_equal(y.cpu().numpy().view(np.uint32), y_o.view(np.uint32))


@pytest.mark.slow
@pytest.mark.parametrize("Lb,order", [(8, 1), (16, 1), (64, 1), (128, 1), (32, 2)])
def test_full_size_nyx(Lb, order):
    """BASELINE's NYX-shaped 512^3 field (537 MB) at REL 1e-4: whole stream and
    reconstruction against the oracle for every variant."""
    x = synth.field_for_config("c4_nyx", device=DEV)
    x_np = x.cpu().numpy()
    st, s_o = oracle.compress_ex(x_np, 1e-4, oracle.REL, Lb, order)
    assert st == oracle.OK
    out, nb = cz.compress(x, 1e-4, "rel", block_len=Lb, order=order)
    torch.cuda.synchronize()
    assert np.array_equal(out[: int(nb.item())].cpu().numpy(), s_o)
    y = cz.decompress(out, x.numel(), in_bytes=int(nb.item()), block_len=Lb, order=order)
    st, y_o = oracle.decompress(s_o, x_np.size)
    assert np.array_equal(y.cpu().numpy().view(np.uint32), y_o.view(np.uint32))


def test_small_L_interleaved_with_word_kernels_and_corrupt_F():
    """L = 8 / 16 (byte-plane path, small_l.cu) and L = 32 / 64 (look-back
    kernels) alternate on one workspace: the small path's tile sums must never
    be read as published look-back words.  A fixed-length byte above 24 in an
    L = 8 stream is ECORRUPT (as for the oracle)."""
    rng = np.random.default_rng(11)
    x_np = np.cumsum(rng.standard_normal(300_001)).astype(np.float32)
    for Lb in (8, 32, 16, 64, 8, 32):
        parity(x_np, 1e-3, oracle.REL, Lb, f"interleaved L={Lb}")
    x = torch.from_numpy(x_np).to(DEV)
    out, nb = cz.compress(x, 1e-3, "rel", block_len=8)
    bad = out.clone()
    bad[32 + 5] = 25
    st, _ = oracle.decompress(bad[: int(nb.item())].cpu().numpy(), x_np.size)
    assert st == oracle.ECORRUPT
    cz.decompress(bad, x_np.size, in_bytes=int(nb.item()), block_len=8)
    assert cz.last_status() == cz.ECORRUPT
    y = cz.decompress(out, x_np.size, in_bytes=int(nb.item()), block_len=8)
    assert cz.last_status() == cz.OK
    assert torch.max(torch.abs(y - x)).item() <= float(cz.read_header(out)["eb_abs"]) * 1.001


@pytest.mark.parametrize("Lb", [8, 16])
def test_small_L_corrupt_and_truncated_streams(Lb):
    """L = 8 / 16 streams are byte-granular (payload sizes need not be a
    multiple of 4): a stream cut by 1..3 bytes, F above 24, F bytes that
    disagree with the header's payload size and random byte flips must only
    ever give a status; the workspace keeps working afterwards."""
    rng = np.random.default_rng(Lb)
    n = 70_001
    x_np = np.cumsum(rng.standard_normal(n)).astype(np.float32)
    x = torch.from_numpy(x_np).to(DEV)
    ws = cz.Workspace(n)
    out, nb = cz.compress(x, 1e-3, "rel", block_len=Lb, ws=ws)
    S = int(nb.item())
    y = torch.empty(n, device=DEV)
    for cut in (1, 2, 3, 17):
        cz.decompress(out, n, out=y, in_bytes=S - cut, ws=ws, block_len=Lb)
        assert cz.last_status(ws) == cz.ECORRUPT, cut
    c = out.clone(); c[32 + 7] = 25                                  # F > 24
    cz.decompress(c, n, out=y, in_bytes=S, ws=ws, block_len=Lb)
    assert cz.last_status(ws) == cz.ECORRUPT
    c = out.clone(); c[32 + 9] = (int(c[32 + 9]) + 1) % 25           # sizes disagree with the header
    cz.decompress(c, n, out=y, in_bytes=S + 400, ws=ws, block_len=Lb)
    assert cz.last_status(ws) == cz.ECORRUPT
    nbk = (n + Lb - 1) // Lb
    for _ in range(40):
        c = out.clone()
        for p in rng.integers(0, 32 + nbk, 3):
            c[int(p)] = int(rng.integers(0, 256))
        cz.decompress(c, n, out=y, in_bytes=S, ws=ws, block_len=Lb)
        assert cz.last_status(ws) in (cz.OK, cz.ECORRUPT, cz.EINVAL, cz.ERANGE)
    cz.decompress(out, n, out=y, in_bytes=S, ws=ws, block_len=Lb)
    assert cz.last_status(ws) == cz.OK
    st, y_o = oracle.decompress(out[:S].cpu().numpy(), n)
    assert st == oracle.OK and np.array_equal(y.cpu().numpy().view(np.uint32), y_o.view(np.uint32))
