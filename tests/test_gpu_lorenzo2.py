"""GPU parity of the 2-layer Lorenzo predictor (SURVEY 8(f) NEXT rank 4,
P:535-545, DESIGN R17) against oracle.compress_ex(..., order=2): compressed
bytes identical, decompressed floats bit-identical; the tightened guard and
a stream/order mismatch give the same statuses as the oracle."""
from __future__ import annotations

import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_huangd0lc23_b200 as cz
import synth

pytestmark = pytest.mark.gpu
DEV = "cuda"


def parity2(x_np, eb, mode, label):
    x = torch.from_numpy(x_np).to(DEV)
    st_o, s_o = oracle.compress_ex(x_np, eb, mode, 32, 2)
    out, nb = cz.compress(x, eb, mode, order=2)
    torch.cuda.synchronize()
    s_g = out[: int(nb.item())].cpu().numpy()
    assert s_g[6] == st_o, (label, s_g[6], st_o)
    if st_o != oracle.OK:
        return
    assert s_g.size == s_o.size and np.array_equal(s_g, s_o), label
    st, y_o = oracle.decompress(s_o, x_np.size)
    y = cz.decompress(out, x_np.size, in_bytes=s_o.size, order=2)
    torch.cuda.synchronize()
    assert np.array_equal(y.cpu().numpy().view(np.uint32), y_o.view(np.uint32)), label


@pytest.mark.parametrize("n", [2, 3, 31, 33, 4096, 4099, 100_003, 1 << 20])
def test_sizes(n):
    rng = np.random.default_rng(n)
    x = np.cumsum(rng.standard_normal(n)).astype(np.float32) + 2
    x[n // 3: n // 2] = 0.0
    parity2(x, 1e-3, oracle.REL, f"n={n}")


@pytest.mark.parametrize("field,rel", [("U", 1e-2), ("QCLOUD", 1e-3), ("TC", 1e-4)])
def test_hurricane_fields(field, rel):
    x = synth.hurricane_like(field, shape=(20, 100, 100), device="cpu").numpy()
    parity2(x, rel, oracle.REL, f"{field}@{rel}")


def test_guard_and_wide_blocks():
    rng = np.random.default_rng(7)
    x = (rng.standard_normal(200_000) * 1e3).astype(np.float32)
    for eb in (1e-3, 0.3, 30.0):                     # F up to 24 and the 2^21 guard
        parity2(x, eb, oracle.ABS, f"abs eb={eb}")
    big = np.full(1000, float((1 << 21) + 9), np.float32)
    parity2(big, 0.5, oracle.ABS, "guard 2^21")      # order 1 would accept it


def test_order_mismatch_and_bad_args():
    x = torch.from_numpy(synth.smooth1d(50_000, seed=2, device="cpu").numpy()).to(DEV)
    out, nb = cz.compress(x, 1e-3, "rel", order=2)
    cz.decompress(out, x.numel())                      # decoded as order 1
    assert cz.last_status() == cz.ECORRUPT
    with pytest.raises(cz.CuszpError):
        cz.compress(x, 1e-3, "rel", order=3)
    with pytest.raises(cz.CuszpError):
        cz.compress(x, 1e-3, "rel", order=2, block_len=64)
