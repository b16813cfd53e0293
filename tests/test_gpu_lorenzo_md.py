"""GPU parity of the multi-dimensional Lorenzo predictor (SURVEY 8(f) NEXT
rank 4, DESIGN R18) through cuszp_compress_md /
cuszp_decompress_md: stream bytes identical to oracle.compress_md and floats
bit-identical to oracle.decompress_md, on ragged shapes (edge blocks with
points outside the field, nx % 4 != 0 -> the scalar gather path), the
Hurricane- and NYX-shaped fields of BASELINE configs[1] / [3] at reduced and
full size, ABS bounds, the R18 guard and error statuses."""
from __future__ import annotations

import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_huangd0lc23_b200 as cz
import synth

pytestmark = pytest.mark.gpu
DEV = "cuda"


def _parity(f_np: np.ndarray, dims: int, eb: float, mode: int, label: str = ""):
    shape = f_np.shape
    x = torch.from_numpy(np.ascontiguousarray(f_np)).to(DEV)
    st_o, s_o = oracle.compress_md(f_np, shape, dims, eb, mode)
    out, nb = cz.compress_md(x, eb, mode, dims=dims)
    torch.cuda.synchronize()
    S = int(nb.item())
    assert int(out[6].item()) == st_o, (label, int(out[6].item()), st_o)
    if st_o != oracle.OK:
        return
    assert S == s_o.size, (label, S, s_o.size)
    s_g = out[:S].cpu().numpy()
    if not np.array_equal(s_g, s_o):
        bad = np.nonzero(s_g != s_o)[0]
        raise AssertionError(f"{label}: {bad.size} bytes differ, first at {bad[0]} of {S}")
    st, y_o = oracle.decompress_md(s_o, shape, dims)
    assert st == oracle.OK
    y = cz.decompress_md(out, shape, dims, in_bytes=S)
    torch.cuda.synchronize()
    assert np.array_equal(y.cpu().numpy().ravel().view(np.uint32), y_o.view(np.uint32)), label


@pytest.mark.parametrize("dims,shape", [
    (2, (4, 8)), (2, (13, 37)), (2, (64, 1024)), (2, (100, 500)), (2, (257, 129)), (2, (3, 4100)),
    (2, (5, 7, 33)), (3, (2, 4, 4)), (3, (5, 9, 11)), (3, (20, 50, 50)), (3, (17, 33, 64)), (3, (3, 130, 7)),
])
def test_ragged_shapes(dims, shape):
    rng = np.random.default_rng(sum(shape) + dims)
    f = rng.standard_normal(shape).astype(np.float32)
    for ax in range(len(shape)):
        f = np.cumsum(f, axis=ax).astype(np.float32)
    _parity(f, dims, 1e-3, oracle.REL, f"{dims}D {shape} rel")
    _parity(f, dims, 0.05, oracle.ABS, f"{dims}D {shape} abs")


@pytest.mark.parametrize("field", ["U", "QCLOUD", "TC"])
def test_hurricane_fields(field):
    f = synth.field_for_config("c2_hurricane", device=DEV, scale=0.3, field=field)   # (30, 150, 150) z, y, x
    f = f.reshape(30, 150, 150).cpu().numpy()
    for rel in (1e-2, 1e-4):
        _parity(f, 3, rel, oracle.REL, f"{field} 3D {rel}")
        _parity(f[0], 2, rel, oracle.REL, f"{field} 2D slice {rel}")


def test_guard_and_statuses():
    f = np.zeros((8, 16), np.float32)
    f[3, 5] = 2.0 ** 21                                     # |r0| = 2^21 at 2eb = 1: dims 2 guard
    _parity(f, 2, 0.5, oracle.ABS, "guard 2D")
    f[3, 5] = 2.0 ** 21 - 1
    _parity(f, 2, 0.5, oracle.ABS, "below guard 2D")
    g = np.zeros((4, 8, 8), np.float32)
    g[1, 2, 3] = 2.0 ** 20
    _parity(g, 3, 0.5, oracle.ABS, "guard 3D")
    g[1, 2, 3] = float("nan")
    _parity(g, 3, 0.5, oracle.ABS, "nan 3D")
    # a 1D/2D stream is not a 3D stream
    x = torch.randn(4, 8, 8, device=DEV)
    out, nb = cz.compress_md(x, 1e-3, "rel", dims=3)
    ws = cz.WorkspaceMD((4, 8, 8), 2, DEV)
    cz.decompress_md(out, (4, 8, 8), 2, in_bytes=int(nb.item()), ws=ws)
    assert cz.last_status(ws) == cz.ECORRUPT
    with pytest.raises(ValueError):
        cz.compress_md(x, 1e-3, "rel", dims=4)


@pytest.mark.slow
def test_full_size_nyx_3d():
    """BASELINE configs[3], the NYX-shaped 512^3 field, with the 3D predictor."""
    f = synth.field_for_config("c4_nyx", device=DEV).reshape(512, 512, 512)
    _parity(f.cpu().numpy(), 3, 1e-4, oracle.REL, "nyx 3D")
