"""GPU parity of the fused quality reduction (cuszp_quality, SURVEY 8(f)
NEXT rank 2) against oracle.quality on the same seeded inputs.

Bar: exact for the order-independent statistics (min, max, range, max
absolute / relative / point-wise relative error, n, n_over_bound: each a max
or count of identically rounded fp64 values).  Sums are folded in another
order (per-thread, shifted by x[0], then a fixed tree): the fp64 sums of n
terms differ by at most ~n * 2^-53 relative to the sum of magnitudes, so
mse, psnr, nrmse, norm_err and norm_err_norm are compared with rtol 1e-9 and
the Pearson coefficient with atol 1e-9."""
from __future__ import annotations

import math

import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_huangd0lc23_b200 as cz
import synth

pytestmark = pytest.mark.gpu
DEV = "cuda"
EXACT = ("min", "max", "range", "max_abs_err", "max_rel_err", "max_pw_rel_err", "n", "n_over_bound")
RTOL = ("mse", "nrmse", "norm_err", "norm_err_norm")


def same(a, b):
    return a == b or (math.isnan(a) and math.isnan(b))


def check(x_np, y_np, bound, label):
    q_o = oracle.quality(x_np, y_np, bound)
    q_g = cz.quality(torch.from_numpy(x_np).to(DEV), torch.from_numpy(y_np).to(DEV), bound)
    for k in EXACT:
        assert same(q_g[k], q_o[k]), (label, k, q_g[k], q_o[k])
    for k in RTOL:
        assert same(q_g[k], q_o[k]) or math.isclose(q_g[k], q_o[k], rel_tol=1e-9, abs_tol=0.0), (label, k, q_g[k], q_o[k])
    assert same(q_g["psnr"], q_o["psnr"]) or abs(q_g["psnr"] - q_o["psnr"]) < 1e-7, (label, q_g["psnr"], q_o["psnr"])
    if x_np.size > 2:   # n <= 2: 0/0 or +-1 up to rounding
        assert abs(q_g["pearson"] - q_o["pearson"]) < 1e-9, (label, q_g["pearson"], q_o["pearson"])
    return q_g


@pytest.mark.parametrize("n", [1, 3, 4, 5, 31, 4096, 4099, 65_537, 1_000_003])
def test_quality_sizes_and_tails(n):
    rng = np.random.default_rng(n)
    x = (rng.standard_normal(n) * 40 + 7).astype(np.float32)
    y = (x + rng.uniform(-0.01, 0.01, n)).astype(np.float32)
    check(x, y, 0.005, f"n={n}")


def test_quality_misaligned_views():
    rng = np.random.default_rng(3)
    x = rng.standard_normal(10_001).astype(np.float32)
    y = (x * np.float32(1.0001)).astype(np.float32)
    xt, yt = torch.from_numpy(x).to(DEV), torch.from_numpy(y).to(DEV)
    q_o = oracle.quality(x[1:], y[1:], 1e-4)
    q_g = cz.quality(xt[1:], yt[1:], 1e-4)      # 4-byte aligned, not 16: scalar path
    for k in EXACT:
        assert q_g[k] == q_o[k], (k, q_g[k], q_o[k])


@pytest.mark.parametrize("field,rel", [("U", 1e-3), ("QCLOUD", 1e-2), ("TC", 1e-4)])
def test_quality_of_round_trip(field, rel):
    # a real round trip through the CUDA path at reduced Hurricane shape
    x = synth.hurricane_like(field, shape=(20, 100, 100), device=DEV)
    out, nb = cz.compress(x, rel, "rel")
    y = cz.decompress(out, x.numel())
    eb = cz.read_header(out)["eb_abs"]
    q = check(x.cpu().numpy(), y.cpu().numpy(), float(eb), f"{field}@{rel}")
    assert q["max_abs_err"] <= eb + float(np.spacing(np.abs(x.cpu().numpy())).max())


def test_quality_deterministic_and_workspace_reset():
    x = torch.randn(3_000_000, device=DEV)
    y = x + 1e-3 * torch.randn(3_000_000, device=DEV)
    a = cz.quality(x, y, 1e-3)
    b = cz.quality(x, y, 1e-3)
    assert a == b


def test_quality_rejects_bad_args():
    x = torch.zeros(10, device=DEV)
    with pytest.raises(cz.CuszpError):
        cz.quality(x[:0], x[:0])
