"""Pins of oracle.quality against what the paper
and the mathematics fix -- not against a retyped formula:

* the artifact's printed compareData output for the NYX
  temperature field: its PSNR, NRMSE, max relative error and normErr are
  reproduced from inputs constructed to have the printed range and RMSE;
* closed forms on inputs with exactly known errors (every e_i = +-d with d a
  power of two, so MSE = d^2 exactly);
* numpy's corrcoef (a library routine) for the Pearson coefficient;
* brute-force counting for n_over_bound and exact max for the max errors.
"""
from __future__ import annotations

import math

import numpy as np

import oracle

# P:1920-1928 (artifact, NYX temperature.f32, 512^3 points)
P_MIN, P_MAX = 2280.975830078125, 4782583.5
P_RANGE = 4780302.524169921875
P_MAX_ABS = 478.0390625
P_MAX_REL = 0.000100
P_PSNR = 84.770561
P_NRMSE = 5.7739355526161066342e-05
P_NORM_ERR = 3197659.788566
P_N = 512 ** 3


def test_printed_artifact_values_are_consistent():
    # the printed numbers themselves satisfy the definitions the oracle uses
    assert P_MAX - P_MIN == P_RANGE
    assert abs(P_MAX_ABS / P_RANGE - P_MAX_REL) < 5e-7
    assert abs(-20 * math.log10(P_NRMSE) - P_PSNR) < 5e-6
    assert abs(P_NRMSE * P_RANGE * math.sqrt(P_N) - P_NORM_ERR) / P_NORM_ERR < 1e-9


def test_oracle_reproduces_printed_psnr_nrmse():
    # x carries the printed min / max (zero error there); every other point
    # is 3000.0 reconstructed as 3000 +- d with d the printed RMSE rounded to
    # the fp32 grid at 3000 (ulp 2^-12), so y is exact and e_i = -+d.
    n = 1 << 16
    d = round(P_NRMSE * P_RANGE * 4096) / 4096
    x = np.full(n, 3000.0, np.float32)
    x[0], x[1] = P_MIN, P_MAX
    y = x.copy()
    sgn = np.where(np.arange(n) % 2 == 0, 1.0, -1.0)
    y[2:] = (x[2:].astype(np.float64) + sgn[2:] * d).astype(np.float32)
    assert np.all(np.abs(x[2:].astype(np.float64) - y[2:].astype(np.float64)) == d)
    q = oracle.quality(x, y)
    mse = d * d * (n - 2) / n
    assert q["min"] == P_MIN and q["max"] == P_MAX and q["range"] == P_RANGE
    assert q["max_abs_err"] == d
    assert abs(q["mse"] - mse) <= 1e-12 * mse
    # printed PSNR / NRMSE up to the RMSE change of the construction
    rmse_ratio = math.sqrt(mse) / (P_NRMSE * P_RANGE)
    assert abs(q["psnr"] - (P_PSNR - 20 * math.log10(rmse_ratio))) < 2e-6
    assert abs(q["nrmse"] / rmse_ratio - P_NRMSE) < 1e-12
    assert abs(q["norm_err"] - d * math.sqrt(n - 2)) <= 1e-9 * q["norm_err"]


def test_closed_forms_power_of_two_errors():
    rng = np.random.default_rng(11)
    n = 10_007
    x = rng.integers(-1000, 1000, n).astype(np.float32)   # small integers: y = x +- 1/8 exact
    e = np.where(rng.random(n) < 0.5, 0.125, -0.125)
    e[::97] = 0.0
    y = (x.astype(np.float64) - e).astype(np.float32)
    q = oracle.quality(x, y, bound=0.1)
    k = int(np.count_nonzero(e))
    assert q["max_abs_err"] == 0.125
    assert q["mse"] == 0.125 ** 2 * k / n
    assert q["norm_err"] == math.sqrt(0.125 ** 2 * k)
    rng_ = float(x.max()) - float(x.min())
    assert q["range"] == rng_ and q["max_rel_err"] == 0.125 / rng_
    assert abs(q["psnr"] - (20 * math.log10(rng_) - 10 * math.log10(q["mse"]))) < 1e-12
    assert q["n_over_bound"] == k and q["n"] == n
    nz = x != 0
    assert q["max_pw_rel_err"] == float(np.max(np.abs(e[nz]) / np.abs(x[nz].astype(np.float64))))
    assert abs(q["norm_err_norm"] - math.sqrt(0.125 ** 2 * k) / math.sqrt(float(np.sum(x.astype(np.float64) ** 2)))) < 1e-15


def test_pearson_against_numpy_corrcoef():
    rng = np.random.default_rng(12)
    for n in (2, 3, 100, 5000):
        x = rng.standard_normal(n).astype(np.float32) * 300 + 250   # offset field, like Hurricane TC
        y = (x + rng.standard_normal(n).astype(np.float32)).astype(np.float32)
        q = oracle.quality(x, y)
        ref = np.corrcoef(x.astype(np.float64), y.astype(np.float64))[0, 1]
        assert abs(q["pearson"] - ref) < 1e-12, (n, q["pearson"], ref)


def test_lossless_and_degenerate():
    x = np.linspace(-3, 5, 1000, dtype=np.float32)
    q = oracle.quality(x, x.copy(), bound=0.0)
    assert q["max_abs_err"] == 0 and q["mse"] == 0 and q["psnr"] == math.inf and q["n_over_bound"] == 0
    # point-wise relative error skips x = 0
    x = np.array([0.0, 2.0], np.float32)
    y = np.array([1.0, 2.5], np.float32)
    q = oracle.quality(x, y)
    assert q["max_abs_err"] == 1.0 and q["max_pw_rel_err"] == 0.25


def test_round_trip_bound_count_matches_bruteforce():
    # on a real round trip the count of |e| > eb equals a brute-force count
    x = np.sin(np.arange(20_000, dtype=np.float64) / 300).astype(np.float32) * 50
    st, s = oracle.compress(x, 1e-3, oracle.REL)
    assert st == oracle.OK
    st, y = oracle.decompress(s, x.size)
    eb = np.frombuffer(bytes(s[16:20]), np.float32)[0]
    q = oracle.quality(x, y, bound=float(eb))
    brute = int(np.count_nonzero(np.abs(x.astype(np.float64) - y.astype(np.float64)) > float(eb)))
    assert q["n_over_bound"] == brute
    assert q["max_abs_err"] <= float(eb) + float(np.spacing(np.abs(x)).max())


# ---- normErr_norm: the normalisation is fixed by the printed output
P_NORM_ERR_NORM = 0.015479
P_PEARSON = 0.999845


def test_norm_err_norm_reading_forced_by_printed_pearson():
    """Which norm divides normErr?  For ANY x, y: var(x - y) >= var(x) (1 - r^2)
    (minimise sigma_x^2 + sigma_y^2 - 2 r sigma_x sigma_y over sigma_y), so a
    CENTRED normalisation ||e|| / ||x - mean(x)|| >= sqrt(1 - r^2); with the
    printed r = 0.999845 that bound is 0.0176 > the printed 0.015479: the
    centred reading is impossible.  The range-based one is NRMSE (5.77e-5),
    also not the printed value.  The reading ||e||_2 / ||x||_2 needs
    RMS(x) = normErr / normErr_norm / sqrt(n) between sigma_x and max|x| --
    consistent (checked with the construction below)."""
    lower_centred = math.sqrt(1 - P_PEARSON ** 2)
    assert lower_centred > P_NORM_ERR_NORM * 1.1
    assert abs(P_NRMSE - P_NORM_ERR_NORM) > 0.01
    rms_x = P_NORM_ERR / P_NORM_ERR_NORM / math.sqrt(P_N)
    assert P_MIN < rms_x < P_MAX


def test_oracle_reproduces_printed_norm_err_norm_and_pearson():
    """An input with the printed RMSE, Pearson coefficient and normErr_norm
    under the ||x||_2 reading: x = mu + s z, e = d w with z, w = +-1 patterns
    orthogonal to each other and to 1 (mean error 0, cov(x, e) = 0), so
    r = s / sqrt(s^2 + d^2) and normErr_norm = d / sqrt(mu^2 + s^2).  The
    oracle must print both values back to the paper's 6 digits."""
    n = 1 << 16
    d = 0.25 * round(P_NRMSE * P_RANGE * 4)                    # 276.0, exact in fp32 arithmetic below
    s = d * P_PEARSON / math.sqrt(1 - P_PEARSON ** 2)
    rms = d / P_NORM_ERR_NORM
    mu = math.sqrt(rms * rms - s * s)
    s, mu = float(np.float32(s)), float(np.float32(mu))
    i = np.arange(n)
    z = np.where((i // 2) % 2 == 0, 1.0, -1.0)                 # + + - - ...
    w = np.where(i % 2 == 0, 1.0, -1.0)                        # + - + - ...
    assert z.sum() == 0 and w.sum() == 0 and (z * w).sum() == 0
    x = (mu + s * z).astype(np.float32)
    y = (x.astype(np.float64) - d * w).astype(np.float32)
    assert np.array_equal(x.astype(np.float64) - y.astype(np.float64), d * w)   # errors exact
    q = oracle.quality(x, y)
    assert abs(q["norm_err"] / math.sqrt(n) - d) < 1e-9 * d
    assert round(q["pearson"], 6) == P_PEARSON, q["pearson"]
    assert round(q["norm_err_norm"], 6) == P_NORM_ERR_NORM, q["norm_err_norm"]
    # and the centred reading would have printed a different number
    xc = x.astype(np.float64) - x.astype(np.float64).mean()
    assert round(q["norm_err"] / math.sqrt(float((xc * xc).sum())), 6) != P_NORM_ERR_NORM


def test_norm_err_norm_closed_forms():
    """Hand-computed values: x = 4 everywhere, e = +-1/4 -> ||e|| = sqrt(n)/4,
    ||x|| = 4 sqrt(n), ratio exactly 1/16; x = (3, 4) pairs with e = 1/2 on
    the 4s only -> ratio = sqrt(n/2 * 1/4) / sqrt(n/2 * 25) = 1/10."""
    n = 1024
    x = np.full(n, 4.0, np.float32)
    y = (x + np.where(np.arange(n) % 2 == 0, 0.25, -0.25)).astype(np.float32)
    assert oracle.quality(x, y)["norm_err_norm"] == 1 / 16
    x = np.tile(np.array([3.0, 4.0], np.float32), n // 2)
    y = x.copy()
    y[1::2] = 3.5
    assert abs(oracle.quality(x, y)["norm_err_norm"] - 0.1) < 1e-16
