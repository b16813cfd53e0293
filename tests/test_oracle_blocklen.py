"""Pins of the oracle's block-length variants:
L in {8, 16, 64, 128} besides the default 32.

* Eq 2 with Fig 5's printed example: an L = 8 block whose
  largest magnitude is 134 has F = 8 and CmpL = (8 + 1) * 8/8 = 9 bytes;
* a hand-worked L = 8 block (sign byte + 8 plane bytes, "bits with the k-th
  offset into Byte k") and an L = 64 block built from two
  hand-worked 32-element blocks (tests/golden/blocks.txt): a plane of an
  L-block is L/8 bytes with element j at byte j/8, bit j%8;
* the CR ceiling 4L of an all-zero field (one F byte per L values, the
  L = 32 case being Table 3's 127.99);
* the independent bit-level reader (tests/format_reader.py) decodes every
  stream, and the exact size formula 32 + align16(nb) + sum (F+1) L/8;
* the reconstruction does not depend on L (quantisation is per element and
  the in-block Lorenzo step is inverted exactly): floats are bit-identical
  to the L = 32 ones, and the bound of DESIGN sec 5 holds.
"""
from __future__ import annotations

import numpy as np
import pytest

import oracle
from tests import format_reader as fr
from tests.conftest import read_golden_blocks

LS = (8, 16, 64, 128)


def test_fig5_eq2_nine_bytes_at_L8():
    l = np.array([3, -2, 134, 0, -7, 1, 0, 5], np.int32)
    F, payload = oracle.encode_block_L(l, 8)
    assert F == 8 and len(payload) == 9 == oracle.block_bytes(8, 8)
    # hand-worked: sign byte (elements 1 and 4 negative), then planes 0..7
    assert payload.hex() == "12b1179400000000" + "04"
    assert np.array_equal(oracle.decode_block_L(payload, F, 8), l)


def test_L64_block_from_two_golden_32_blocks():
    rows = {name: (vals, hexs) for name, vals, F, cmpl, hexs in read_golden_blocks()}
    pi_vals, pi_hex = rows["pi"]
    ramp_vals, ramp_hex = rows["ramp"]
    l = np.concatenate([oracle.block_lorenzo(np.array(pi_vals, np.int32)),
                        oracle.block_lorenzo(np.array(ramp_vals, np.int32))])
    F, payload = oracle.encode_block_L(l, 64)
    assert F == 3
    # each 8-byte group = the 4-byte group of the first half, then of the second
    pi = [pi_hex[4 * k: 4 * k + 4] for k in range(4)]
    ramp = [ramp_hex[4 * k: 4 * k + 4] if 4 * k + 4 <= len(ramp_hex) else bytes(4) for k in range(4)]
    assert payload == b"".join(a + b for a, b in zip(pi, ramp))
    assert np.array_equal(oracle.decode_block_L(payload, F, 64), l)


@pytest.mark.parametrize("Lb", LS)
def test_cr_ceiling_4L(Lb):
    n = 1 << 20
    st, s = oracle.compress_L(np.zeros(n, np.float32), 1e-3, oracle.ABS, Lb)
    nb = n // Lb
    assert st == oracle.OK and s.size == 32 + ((nb + 15) // 16) * 16
    assert abs(4 * n / s.size - 4 * Lb) / (4 * Lb) < 0.01


@pytest.mark.parametrize("Lb", LS)
@pytest.mark.parametrize("n", [1, 7, 8, 31, 64, 65, 129, 1000, 4099])
def test_reader_size_and_L_independence(Lb, n):
    rng = np.random.default_rng(n * Lb)
    x = np.cumsum(rng.standard_normal(n)).astype(np.float32)
    x[n // 3: n // 2] = 0.0
    x[0] = 50.0
    st, s = oracle.compress_L(x, 1e-3, oracle.REL, Lb)
    if n == 1:      # constant field: REL range 0 (R5)
        assert st == oracle.ERANGE and s[6] == oracle.ERANGE
        return
    assert st == oracle.OK and s[7] == Lb.bit_length() - 1
    h, F, r = fr.decode_to_ints(bytes(s))
    nb = (n + Lb - 1) // Lb
    assert len(F) == nb
    assert s.size == 32 + ((nb + 15) // 16) * 16 + sum((f + 1) * Lb // 8 for f in F if f) == h["consumed"]
    st2, y = oracle.decompress(s, n)
    assert st2 == oracle.OK
    _, y_reader = fr.decode_to_floats(bytes(s))
    assert np.array_equal(y.view(np.uint32), y_reader.view(np.uint32))
    st3, s32 = oracle.compress(x, 1e-3, oracle.REL)
    _, y32 = oracle.decompress(s32, n)
    assert np.array_equal(y.view(np.uint32), y32.view(np.uint32))     # floats independent of L
    eb = np.frombuffer(bytes(s[16:20]), np.float32)[0]
    assert np.all(np.abs(x.astype(np.float64) - y) <= float(eb) + np.spacing(np.abs(x)).astype(np.float64))


@pytest.mark.parametrize("Lb", LS)
def test_brute_force_encode_decode_all_widths(Lb):
    rng = np.random.default_rng(Lb)
    for F in range(0, 25):
        hi = (1 << F) - 1
        l = rng.integers(-hi, hi + 1, Lb).astype(np.int32) if F else np.zeros(Lb, np.int32)
        if F:
            l[rng.integers(Lb)] = hi * (1 if rng.random() < 0.5 else -1)   # the width is reached
        f, p = oracle.encode_block_L(l, Lb)
        assert f == F and len(p) == oracle.block_bytes(F, Lb)
        assert np.array_equal(oracle.decode_block_L(p, f, Lb), l)


def test_invalid_block_length_rejected():
    st, _ = oracle.compress_L(np.ones(10, np.float32), 1e-3, oracle.REL, 48)
    assert st == oracle.EINVAL
