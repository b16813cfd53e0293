"""Pins of the 2-layer Lorenzo predictor (the
"Lorenzo predictions with higher ... layers" of P:535-545; DESIGN R17):
l_i = r_i - 2 r_{i-1} + r_{i-2} inside each block, r_{-1} = r_{-2} = 0.

* closed forms: a linear ramp r_i = a + b i leaves l = [a, b - a, 0, ...];
  a quadratic r_i = i^2 leaves l = [0, 1, 2, 2, ...] (hand-worked payloads);
* the guard tightens to |r0| < 2^21 (so |l| <= 2^23, F <= 24);
* the reconstruction equals the 1-layer one bit for bit (the predictor is
  inverted exactly), the independent reader decodes every stream.
"""
from __future__ import annotations

import numpy as np
import pytest

import oracle
from tests import format_reader as fr


def _stream_of_block(r_block, order):
    # x = r * 2eb with 2eb = 1 (eb = 0.5, ABS): quantisation is exact
    x = np.asarray(r_block, np.float32)
    st, s = oracle.compress_ex(x, 0.5, oracle.ABS, 32, order)
    assert st == oracle.OK
    return s


def test_linear_ramp_payload_hand_worked():
    # r_i = 5 + 3 i: l = [5, -2, 0, ...] -> F = 3; sign map bit 1;
    # planes: bit0 {5} -> elem 0; bit1 {2} -> elem 1; bit2 {5} -> elem 0
    s = _stream_of_block([5 + 3 * i for i in range(32)], 2)
    assert s[5] == 0x10 and s[32] == 3
    assert bytes(s[48:]).hex() == "02000000" "01000000" "02000000" "01000000"


def test_quadratic_payload_hand_worked():
    # r_i = i^2: l = [0, 1, 2, 2, ..., 2] -> F = 2, no signs;
    # plane 0: elem 1; plane 1: elems 2..31
    s = _stream_of_block([i * i for i in range(32)], 2)
    assert s[32] == 2
    assert bytes(s[48:]).hex() == "00000000" "02000000" "fcffffff"


def test_guard_is_2_to_21_for_order_2():
    x = np.full(64, float((1 << 21) + 7), np.float32)          # |r0| in [2^21, 2^22)
    st1, _ = oracle.compress_ex(x, 0.5, oracle.ABS, 32, 1)
    st2, s2 = oracle.compress_ex(x, 0.5, oracle.ABS, 32, 2)
    assert st1 == oracle.OK and st2 == oracle.ERANGE and s2[6] == oracle.ERANGE
    x[:] = float((1 << 21) - 1)
    assert oracle.compress_ex(x, 0.5, oracle.ABS, 32, 2)[0] == oracle.OK


@pytest.mark.parametrize("n", [1, 2, 3, 31, 33, 1000, 70_001])
def test_round_trip_equals_order_1_and_reader(n):
    rng = np.random.default_rng(n)
    x = np.cumsum(rng.standard_normal(n)).astype(np.float32) + 3
    x[: n // 4] = 0.0
    st, s2 = oracle.compress_ex(x, 1e-3, oracle.ABS, 32, 2)
    assert st == oracle.OK and s2[5] == 0x10
    st, y2 = oracle.decompress(s2, n)
    st1, s1 = oracle.compress_ex(x, 1e-3, oracle.ABS, 32, 1)
    _, y1 = oracle.decompress(s1, n)
    assert np.array_equal(y2.view(np.uint32), y1.view(np.uint32))
    h, F, r = fr.decode_to_ints(bytes(s2))
    assert h["consumed"] == s2.size
    _, y_reader = fr.decode_to_floats(bytes(s2))
    assert np.array_equal(y_reader.view(np.uint32), y2.view(np.uint32))
