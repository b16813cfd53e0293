"""Pins of the CPU oracle against what the paper and the mathematics fix
(-m "not gpu").  Each test names the passage it checks.  None of them
re-types the oracle's formula: they use printed values, hand-worked
blocks, exact rational arithmetic, library routines (numpy cumsum /
min / max, int.bit_length) and an independent bit-level reader."""
from __future__ import annotations

import math
import struct
from fractions import Fraction

import numpy as np
import pytest

import oracle
from tests.conftest import read_golden_blocks, read_paper_values
from tests.format_reader import decode_to_floats, decode_to_ints, parse_header


def f32(v) -> float:
    return float(np.float32(v))


def ulp(x: float) -> float:
    x = abs(np.float32(x))
    return float(np.spacing(x)) if x != 0 else float(np.float32(1.4e-45))


# ---------------------------------------------------------------- paper values

def test_bit_length_printed_values():
    """sec 4.2, Fig 5, Fig 4."""
    rows = [r for r in read_paper_values() if r[0] == "bit_length"]
    assert len(rows) == 4
    for _, m, F in rows:
        assert oracle.bit_length(int(m)) == int(F)
    # special cases: 0 -> 0 (zero block), powers of two, the guard maximum
    assert oracle.bit_length(0) == 0
    for k in range(32):
        assert oracle.bit_length(1 << k) == k + 1 == (1 << k).bit_length()
        assert oracle.bit_length((1 << (k + 1)) - 1) == k + 1


def test_eq2_block_bytes():
    """Eq 2: CmpL = (F+1) L / 8; Fig 5: F=8, L=8 -> 9 bytes."""
    rows = [r for r in read_paper_values() if r[0] == "block_bytes"]
    for _, F, Lb, nb in rows:
        assert oracle.block_bytes(int(F), int(Lb)) == int(nb)
    for F in range(1, 25):
        assert oracle.block_bytes(F, 32) == 4 * (F + 1)
    assert oracle.block_bytes(0, 32) == 0          # zero block


def test_fixed_length_text_example():
    """sec 4.2 example {1,2,5,11,2,0,0,1,0}: max 11 -> 4 bits."""
    row = [r for r in read_paper_values() if r[0] == "fixed_length_example"][0]
    vals = [int(v) for v in row[1].split(",")]
    l = np.zeros(32, np.int32)
    l[: len(vals)] = vals
    F, payload = oracle.encode_block(l)
    assert F == int(row[2]) == 4
    assert len(payload) == 4 * (F + 1)


def test_fig4_lorenzo_reduces_effective_bits():
    """Fig 4: r = 11604 needs 14 bits; with Lorenzo
    the three points become {14, 1, 1} and need 4."""
    r = np.zeros(32, np.int32)
    r[:] = 11606
    r[0:4] = [11590, 11604, 11605, 11606]
    l = oracle.block_lorenzo(r)
    assert list(l[1:4]) == [14, 1, 1]
    assert oracle.bit_length(11604) == 14
    assert oracle.bit_length(max(l[1:4])) == 4
    # the first integer of a block is always predicted from 0
    assert l[0] == r[0]


def test_lorenzo_is_inverted_by_blockwise_cumsum():
    """l_i = r_i - r_{i-1} inside blocks: numpy's cumsum per
    block must give r back, and no block sees its neighbour."""
    rng = np.random.default_rng(0)
    q = rng.integers(-(1 << 22), (1 << 22) + 1, size=32 * 50).astype(np.int32)
    l = oracle.block_lorenzo(q)
    back = np.cumsum(l.reshape(-1, 32).astype(np.int64), axis=1).reshape(-1)
    assert np.array_equal(back, q)
    q2 = q.copy()
    q2[31] += 5                                      # change last of block 0
    l2 = oracle.block_lorenzo(q2)
    assert np.array_equal(l2[32:], l[32:])           # block 1 untouched


def test_eq3_exclusive_scan():
    """Eq 3 / Fig 8: SyncOffset = {0, C0, C0+C1, ...}; the last
    offset plus the last CmpL is the total size."""
    toy = [12, 0, 8, 100]
    assert list(oracle.exclusive_scan(toy)) == [0, 12, 12, 20]
    rng = np.random.default_rng(1)
    c = (rng.integers(0, 26, 10_000) * 4).astype(np.uint64)
    s = oracle.exclusive_scan(c)
    ref = np.concatenate([[0], np.cumsum(c)[:-1]]).astype(np.uint64)
    assert np.array_equal(s, ref)
    assert int(s[-1] + c[-1]) == int(c.sum())


# ---------------------------------------------------------- hand-worked blocks

@pytest.mark.parametrize("row", read_golden_blocks(), ids=lambda r: r[0])
def test_golden_block(row):
    """tests/golden/blocks.txt: payload bytes derived by hand (sec 4.2, 4.4)."""
    name, r, F_exp, cmpl, payload_exp = row
    l = oracle.block_lorenzo(np.array(r, np.int32))
    F, payload = oracle.encode_block(l)
    assert F == F_exp
    assert len(payload) == cmpl == oracle.block_bytes(F, 32)
    assert payload == payload_exp
    assert np.array_equal(oracle.decode_block(payload, F), l)


def test_golden_blocks_through_whole_stream():
    """The same golden blocks placed in one stream with ABS eb = 0.5
    (2eb = 1, so x = r exactly): payloads appear at the exclusive-scan
    offsets after header + align16(nb) (Fig 12)."""
    rows = read_golden_blocks()
    x = np.concatenate([np.array(r, np.float32) for _, r, *_ in rows])
    st, s = oracle.compress(x, 0.5, oracle.ABS)
    assert st == oracle.OK
    nb = len(rows)
    p0 = 32 + ((nb + 15) // 16) * 16
    assert list(s[32:32 + nb]) == [F for _, _, F, _, _ in rows]
    expect = b"".join(p for *_, p in rows)
    assert bytes(s[p0:]) == expect
    assert parse_header(bytes(s))["payload_bytes"] == len(expect)


# ------------------------------------------------------- encode/decode bijection

def _adversarial_blocks():
    rng = np.random.default_rng(2)
    out = []
    for F in range(0, 25):
        hi = (1 << F) - 1
        for _ in range(3):
            l = rng.integers(-hi, hi + 1, 32) if hi > 0 else np.zeros(32, np.int64)
            if F > 0:
                l[rng.integers(0, 32)] = hi if rng.random() < 0.5 else -hi
            out.append(l)
    out.append(-np.arange(1, 33))                       # all negative
    out.append(np.array([(-1) ** j * (j + 1) for j in range(32)]))
    for j in range(32):                                 # single spike per lane
        s = np.zeros(32, np.int64)
        s[j] = 1 << 23
        out.append(s)
        out.append(-s)
    return [np.asarray(b, np.int32) for b in out]


def test_encode_decode_bijection_all_F():
    for l in _adversarial_blocks():
        F, payload = oracle.encode_block(l)
        assert F == int(np.abs(l.astype(np.int64)).max()).bit_length()
        assert len(payload) == (4 * (F + 1) if F else 0)
        assert np.array_equal(oracle.decode_block(payload, F), l)


# ------------------------------------------------------------------ quantiser

def _exact_q_check(x: np.ndarray, eb: float, q: np.ndarray):
    """|x - q 2eb| <= eb in exact rational arithmetic, and q is
    the nearest integer to x / 2eb except at exact ties."""
    E = Fraction(float(np.float32(eb)))
    for xi, qi in zip(x.tolist(), q.tolist()):
        X = Fraction(float(np.float32(xi)))
        res = X - qi * 2 * E
        assert abs(res) <= E, (xi, qi, eb)
        t = X / (2 * E)
        fl = math.floor(t)
        frac = t - fl
        if frac != Fraction(1, 2):
            assert qi == (fl if frac < Fraction(1, 2) else fl + 1)
        else:
            assert qi in (fl, fl + 1)


def test_prequantize_exact_rounding_random():
    rng = np.random.default_rng(3)
    for eb in (1e-4, 0.37, 3.0e-3, 1e-30, 7.0, 2.0 ** -7):
        x = (rng.standard_normal(3000) * rng.choice([1e-3, 1.0, 1e3], 3000) * eb * 1e3).astype(np.float32)
        x = x[np.abs(x / (2 * eb)) < 4e6]
        st, q = oracle.prequantize(x, eb)
        assert st == oracle.OK
        _exact_q_check(x, eb, q)


def test_prequantize_near_half_integers():
    """Inputs one ulp around (k + 1/2) 2eb -- where a plain
    rint(x * (1/2eb)) can pick the wrong neighbour."""
    rng = np.random.default_rng(4)
    xs = []
    for eb in (np.float32(1e-3), np.float32(0.1), np.float32(3.3)):
        k = rng.integers(-(1 << 21), 1 << 21, 400)
        centre = ((k.astype(np.float64) + 0.5) * 2 * float(eb)).astype(np.float32)
        for d in (-2, -1, 0, 1, 2):
            xs.append((np.nextafter(centre, np.float32(np.inf) if d > 0 else np.float32(-np.inf)) if d else centre, eb))
            if abs(d) == 2:
                c2 = np.nextafter(centre, np.float32(np.inf) if d > 0 else np.float32(-np.inf))
                xs.append((np.nextafter(c2, np.float32(np.inf) if d > 0 else np.float32(-np.inf)), eb))
    for x, eb in xs:
        x = x.astype(np.float32)
        st, q = oracle.prequantize(x, float(eb))
        assert st == oracle.OK
        _exact_q_check(x, float(eb), q)


def test_prequantize_guard_and_special_values():
    """R5: |x / 2eb| >= 2^22, NaN or Inf -> ERANGE; -0 -> 0."""
    eb = 0.5
    ok = np.array([4194303.0, -4194303.0, -0.0, 0.0], np.float32)
    st, q = oracle.prequantize(ok, eb)
    assert st == oracle.OK and list(q) == [4194303, -4194303, 0, 0]
    for bad in (4194304.0, -4194304.0, np.inf, -np.inf, np.nan):
        st, _ = oracle.prequantize(np.array([1.0, bad], np.float32), eb)
        assert st == oracle.ERANGE


def test_lossless_when_data_on_the_grid():
    """Special case: x = k 2eb with 2eb a power of two is reproduced
    bit-exactly (the quantiser then loses nothing)."""
    rng = np.random.default_rng(5)
    two_eb = 2.0 ** -7
    k = rng.integers(-(1 << 20), 1 << 20, 5000)
    x = (k * two_eb).astype(np.float32)
    st, s = oracle.compress(x, two_eb / 2, oracle.ABS)
    assert st == oracle.OK
    st, y = oracle.decompress(s, x.size)
    assert st == oracle.OK
    assert np.array_equal(y.view(np.uint32), (x + np.float32(0)).view(np.uint32))


# ------------------------------------------------------------- whole-stream pins

def test_all_zero_input_cr_ceiling():
    """Zero blocks store only their F byte: an
    all-zero field costs header + align16(nb), i.e. CR -> 4L = 128.  Table 3's
    maxima 127.99 / 127.96 / 127.83 / 127.59 all lie below."""
    n = 1 << 24
    st, s = oracle.compress(np.zeros(n, np.float32), 1e-3, oracle.ABS)
    assert st == oracle.OK
    nb = n // 32
    assert s.size == 32 + nb
    cr = 4 * n / s.size
    assert f"{cr:.2f}" == "127.99"
    for r in read_paper_values():
        if r[0] == "cr_ceiling":
            assert float(r[1]) <= 128.0


def _fields():
    rng = np.random.default_rng(6)
    yield "smooth", np.sin(np.arange(4000) / 50.0).astype(np.float32) * 3
    yield "noise", rng.standard_normal(3001).astype(np.float32)
    yield "sparse", (rng.standard_normal(5000) * (rng.random(5000) < 0.05)).astype(np.float32)
    yield "offset", (250.0 + np.cumsum(rng.standard_normal(4097) * 0.01)).astype(np.float32)
    yield "lognormal", np.exp(rng.standard_normal(2000) * 3).astype(np.float32)


@pytest.mark.parametrize("mode", [oracle.ABS, oracle.REL])
def test_stream_matches_independent_reader_and_size_formula(mode):
    """Stream layout read back bit by bit by an independent
    reader; exact size S = 32 + align16(nb) + sum_{F>0} 4 (F+1) (Eq 2)."""
    for name, x in _fields():
        eb = 1e-3 if mode == oracle.REL else 1e-2
        st, s = oracle.compress(x, eb, mode)
        assert st == oracle.OK, name
        buf = bytes(s)
        h, F, r = decode_to_ints(buf)
        assert h["magic"] == b"CSZP" and h["n"] == x.size and h["status"] == 0
        nb = (x.size + 31) // 32
        S = 32 + ((nb + 15) // 16) * 16 + sum(4 * (f + 1) for f in F if f)
        assert len(buf) == S == h["consumed"]
        assert h["payload_bytes"] == S - 32 - ((nb + 15) // 16) * 16
        # pad integers past n are 0 (R8)
        assert all(v == 0 for v in r[x.size:])
        _, y_ref = decode_to_floats(buf)
        st, y = oracle.decompress(s, x.size)
        assert st == oracle.OK
        assert np.array_equal(y.view(np.uint32), y_ref.view(np.uint32))


def test_rel_error_bound_definition():
    """Eq 1: REL eb = lambda (max - min), with numpy's min/max."""
    for _, x in _fields():
        for lam in (1e-2, 1e-3, 1e-4):
            st, s = oracle.compress(x, lam, oracle.REL)
            h = parse_header(bytes(s))
            rng = np.float32(x.max()) - np.float32(x.min())
            assert h["eb_abs"] == f32(np.float32(lam) * rng)
            assert h["eb_in"] == f32(lam) and h["mode"] == 1


@pytest.mark.parametrize("n", list(range(0, 131)))
def test_bruteforce_roundtrip_tiny(n):
    """Every n in [0, 130] (tail blocks): error bounds and exact size."""
    rng = np.random.default_rng(100 + n)
    x = (rng.standard_normal(n) * 10).astype(np.float32)
    if n > 3:
        x[rng.integers(0, n)] = -0.0
    for mode, eb in ((oracle.ABS, 0.01), (oracle.REL, 1e-3), (oracle.ABS, 5.0)):
        st, s = oracle.compress(x, eb, mode)
        if mode == oracle.REL and n > 0 and x.max() == x.min():
            assert st == oracle.ERANGE
            continue
        assert st == oracle.OK
        h = parse_header(bytes(s))
        nb = (n + 31) // 32
        assert s.size == 32 + ((nb + 15) // 16) * 16 + h["payload_bytes"]
        st, y = oracle.decompress(s, n)
        assert st == oracle.OK
        E = h["eb_abs"]
        d = np.abs(y.astype(np.float64) - x.astype(np.float64))
        for xi, yi, di in zip(x, y, d):
            assert di <= E + 0.5 * ulp(yi)          # proved bound
            assert di <= E + ulp(xi)                 # north_star tolerance


def test_error_bound_on_synthetic_fields():
    import synth

    for name in ("c1_smooth1d", "c2_hurricane", "c4_nyx", "c5_rtm"):
        x = synth.field_for_config(name, scale=0.05 if name != "c1_smooth1d" else 0.1).numpy()
        for lam in synth.CONFIGS[name]["rel"]:
            st, s = oracle.compress(x, lam, oracle.REL)
            assert st == oracle.OK
            E = parse_header(bytes(s))["eb_abs"]
            st, y = oracle.decompress(s, x.size)
            d = np.abs(y.astype(np.float64) - x.astype(np.float64))
            tol = E + np.spacing(np.abs(x)).astype(np.float64)
            assert np.all(d <= tol), name


def test_artifact_error_consistent_with_bound():
    """Artifact: max abs error 478.0390625 at REL 1e-4 with
    range 4780302.52 exceeds eb = 478.0302 by less than ulp(max) = 0.5,
    the overshoot our dequantisation bound allows."""
    vals = {r[0]: float(r[1]) for r in read_paper_values() if r[0].startswith("artifact")}
    mn, mx = np.float32(vals["artifact_nyx_min"]), np.float32(vals["artifact_nyx_max"])
    eb = f32(np.float32(1e-4) * (mx - mn))
    assert vals["artifact_nyx_max_abs_err"] > eb
    assert vals["artifact_nyx_max_abs_err"] <= eb + ulp(mx)
    # and our own error near that magnitude respects the same bound
    x = np.linspace(mx * 0.9, mx, 20000, dtype=np.float32)
    st, s = oracle.compress(np.concatenate([[mn], x]).astype(np.float32), 1e-4, oracle.REL)
    st, y = oracle.decompress(s, x.size + 1)
    E = parse_header(bytes(s))["eb_abs"]
    assert np.abs(y[1:].astype(np.float64) - x).max() <= E + ulp(mx)


def test_compress_minmax_matches_rel():
    """Sharded REL: a shard compressed against the global
    (min, max) pairs equals REL compression when the pairs cover the data."""
    rng = np.random.default_rng(7)
    x = rng.standard_normal(10_000).astype(np.float32)
    st, ref = oracle.compress(x, 1e-3, oracle.REL)
    parts = np.array_split(x, 3)
    pairs = np.array([[p.min(), p.max()] for p in parts], np.float32)
    st2, got = oracle.compress_minmax(x, 1e-3, pairs)
    assert st == st2 == oracle.OK and np.array_equal(ref, got)


def test_error_paths():
    x = np.arange(100, dtype=np.float32)
    assert oracle.compress(np.array([1, np.nan], np.float32), 1e-3, oracle.REL)[0] == oracle.ERANGE
    assert oracle.compress(np.array([1, np.inf], np.float32), 1e-3, oracle.ABS)[0] == oracle.ERANGE
    assert oracle.compress(np.full(64, 3.0, np.float32), 1e-3, oracle.REL)[0] == oracle.ERANGE
    assert oracle.compress(x, 1e-9, oracle.ABS)[0] == oracle.ERANGE     # |x/2eb| >= 2^22
    assert oracle.compress(x, 0.0, oracle.ABS)[0] == oracle.EINVAL
    assert oracle.compress(x, -1.0, oracle.REL)[0] == oracle.EINVAL
    assert oracle.compress(x, float("nan"), oracle.ABS)[0] == oracle.EINVAL
    st, s = oracle.compress(x, 1e-3, oracle.REL)
    assert st == oracle.OK
    assert oracle.decompress(s, 99)[0] == oracle.EINVAL                  # wrong n
    assert oracle.decompress(s[:-1], 100)[0] == oracle.ECORRUPT          # truncated
    bad = s.copy(); bad[32] = 25                                          # F > 24
    assert oracle.decompress(bad, 100)[0] == oracle.ECORRUPT
    bad = s.copy(); bad[0] = ord("X")                                     # magic
    assert oracle.decompress(bad, 100)[0] == oracle.ECORRUPT
    bad = s.copy(); bad[33] = (bad[33] + 1) % 25                          # size mismatch
    assert oracle.decompress(bad, 100)[0] == oracle.ECORRUPT
    st, e = oracle.compress(np.array([1, np.nan], np.float32), 1e-3, oracle.ABS)
    assert parse_header(bytes(e))["status"] == oracle.ERANGE
    assert oracle.decompress(e, 2)[0] == oracle.ERANGE


def test_n_zero():
    st, s = oracle.compress(np.zeros(0, np.float32), 1e-3, oracle.REL)
    assert st == oracle.OK and s.size == 32
    assert oracle.decompress(s, 0)[0] == oracle.OK
    assert struct.unpack_from("<Q", bytes(s), 8)[0] == 0
