"""Pins of the multi-dimensional Lorenzo predictor of the oracle (SURVEY
8(f) NEXT rank 4; "Lorenzo predictions with higher dimensions", P:535-545;
DESIGN R18): blocks of 1x4x8 (2D) or 2x4x4 (3D) points of the field,
neighbours outside the block count as 0.

What pins it (none of it retypes the oracle's formula):
  * hand-worked blocks: a linear field leaves only the block's edges
    (l = c at the corner, the slopes along the first row / column / plane),
    a bilinear / trilinear one a constant 1 in the interior; one full
    payload worked out by hand to hex;
  * the predictor is the mixed finite difference: numpy.diff along each axis
    of the zero-padded block (a library routine) gives the same l;
  * its inverse is the cumulative sum along each axis: numpy.cumsum over the
    l decoded by the independent format reader reproduces the oracle's
    reconstruction bit for bit;
  * the error bound |x - x'| <= eb + ulp(x) on ragged shapes, the R18 guard,
    and the raster order of the block grid.
"""
from __future__ import annotations

import numpy as np
import pytest

import oracle
from tests.format_reader import decode_l_blocks, parse_header

BOX = {2: (1, 4, 8), 3: (2, 4, 4)}


def _block_coords(dims):
    bz, by, bx = BOX[dims]
    z, y, x = np.meshgrid(np.arange(bz), np.arange(by), np.arange(bx), indexing="ij")
    return z.ravel(), y.ravel(), x.ravel()


def test_linear_block_leaves_only_edges():
    z, y, x = _block_coords(2)
    r = 3 * y - 2 * x + 5
    l = oracle.block_lorenzo_md(r, 2)
    want = np.zeros(32, np.int64)
    want[(y == 0) & (x == 0)] = 5
    want[(y == 0) & (x > 0)] = -2
    want[(y > 0) & (x == 0)] = 3
    assert np.array_equal(l, want)
    z, y, x = _block_coords(3)
    r = 7 * z + 3 * y - 2 * x + 5
    l = oracle.block_lorenzo_md(r, 3)
    want = np.zeros(32, np.int64)
    want[(z == 0) & (y == 0) & (x == 0)] = 5
    want[(z == 0) & (y == 0) & (x > 0)] = -2
    want[(z == 0) & (y > 0) & (x == 0)] = 3
    want[(z > 0) & (y == 0) & (x == 0)] = 7
    assert np.array_equal(l, want)


def test_multilinear_block_is_constant_inside():
    z, y, x = _block_coords(2)
    l = oracle.block_lorenzo_md(x * y, 2)
    assert np.array_equal(l, ((x > 0) & (y > 0)).astype(np.int64))
    z, y, x = _block_coords(3)
    l = oracle.block_lorenzo_md(x * y * z, 3)
    assert np.array_equal(l, ((x > 0) & (y > 0) & (z > 0)).astype(np.int64))


def test_hand_worked_payload_2d():
    """Field 4x8 = one 2D block, r = 3y - 2x + 5 (2eb = 1 so x = r exactly):
    l = 5 at (0,0), -2 on the rest of row 0, 3 on the rest of column 0.
    max |l| = 5 -> F = 3, CmpL = 16 bytes (Eq 2):
      sign map: elements 1..7 negative                      -> fe 00 00 00
      plane 0 : |l| odd at j = 0 (5), 8, 16, 24 (3)         -> 01 01 01 01
      plane 1 : bit 1 at j = 1..7 (2) and 8, 16, 24 (3)     -> fe 01 01 01
      plane 2 : bit 2 at j = 0 (5)                          -> 01 00 00 00"""
    y, x = np.meshgrid(np.arange(4), np.arange(8), indexing="ij")
    f = (3 * y - 2 * x + 5).astype(np.float32)
    st, s = oracle.compress_md(f, (4, 8), 2, 0.5, oracle.ABS)
    assert st == oracle.OK
    h = parse_header(bytes(s))
    assert h["mode"] == 0x20 and h["n"] == 32 and h["payload_bytes"] == 16
    assert s[32] == 3
    assert bytes(s[48:]).hex() == "fe000000" "01010101" "fe010101" "01000000"
    st, y2 = oracle.decompress_md(s, (4, 8), 2)
    assert st == oracle.OK and np.array_equal(y2, f.ravel())


def _blocks_of(field, dims):
    """Field (nz, ny, nx) -> list of zero-padded blocks (bz, by, bx) in raster order."""
    bz, by, bx = BOX[dims]
    nz, ny, nx = field.shape
    pz, py, px = -(-nz // bz) * bz, -(-ny // by) * by, -(-nx // bx) * bx
    pad = np.zeros((pz, py, px), field.dtype)
    pad[:nz, :ny, :nx] = field
    out = []
    for kz in range(pz // bz):
        for ky in range(py // by):
            for kx in range(px // bx):
                out.append(pad[kz * bz:(kz + 1) * bz, ky * by:(ky + 1) * by, kx * bx:(kx + 1) * bx])
    return out, (pz, py, px)


@pytest.mark.parametrize("dims,shape", [(2, (13, 37)), (2, (4, 8)), (2, (9, 1)), (3, (5, 9, 11)), (3, (2, 4, 4)),
                                        (3, (3, 1, 7))])
def test_predictor_is_mixed_difference_and_cumsum_inverts_it(dims, shape):
    rng = np.random.default_rng(sum(shape) * dims)
    shape3 = (1,) * (3 - len(shape)) + tuple(shape)
    f = np.cumsum(np.cumsum(rng.standard_normal(shape3), axis=-1), axis=-2).astype(np.float32)
    eb = 0.05
    st, s = oracle.compress_md(f, shape, dims, eb, oracle.ABS)
    assert st == oracle.OK
    nb = oracle.num_blocks_md(shape, dims)
    h, F, lblocks = decode_l_blocks(bytes(s), nb)
    assert h["consumed"] == s.size
    # r of every block, independently: R2's nearest integer (exact rational)
    two_eb = np.float32(eb) + np.float32(eb)
    st, q = oracle.prequantize(f.ravel(), eb)
    assert st == oracle.OK
    rblocks, _ = _blocks_of(q.reshape(shape3).astype(np.int64), dims)
    bz, by, bx = BOX[dims]
    for k, (rb, lb) in enumerate(zip(rblocks, lblocks)):
        # forward: numpy.diff of the zero-padded block along every axis
        d = np.pad(rb, ((1, 0), (1, 0), (1, 0)))
        for ax in range(3):
            if BOX[dims][ax] > 1:
                d = np.diff(d, axis=ax)
            else:
                d = d[1:] if ax == 0 else d
        assert np.array_equal(np.asarray(lb).reshape(bz, by, bx), d.reshape(bz, by, bx)), k
        # inverse: cumulative sums along every axis
        rr = np.asarray(lb, np.int64).reshape(bz, by, bx)
        for ax in range(3):
            rr = np.cumsum(rr, axis=ax)
        assert np.array_equal(rr, rb), k
    st, y = oracle.decompress_md(s, shape, dims)
    assert st == oracle.OK
    # the reconstruction = r * 2eb (R13) from the independently decoded r
    r_field = np.zeros(_blocks_of(np.zeros(shape3), dims)[1], np.int64)
    pz, py, px = r_field.shape
    k = 0
    for kz in range(pz // bz):
        for ky in range(py // by):
            for kx in range(px // bx):
                rr = np.asarray(lblocks[k], np.int64).reshape(bz, by, bx)
                for ax in range(3):
                    rr = np.cumsum(rr, axis=ax)
                r_field[kz * bz:(kz + 1) * bz, ky * by:(ky + 1) * by, kx * bx:(kx + 1) * bx] = rr
                k += 1
    want = (r_field[:shape3[0], :shape3[1], :shape3[2]].astype(np.float32) * two_eb).astype(np.float32)
    assert np.array_equal(y.view(np.uint32), want.ravel().view(np.uint32))
    ulp = np.spacing(np.abs(f.ravel()).astype(np.float32)).astype(np.float64)
    assert np.all(np.abs(f.ravel().astype(np.float64) - y.astype(np.float64)) <= eb + ulp)


def test_raster_order_of_the_block_grid():
    """Only block (by=1, bx=2) of a 8x24 field is non-zero: F[1*3 + 2] != 0 only."""
    f = np.zeros((8, 24), np.float32)
    f[4:8, 16:24] = 9.0
    st, s = oracle.compress_md(f, (8, 24), 2, 0.5, oracle.ABS)
    F = s[32:32 + 6]
    assert [int(v) for v in F] == [0, 0, 0, 0, 0, 4]
    f3 = np.zeros((4, 8, 8), np.float32)
    f3[2:4, 4:8, 0:4] = 1.0                                # block (kz=1, ky=1, kx=0) of the 2x2x2 grid
    st, s = oracle.compress_md(f3, (4, 8, 8), 3, 0.5, oracle.ABS)
    F = [int(v) for v in s[32:40]]
    assert F == [0, 0, 0, 0, 0, 0, 1, 0]


def test_guard_and_rel_bound():
    # dims 2: |r0| < 2^21; dims 3: < 2^20 (R18: |l| < 2^23)
    for dims, g in ((2, 2 ** 21), (3, 2 ** 20)):
        f = np.zeros((4, 8), np.float32)
        f[1, 1] = g - 1
        assert oracle.compress_md(f, (4, 8), dims, 0.5, oracle.ABS)[0] == oracle.OK
        f[1, 1] = g
        assert oracle.compress_md(f, (4, 8), dims, 0.5, oracle.ABS)[0] == oracle.ERANGE
    # REL: eb_abs = lambda * (max - min) exactly as the 1D path (Eq 1)
    f = np.linspace(-3, 7, 4 * 8 * 5, dtype=np.float32).reshape(5, 4, 8)
    st, s = oracle.compress_md(f, f.shape, 3, 1e-3, oracle.REL)
    st1, s1 = oracle.compress(f.ravel(), 1e-3, oracle.REL)
    assert parse_header(bytes(s))["eb_abs"] == parse_header(bytes(s1))["eb_abs"]
