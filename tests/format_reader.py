"""Independent, bit-by-bit pure-Python reader of the stream layout written
down in DESIGN.md sec 4 (header, fixed-length bytes, 16-byte pad, block
payloads of sign map + bit planes).  Test helper: it pins the oracle's
byte layout against the document (and is used on tiny streams only).
It does not reuse any oracle or product code."""
from __future__ import annotations

import struct


def parse_header(buf: bytes) -> dict:
    magic = buf[0:4]
    version, mode, status, log2l = buf[4], buf[5], buf[6], buf[7]
    (n,) = struct.unpack_from("<Q", buf, 8)
    eb_abs, eb_in = struct.unpack_from("<ff", buf, 16)
    (payload,) = struct.unpack_from("<Q", buf, 24)
    return dict(magic=magic, version=version, mode=mode, status=status, log2l=log2l,
                n=n, eb_abs=eb_abs, eb_in=eb_in, payload_bytes=payload)


def decode_to_ints(buf: bytes) -> tuple[dict, list[int], list[int]]:
    """Returns (header, per-block F list, quantisation integers r_0..r_{32nb-1})."""
    h = parse_header(buf)
    Lb = 1 << h["log2l"]
    n = h["n"]
    nb = (n + Lb - 1) // Lb
    F = list(buf[32:32 + nb])
    pos = 32 + ((nb + 15) // 16) * 16
    r_all = []
    for k in range(nb):
        f = F[k]
        if f == 0:
            r_all.extend([0] * Lb)
            continue
        nbytes = (f + 1) * Lb // 8
        blk = buf[pos:pos + nbytes]
        pos += nbytes
        r, r1, r2 = 0, 0, 0
        order2 = bool(h["mode"] & 0x10)          # 2-layer Lorenzo (DESIGN R17)
        for j in range(Lb):
            neg = (blk[j // 8] >> (j % 8)) & 1
            mag = 0
            for p in range(f):
                byte = blk[(p + 1) * (Lb // 8) + j // 8]
                mag |= ((byte >> (j % 8)) & 1) << p
            l = -mag if neg else mag
            if order2:
                r = l + 2 * r1 - r2
                r2, r1 = r1, r
            else:
                r += l
            r_all.append(r)
    h["consumed"] = pos
    return h, F, r_all


def decode_to_floats(buf: bytes):
    import numpy as np

    h, F, r = decode_to_ints(buf)
    two_eb = np.float32(h["eb_abs"]) + np.float32(h["eb_abs"])
    q = np.array(r[: h["n"]], dtype=np.float32)
    return h, (q * two_eb).astype(np.float32)


def decode_l_blocks(buf: bytes, nb: int) -> tuple[dict, list[int], list[list[int]]]:
    """The Lorenzo integers l of each of nb L-blocks (no inverse prediction):
    for streams whose block count is not ceil(n / L), e.g. the
    multi-dimensional predictor's block grid (DESIGN R18)."""
    h = parse_header(buf)
    Lb = 1 << h["log2l"]
    F = list(buf[32:32 + nb])
    pos = 32 + ((nb + 15) // 16) * 16
    out = []
    for k in range(nb):
        f = F[k]
        if f == 0:
            out.append([0] * Lb)
            continue
        nbytes = (f + 1) * Lb // 8
        blk = buf[pos:pos + nbytes]
        pos += nbytes
        ls = []
        for j in range(Lb):
            neg = (blk[j // 8] >> (j % 8)) & 1
            mag = 0
            for p in range(f):
                mag |= ((blk[(p + 1) * (Lb // 8) + j // 8] >> (j % 8)) & 1) << p
            ls.append(-mag if neg else mag)
        out.append(ls)
    h["consumed"] = pos
    return h, F, out
