"""The C-ABI library loads here (no GPU) and exports every symbol that
include/cuszp.h declares; host-only helpers agree with the closed forms;
synchronous argument errors are reported without touching a GPU."""
from __future__ import annotations

import ctypes as C
import os
import re
import subprocess

import numpy as np
import pytest

import oracle
from paper_conf_sc_huangd0lc23_b200 import _lib, build

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "cuszp.h")
PKG = os.path.join(ROOT, "paper_conf_sc_huangd0lc23_b200")


def declared_functions() -> list[str]:
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(cuszp_[A-Za-z_0-9]+)\s*\(", src)))


def test_library_builds_and_loads():
    path = build.build()
    assert os.path.exists(path)
    h = _lib.lib()
    assert h.cuszp_version() // 100 == 1


def test_every_declared_symbol_is_exported():
    decl = declared_functions()
    assert len(decl) >= 13
    assert sorted(_lib.SYMBOLS) == decl
    out = subprocess.run(["nm", "-D", "--defined-only", _lib.LIB_PATH], capture_output=True, text=True, check=True).stdout
    exported = set(re.findall(r"\bT (cuszp_\w+)", out))
    missing = [s for s in decl if s not in exported]
    assert not missing, missing
    h = _lib.lib()
    for s in decl:
        assert getattr(h, s) is not None


def test_library_carries_sm100a_code():
    out = subprocess.run(["cuobjdump", "--list-elf", _lib.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_host_helpers_match_closed_forms():
    h = _lib.lib()
    for n in (0, 1, 31, 32, 33, 2047, 2048, 2049, 1 << 20, 280_953_867, 1_705_544_460):
        nb = (n + 31) // 32
        # the buffer bound: the oracle's largest valid stream (25 words per
        # block) plus room for guard-failing garbage blocks (32 words, DESIGN 9.5)
        assert h.cuszp_max_compressed_bytes(n) == oracle.max_compressed_bytes(n) + 4 * 7 * nb
        assert h.cuszp_workspace_bytes(n) >= 128 + 8
    rng = np.random.default_rng(0)
    F = rng.integers(0, 25, 1000).astype(np.uint8)
    F[rng.random(1000) < 0.3] = 0
    exact = 32 + ((1000 + 15) // 16) * 16 + int(sum(4 * (int(f) + 1) for f in F if f))
    assert h.cuszp_compressed_bytes_from_F(F.ctypes.data_as(C.c_void_p), F.size) == exact
    assert h.cuszp_status_string(3) == b"CUSZP_ERANGE"


def test_sync_argument_errors_without_gpu():
    """Validation happens before any CUDA call: these return EINVAL here."""
    h = _lib.lib()
    buf = (C.c_uint8 * 64)()
    p = C.cast(buf, C.c_void_p)
    aligned = (C.addressof(buf) + 15) & ~15
    assert h.cuszp_compress(None, 10, 1e-3, 0, aligned, 10**6, None, aligned, 10**6, None) == _lib.EINVAL
    assert h.cuszp_compress(aligned, 10, 0.0, 0, aligned, 10**6, None, aligned, 10**6, None) == _lib.EINVAL
    assert h.cuszp_compress(aligned, 10, float("nan"), 1, aligned, 10**6, None, aligned, 10**6, None) == _lib.EINVAL
    assert h.cuszp_compress(aligned, 10, 1e-3, 7, aligned, 10**6, None, aligned, 10**6, None) == _lib.EINVAL
    assert h.cuszp_compress(aligned, 10, 1e-3, 1, aligned, 10, None, aligned, 10**6, None) == _lib.ENOSPACE
    assert h.cuszp_decompress(None, 10, aligned, 10, aligned, 10**6, None) == _lib.EINVAL
    assert h.cuszp_range(aligned, 0, None, aligned, 10**6, None) == _lib.EINVAL
    assert h.cuszp_compress_minmax(aligned, 10, 1e-3, None, 1, aligned, 10**6, None, aligned, 10**6, None) == _lib.EINVAL
    del p


def test_product_never_touches_the_oracle():
    """the product package neither imports nor links oracle/."""
    for dirpath, _, files in os.walk(PKG):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                src = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in src and "from oracle" not in src, f
                assert "cuszp_oracle" not in src and "oracle_" not in src, f


def test_binding_rejects_cpu_tensors():
    import torch

    import paper_conf_sc_huangd0lc23_b200 as cz

    with pytest.raises(TypeError):
        cz.compress(torch.zeros(10), 1e-3)


def test_max_compressed_bytes_L_matches_oracle():
    h = _lib.lib()
    for Lb in (8, 16, 32, 64, 128):
        for n in (0, 1, 2, 31, 64, 129, 10**6 + 3):
            nb = (n + Lb - 1) // Lb
            assert h.cuszp_max_compressed_bytes_L(n, Lb) == oracle.max_compressed_bytes_L(n, Lb) + Lb // 8 * 7 * nb
    for bad in (0, 4, 24, 48, 256):
        assert h.cuszp_max_compressed_bytes_L(100, bad) == 0
