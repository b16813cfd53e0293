"""Look-back robustness (SURVEY sec 4 test strategy).

The decoupled look-back of the two scan kernels (internal.cuh: ticketed
persistent CTAs, epoch-tagged status words, ring release in CTA tile order)
is the riskiest concurrency in the library.  Beyond the production grid it is
exercised here by
  * a grid-size sweep: 1, 2, 3, 7 CTAs up to 4 x the SM count (more CTAs than
    can be resident), parity with the oracle at every size;
  * a STRESS build of the library (-DCUSZP_STRESS): pseudo-random sleeps of up
    to ~4 us before 1 in 4 status-word publications, tickets and ring
    releases, so predecessors publish late and out of order -- parity with
    the oracle on every call;
  * compute-sanitizer memcheck / racecheck / synccheck runs of a torch-free
    C driver (tools/sanitize_driver.cu) with exact-size allocations, ragged
    sizes, every block length, the 2-layer predictor and grids of 1, 3 and
    4 x SMs CTAs.
"""
from __future__ import annotations

import ctypes as C
import os
import re
import shutil
import subprocess

import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_huangd0lc23_b200 as cz
import synth
from paper_conf_sc_huangd0lc23_b200 import build as B

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
DEV = "cuda"


def _load(path):
    h = C.CDLL(path)
    sz, vp, i32, f32 = C.c_size_t, C.c_void_p, C.c_int, C.c_float
    h.cuszp_compress_ex.argtypes = [vp, sz, f32, i32, i32, i32, vp, sz, vp, vp, sz, vp]
    h.cuszp_decompress_ex.argtypes = [vp, sz, vp, sz, i32, i32, vp, sz, vp]
    h.cuszp_workspace_bytes.argtypes = [sz]
    h.cuszp_workspace_bytes.restype = sz
    h.cuszp_max_compressed_bytes_L.argtypes = [sz, i32]
    h.cuszp_max_compressed_bytes_L.restype = sz
    h.cuszp_last_status.argtypes = [vp, vp]
    h.cuszp_debug_set_grid.argtypes = [i32, i32]
    return h


def _inputs():
    rng = np.random.default_rng(21)
    return {
        "walk": (np.cumsum(rng.standard_normal(300_001)) * 0.3).astype(np.float32),
        "hurricane_U": synth.field_for_config("c2_hurricane", device=DEV, scale=0.2, field="U").cpu().numpy(),
        "qcloud": synth.field_for_config("c2_hurricane", device=DEV, scale=0.2, field="QCLOUD").cpu().numpy(),
    }


def _round_trip(h, x_np, rel, L=32, order=1):
    """compress + decompress through library handle h; returns (stream, floats)."""
    n = x_np.size
    x = torch.from_numpy(x_np).to(DEV)
    cap = h.cuszp_max_compressed_bytes_L(n, L)
    wsb = h.cuszp_workspace_bytes(n)
    ws = torch.zeros(wsb, dtype=torch.uint8, device=DEV)
    out = torch.empty(cap, dtype=torch.uint8, device=DEV)
    nb = torch.zeros(1, dtype=torch.int64, device=DEV)
    y = torch.empty(n, dtype=torch.float32, device=DEV)
    sp = torch.cuda.current_stream().cuda_stream
    assert h.cuszp_compress_ex(x.data_ptr(), n, rel, cz.REL, L, order, out.data_ptr(), cap, nb.data_ptr(),
                               ws.data_ptr(), wsb, sp) == 0
    assert h.cuszp_last_status(ws.data_ptr(), sp) == 0
    S = int(nb.item())
    assert h.cuszp_decompress_ex(out.data_ptr(), S, y.data_ptr(), n, L, order, ws.data_ptr(), wsb, sp) == 0
    assert h.cuszp_last_status(ws.data_ptr(), sp) == 0
    return out[:S].cpu().numpy(), y.cpu().numpy()


def _check(h, x_np, rel, L=32, order=1, label=""):
    st, s_o = oracle.compress_ex(x_np, rel, oracle.REL, L, order)
    assert st == oracle.OK
    st, y_o = oracle.decompress(s_o, x_np.size)          # reads L and the order from the header
    assert st == oracle.OK
    s_g, y_g = _round_trip(h, x_np, rel, L, order)
    assert np.array_equal(s_g, s_o), label
    assert np.array_equal(y_g.view(np.uint32), y_o.view(np.uint32)), label


def test_grid_size_sweep_matches_oracle():
    """Persistent grids from 1 CTA to 4 x SMs (beyond residency): the same bytes."""
    h = _load(B.LIB)
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    xs = _inputs()
    try:
        for g in (1, 2, 3, 7, sms, 2 * sms, 3 * sms, 4 * sms):
            h.cuszp_debug_set_grid(g, g)
            for name, x_np in xs.items():
                _check(h, x_np, 1e-3, label=f"grid={g} {name}")
            _check(h, xs["walk"], 1e-4, L=64, label=f"grid={g} L=64")
            _check(h, xs["walk"], 1e-4, L=8, label=f"grid={g} L=8")
            _check(h, xs["hurricane_U"], 1e-3, L=16, label=f"grid={g} L=16")
            _check(h, xs["walk"], 1e-4, order=2, label=f"grid={g} order=2")
    finally:
        h.cuszp_debug_set_grid(0, 0)


@pytest.fixture(scope="module")
def stress_lib():
    out = os.path.join(ROOT, "build_variants", "stress.so")
    os.makedirs(os.path.dirname(out), exist_ok=True)
    B.build(defines=["CUSZP_STRESS"], out=out)
    return _load(out)


def test_stress_build_matches_oracle(stress_lib):
    """Random publication delays: every stream and every float still exact,
    including across grid sizes, block lengths and the 2-layer predictor."""
    h = stress_lib
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    xs = _inputs()
    try:
        for g in (0, 5, sms, 4 * sms):
            h.cuszp_debug_set_grid(g, g)
            for rep in range(2):
                for name, x_np in xs.items():
                    _check(h, x_np, 1e-3, label=f"stress grid={g} rep={rep} {name}")
            _check(h, xs["hurricane_U"], 1e-4, L=128, label=f"stress grid={g} L=128")
            _check(h, xs["walk"], 1e-3, L=8, label=f"stress grid={g} L=8")
            _check(h, xs["qcloud"], 1e-4, L=16, label=f"stress grid={g} L=16")
            _check(h, xs["hurricane_U"], 1e-3, order=2, label=f"stress grid={g} order=2")
    finally:
        h.cuszp_debug_set_grid(0, 0)


def _sanitizer():
    for c in (shutil.which("compute-sanitizer"), "/usr/local/cuda/bin/compute-sanitizer"):
        if c and os.path.exists(c):
            return c
    pytest.skip("compute-sanitizer not found")


@pytest.fixture(scope="module")
def sanitize_driver(tmp_path_factory):
    exe = str(tmp_path_factory.mktemp("san") / "sanitize_driver")
    lib_dir = os.path.dirname(B.LIB)
    cz.lib()                                           # the in-tree library exists and is current
    subprocess.run([B.nvcc(), "-gencode", "arch=compute_100a,code=sm_100a", "-o", exe,
                    os.path.join(ROOT, "tools", "sanitize_driver.cu"), "-I", os.path.join(ROOT, "include"),
                    "-L", lib_dir, "-lcuszp", "-Xlinker", "-rpath", "-Xlinker", lib_dir], check=True)
    return exe


def _run_tool(driver, tool, extra=()):
    cmd = [_sanitizer(), "--tool", tool, *extra, driver]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=1500)
    log = r.stdout + r.stderr
    if os.path.isdir(os.path.join(ROOT, "gpurun_out")):
        with open(os.path.join(ROOT, "gpurun_out", f"sanitizer_{tool}.log"), "w") as f:
            f.write(log)
    if "sanitize_driver:" not in log and "ERROR SUMMARY" not in log:
        # the tool refused to run at all (e.g. a pool where compute-sanitizer
        # is administratively disabled): nothing was checked, so skip
        pytest.skip(f"compute-sanitizer did not run the driver: {log.strip()[-300:]}")
    assert "sanitize_driver: 0 failure(s)" in log, log[-4000:]
    return r, log


@pytest.mark.slow
@pytest.mark.parametrize("tool", ["memcheck", "synccheck", "initcheck"])
def test_compute_sanitizer(sanitize_driver, tool):
    extra = ["--error-exitcode", "9"] + (["--leak-check", "full"] if tool == "memcheck" else [])
    r, log = _run_tool(sanitize_driver, tool, extra)
    assert r.returncode == 0, log[-4000:]
    assert "ERROR SUMMARY: 0 errors" in log, log[-4000:]


_SITE = re.compile(r"(\w+\.cu):(\d+)")


@pytest.mark.slow
def test_racecheck_hazards_only_at_documented_handoffs(sanitize_driver):
    """racecheck models __syncthreads / named barriers, but not mbarrier
    arrive/try_wait pairs, acq_rel atomics or fence + volatile-flag protocols:
    it reports every shared-memory hand-off built on those as a hazard.  Each
    such site carries a `// sync: <mechanism>` annotation in the source; this
    test fails on any reported hazard with an endpoint that is not an
    annotated hand-off (a real race), and the stress build and the grid sweep
    above check the protocols themselves."""
    r, log = _run_tool(sanitize_driver, "racecheck", ["--print-limit", "100000"])
    assert "hazards displayed" not in log or "RACECHECK SUMMARY" in log
    src = {}
    for f in os.listdir(os.path.join(ROOT, "paper_conf_sc_huangd0lc23_b200", "csrc")):
        if f.endswith(".cu") or f.endswith(".cuh"):
            with open(os.path.join(ROOT, "paper_conf_sc_huangd0lc23_b200", "csrc", f)) as fh:
                src[f] = fh.read().split("\n")
    bad = set()
    for block in log.split("Race reported between")[1:]:
        for f, ln in _SITE.findall(block.split("========= \n")[0]):
            lines = src.get(f)
            if lines is None or "sync:" not in lines[int(ln) - 1]:
                bad.add(f"{f}:{ln}")
    assert not bad, f"racecheck hazards outside the documented hand-offs: {sorted(bad)}"
