"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bar: compressed bytes identical (hence CR identical) and
decompressed floats bit-identical, on the same seeded inputs.  Sizes span
many tiles (4096 elements each) and ragged tails; full BASELINE sizes are
compared byte for byte and bit for bit on every config (c1-c4 every field and
bound; c5 as one 6.82 GB stream and as an 8-shard container)."""
from __future__ import annotations

import numpy as np
import pytest
import torch

import oracle
import paper_conf_sc_huangd0lc23_b200 as cz
import synth
from tests.conftest import read_golden_blocks

pytestmark = pytest.mark.gpu
DEV = "cuda"


def gpu_compress(x: torch.Tensor, eb: float, mode: int, ws=None):
    out, nbytes = cz.compress(x, eb, mode, ws=ws)
    torch.cuda.synchronize()
    n = int(nbytes.item())
    return out[:n].cpu().numpy(), out


def gpu_decompress(stream_np: np.ndarray, n: int, ws=None):
    buf = torch.zeros(max(stream_np.size, 16) + 16, dtype=torch.uint8, device=DEV)
    buf[: stream_np.size] = torch.from_numpy(stream_np).to(DEV)
    y = cz.decompress(buf, n, in_bytes=stream_np.size, ws=ws)
    torch.cuda.synchronize()
    return y.cpu().numpy()


def assert_parity(x_np: np.ndarray, eb: float, mode: int, ws=None, label=""):
    x = torch.from_numpy(x_np).to(DEV)
    st_o, s_o = oracle.compress(x_np, eb, mode)
    s_g, _ = gpu_compress(x, eb, mode, ws=ws)
    assert s_g[6] == st_o, (label, int(s_g[6]), st_o)    # header status byte
    if st_o != oracle.OK:
        return s_o, None
    assert s_g.size == s_o.size, (label, s_g.size, s_o.size)
    if not np.array_equal(s_g, s_o):
        bad = np.nonzero(s_g != s_o)[0]
        raise AssertionError(f"{label}: {bad.size} bytes differ, first at {bad[0]} of {s_o.size}")
    st, y_o = oracle.decompress(s_o, x_np.size)
    assert st == oracle.OK
    y_g = gpu_decompress(s_o, x_np.size, ws=ws)
    assert np.array_equal(y_g.view(np.uint32), y_o.view(np.uint32)), label
    return s_o, y_o


# --------------------------------------------------------------- small cases

def test_golden_blocks_on_gpu():
    rows = read_golden_blocks()
    x = np.concatenate([np.array(r, np.float32) for _, r, *_ in rows])
    s, _ = assert_parity(x, 0.5, oracle.ABS, label="golden")
    nb = len(rows)
    p0 = 32 + ((nb + 15) // 16) * 16
    assert bytes(s[p0:]) == b"".join(p for *_, p in rows)


@pytest.mark.parametrize("n", [0, 1, 2, 31, 32, 33, 63, 64, 65, 127, 128, 129, 2047, 2048, 2049,
                               4095, 4096, 4097, 2048 * 7 + 33, 2048 * 64 - 1, 2048 * 148 + 5])
def test_sizes_and_tails(n):
    rng = np.random.default_rng(n)
    x = (np.cumsum(rng.standard_normal(n)) * 0.3).astype(np.float32)
    if n == 0:
        s_g, _ = gpu_compress(torch.zeros(0, device=DEV), 1e-3, oracle.REL)
        st, s_o = oracle.compress(x, 1e-3, oracle.REL)
        assert np.array_equal(s_g, s_o)
        return
    for mode, eb in ((oracle.REL, 1e-3), (oracle.ABS, 0.05), (oracle.REL, 1e-5)):
        if mode == oracle.REL and x.max() == x.min():
            continue
        assert_parity(x, eb, mode, label=f"n={n} mode={mode} eb={eb}")


def test_distributions_and_special_values():
    rng = np.random.default_rng(11)
    n = 50_000
    cases = {
        "gauss": rng.standard_normal(n),
        "sparse": rng.standard_normal(n) * (rng.random(n) < 0.02),
        "zeros_and_negzero": np.where(rng.random(n) < 0.5, -0.0, 0.0) + (np.arange(n) > n // 2) * 1.0,
        "lognormal": np.exp(rng.standard_normal(n) * 2),
        "lognormal_overflow": np.exp(rng.standard_normal(n) * 4),   # ERANGE at ABS 1e-3 on both sides
        "subnormal": rng.standard_normal(n) * 1e-39,
        "grid": rng.integers(-1000, 1000, n) * 2.0 ** -7,
        "halfpoints": (rng.integers(-(1 << 20), 1 << 20, n) + 0.5) * 2e-3,
        "steps": np.repeat(rng.standard_normal(n // 100 + 1), 100)[:n],
    }
    for name, v in cases.items():
        x = v.astype(np.float32)
        assert_parity(x, 1e-3, oracle.ABS, label=name + "/abs")
        if x.max() > x.min():
            assert_parity(x, 1e-4, oracle.REL, label=name + "/rel")


@pytest.mark.parametrize("name", ["c1_smooth1d", "c2_hurricane", "c3_hacc", "c4_nyx", "c5_rtm"])
def test_config_recipes_small(name):
    """Every BASELINE config's recipe at reduced size, every eb, every field."""
    fields = synth.CONFIGS[name].get("fields", [None])
    for f in fields:
        x = synth.field_for_config(name, device=DEV, scale=0.08 if name != "c1_smooth1d" else 1.0, field=f)
        x_np = x.cpu().numpy()
        for rel in synth.CONFIGS[name]["rel"]:
            assert_parity(x_np, rel, oracle.REL, label=f"{name}/{f}/{rel}")


def test_cross_decode_and_determinism():
    x_np = synth.field_for_config("c2_hurricane", device=DEV, scale=0.2, field="U").cpu().numpy()
    x = torch.from_numpy(x_np).to(DEV)
    first, _ = gpu_compress(x, 1e-3, oracle.REL)
    for _ in range(20):
        again, _ = gpu_compress(x, 1e-3, oracle.REL)
        assert np.array_equal(first, again)
    # oracle decodes the GPU stream (and the GPU the oracle stream, above)
    st, y_o = oracle.decompress(first, x_np.size)
    assert st == oracle.OK
    y_g = gpu_decompress(first, x_np.size)
    assert np.array_equal(y_g.view(np.uint32), y_o.view(np.uint32))


def test_value_range_and_minmax_api():
    rng = np.random.default_rng(3)
    x_np = (rng.standard_normal(1_000_003) * 7 + 3).astype(np.float32)
    x = torch.from_numpy(x_np).to(DEV)
    mm = cz.value_range(x).cpu().numpy()
    assert mm[0] == x_np.min() and mm[1] == x_np.max()
    for off in range(1, 4):   # unaligned starts take the scalar path
        mm = cz.value_range(x[off:]).cpu().numpy()
        assert mm[0] == x_np[off:].min() and mm[1] == x_np[off:].max()
    parts = np.array_split(x_np, 4)
    pairs = np.array([[p.min(), p.max()] for p in parts], np.float32)
    st, s_o = oracle.compress_minmax(x_np, 1e-3, pairs)
    out, nb = cz.compress_minmax(x, 1e-3, torch.from_numpy(pairs.ravel()).to(DEV))
    torch.cuda.synchronize()
    assert np.array_equal(out[: int(nb.item())].cpu().numpy(), s_o)


def test_async_error_statuses():
    ws = cz.Workspace(1 << 16)
    x = torch.arange(1000, dtype=torch.float32, device=DEV)
    bad = x.clone(); bad[500] = float("nan")
    cz.compress(bad, 1e-3, "rel", ws=ws)
    assert cz.last_status(ws) == cz.ERANGE
    cz.compress(bad, 1e-3, "abs", ws=ws)
    assert cz.last_status(ws) == cz.ERANGE
    cz.compress(torch.full((100,), 2.0, device=DEV), 1e-3, "rel", ws=ws)
    assert cz.last_status(ws) == cz.ERANGE
    cz.compress(x, 1e-9, "abs", ws=ws)                       # |x/2eb| >= 2^22
    assert cz.last_status(ws) == cz.ERANGE
    out, nb = cz.compress(x, 1e-3, "rel", ws=ws)
    assert cz.last_status(ws) == cz.OK
    n = int(nb.item())
    y = torch.empty(1000, device=DEV)
    cz.decompress(out, 999, out=torch.empty(999, device=DEV), in_bytes=n, ws=ws)
    assert cz.last_status(ws) == cz.EINVAL
    cz.decompress(out, 1000, out=y, in_bytes=n - 4, ws=ws)      # truncated
    assert cz.last_status(ws) == cz.ECORRUPT
    c = out.clone(); c[32] = 25                                   # F > 24
    cz.decompress(c, 1000, out=y, in_bytes=n, ws=ws)
    assert cz.last_status(ws) == cz.ECORRUPT
    c = out.clone(); c[33] = (int(c[33]) + 1) % 25                # sizes disagree with header
    cz.decompress(c, 1000, out=y, in_bytes=n + 400, ws=ws)
    assert cz.last_status(ws) == cz.ECORRUPT
    c = out.clone(); c[0] = 0                                     # magic
    cz.decompress(c, 1000, out=y, in_bytes=n, ws=ws)
    assert cz.last_status(ws) == cz.ECORRUPT
    cz.decompress(out, 1000, out=y, in_bytes=n, ws=ws)            # and the workspace still works
    assert cz.last_status(ws) == cz.OK
    st, y_o = oracle.decompress(out[:n].cpu().numpy(), 1000)
    assert np.array_equal(y.cpu().numpy(), y_o)


def test_fuzzed_streams_never_fault():
    """Byte-flipped F arrays / headers must only ever produce a status."""
    rng = np.random.default_rng(5)
    x = torch.from_numpy(rng.standard_normal(70_000).astype(np.float32)).to(DEV)
    out, nb = cz.compress(x, 1e-3, "rel")
    n = int(nb.item())
    assert cz.read_header(out)["status"] == cz.OK, cz.read_header(out)
    assert n > 32 + 2200 + 16, n
    base = out[:n].clone()
    ws = cz.Workspace(70_000)
    y = torch.empty(70_000, device=DEV)
    for i in range(60):
        c = base.clone()
        pos = rng.integers(0, 32 + 2200, 3)
        for p in pos:
            c[int(p)] = int(rng.integers(0, 256))
        cz.decompress(c, 70_000, out=y, in_bytes=n, ws=ws)
        st = cz.last_status(ws)
        assert st in (cz.OK, cz.ECORRUPT, cz.EINVAL, cz.ERANGE)
    cz.decompress(base, 70_000, out=y, in_bytes=n, ws=ws)
    assert cz.last_status(ws) == cz.OK


def test_workspace_reuse_and_epoch_wrap():
    """Epoch-tagged look-back words: many calls of varying
    size on one workspace, including across the epoch limit, stay exact."""
    ws = cz.Workspace(300_000)
    rng = np.random.default_rng(9)
    xs = [rng.standard_normal(int(m)).astype(np.float32) for m in (300_000, 5000, 120_001, 2048, 299_999)]
    refs = [oracle.compress(v, 1e-3, oracle.REL)[1] for v in xs]
    for rep in range(3):
        for v, r in zip(xs, refs):
            s, _ = gpu_compress(torch.from_numpy(v).to(DEV), 1e-3, oracle.REL, ws=ws)
            assert np.array_equal(s, r)
    # jump to just below the epoch limit (ws ctrl word 0 = epoch)
    ws.buf[:4] = torch.tensor([(1 << 23) - 3], dtype=torch.int32).view(torch.uint8).to(DEV)
    for rep in range(3):
        for v, r in zip(xs, refs):
            s, _ = gpu_compress(torch.from_numpy(v).to(DEV), 1e-3, oracle.REL, ws=ws)
            assert np.array_equal(s, r)
            y = gpu_decompress(r, v.size, ws=ws)
            assert np.array_equal(y, oracle.decompress(r, v.size)[1])


def test_host_e2e_api():
    x_np = synth.field_for_config("c4_nyx", device=DEV, scale=0.1).cpu().numpy()
    n = x_np.size
    ws = cz.Workspace(n)
    d_in = torch.empty(n, dtype=torch.float32, device=DEV)
    d_out = torch.empty(cz.max_compressed_bytes(n), dtype=torch.uint8, device=DEV)
    h_in = torch.from_numpy(x_np).pin_memory()
    h_out = torch.empty(cz.max_compressed_bytes(n), dtype=torch.uint8).pin_memory()
    nbytes = cz.compress_host(h_in, 1e-4, "rel", h_out, d_in, d_out, ws)
    st, s_o = oracle.compress(x_np, 1e-4, oracle.REL)
    assert nbytes == s_o.size and np.array_equal(h_out[:nbytes].numpy(), s_o)
    h_y = torch.empty(n, dtype=torch.float32).pin_memory()
    d_y = torch.empty(n, dtype=torch.float32, device=DEV)
    cz.decompress_host(h_out, nbytes, h_y, d_out, d_y, ws)
    assert np.array_equal(h_y.numpy(), oracle.decompress(s_o, n)[1])


# ------------------------------------------------------- full BASELINE sizes

def _equal_chunked(dev_t: torch.Tensor, ref: np.ndarray, step: int = 1 << 28) -> bool:
    """dev_t (any CUDA tensor) byte-identical to the numpy array ref, compared
    in chunks so multi-GB arrays never need a second full host copy."""
    a = dev_t.contiguous().view(torch.uint8)
    b = ref.view(np.uint8)
    if a.numel() != b.size:
        return False
    for s0 in range(0, b.size, step):
        if not np.array_equal(a[s0:s0 + step].cpu().numpy(), b[s0:s0 + step]):
            return False
    return True


@pytest.mark.slow
@pytest.mark.parametrize("name", ["c1_smooth1d", "c2_hurricane", "c3_hacc", "c4_nyx"])
def test_full_size_bytes(name):
    """Full BASELINE sizes in the bench's launch configuration: for every
    field and every REL bound of the config the whole stream and the whole
    reconstruction are compared with the oracle."""
    for f in synth.CONFIGS[name].get("fields", [None]):
        x = synth.field_for_config(name, device=DEV, field=f)
        x_np = x.cpu().numpy()
        for rel in synth.CONFIGS[name]["rel"]:
            st, s_o = oracle.compress(x_np, rel, oracle.REL)
            assert st == oracle.OK, (name, f, rel, st)
            out, nb = cz.compress(x, rel, "rel")
            torch.cuda.synchronize()
            assert int(nb.item()) == s_o.size, (name, f, rel)
            assert _equal_chunked(out[: s_o.size], s_o), (name, f, rel)
            y = cz.decompress(out, x.numel(), in_bytes=int(nb.item()))
            st, y_o = oracle.decompress(s_o, x_np.size)
            assert st == oracle.OK
            assert _equal_chunked(y, y_o), (name, f, rel)
            del out, y, y_o, s_o
        del x, x_np
        torch.cuda.empty_cache()


@pytest.mark.slow
@pytest.mark.parametrize("name", list(synth.DATASETS))
def test_full_size_datasets(name):
    """The bench's six-dataset table (synth.DATASETS: the paper's Table 2 field
    shapes) at every bound it reports, REL 1e-2 / 1e-3 / 1e-4:
    every field's whole stream and whole reconstruction against the oracle,
    in the launch configuration bench.py times."""
    for f in synth.DATASETS[name]["fields"]:
        x = synth.dataset_field(name, f, device=DEV)
        x_np = x.cpu().numpy()
        for rel in synth.DATASET_RELS:
            st, s_o = oracle.compress(x_np, rel, oracle.REL)
            assert st == oracle.OK, (name, f, rel, st)
            out, nb = cz.compress(x, rel, "rel")
            torch.cuda.synchronize()
            assert int(nb.item()) == s_o.size, (name, f, rel)
            assert _equal_chunked(out[: s_o.size], s_o), (name, f, rel)
            y = cz.decompress(out, x.numel(), in_bytes=int(nb.item()))
            st, y_o = oracle.decompress(s_o, x_np.size)
            assert st == oracle.OK
            assert _equal_chunked(y, y_o), (name, f, rel)
            del out, y, y_o, s_o
        del x, x_np
        torch.cuda.empty_cache()


@pytest.mark.slow
def test_full_size_rtm_bit_exact():
    """The 6.82 GB RTM-shaped set (BASELINE configs[4], 1,705,544,460 fp32),
    every byte and every float:
      P = 1: the whole-array stream equals oracle.compress's byte for byte and
             decompresses to oracle.decompress's floats bit for bit;
      P = 8: the 8-shard container (block-aligned slabs, REL against the
             GLOBAL range -- the north_star split) holds, shard by
             shard, oracle.compress_minmax of that slab with the global range,
             and the container decompresses to the same whole-array floats."""
    from paper_conf_sc_huangd0lc23_b200 import dist as czd

    rel = synth.CONFIGS["c5_rtm"]["rel"][0]
    x = synth.field_for_config("c5_rtm", device=DEV)
    n = x.numel()
    assert n == 1_705_544_460
    x_np = x.cpu().numpy()
    lo, hi = oracle.value_range(x_np)
    mm = cz.value_range(x).cpu().numpy()
    assert (mm[0], mm[1]) == (np.float32(lo), np.float32(hi))

    # P = 1, whole array
    st, s_o = oracle.compress(x_np, rel, oracle.REL)
    assert st == oracle.OK
    out, nb = cz.compress(x, rel, "rel")
    torch.cuda.synchronize()
    assert int(nb.item()) == s_o.size
    assert _equal_chunked(out[: s_o.size], s_o)
    y = cz.decompress(out, n, in_bytes=int(nb.item()))
    del out
    st, y_o = oracle.decompress(s_o, n)
    assert st == oracle.OK
    assert _equal_chunked(y, y_o)
    del y, s_o
    torch.cuda.empty_cache()

    # P = 8 shards against the global range
    P = 8
    buf = czd.compress_to_container(x, rel, P)
    h, shards = czd.container_shards(buf)
    assert h["P"] == P and h["n_total"] == n
    mm_np = np.array([lo, hi], np.float32)
    for p in range(P):
        s0, s1 = czd.slab_bounds(n, p, P)
        assert s0 % 32 == 0 and h["n"][p] == s1 - s0
        st, s_p = oracle.compress_minmax(x_np[s0:s1], rel, mm_np)
        assert st == oracle.OK
        assert _equal_chunked(shards[p], s_p), p
        del s_p
    del x
    torch.cuda.empty_cache()
    yc = czd.decompress_container(buf)
    assert _equal_chunked(yc, y_o)


@pytest.mark.parametrize("Lb", [32, 64, 128])
def test_guard_failures_never_write_past_capacity(Lb):
    """Data failing the R5 guard (|x/2eb| >= 2^22, NaN, Inf) encode garbage
    blocks before the status is known: the kernel must still stay inside
    cuszp_max_compressed_bytes_L(n, L) (a canary after the buffer)."""
    n = 1000
    cap = cz.max_compressed_bytes(n, Lb)
    for x in (torch.arange(n, dtype=torch.float32, device=DEV) * 1e6,
              torch.full((n,), float("inf"), device=DEV),
              torch.full((n,), float("nan"), device=DEV)):
        buf = torch.full((cap + 4096,), 0xA5, dtype=torch.uint8, device=DEV)
        out_bytes = torch.zeros(1, dtype=torch.int64, device=DEV)
        cz.compress(x, 1e-9, "abs", out=buf[:cap], out_bytes=out_bytes, block_len=Lb)
        torch.cuda.synchronize()
        assert cz.read_header(buf)["status"] == cz.ERANGE
        assert bool((buf[cap:] == 0xA5).all()), "wrote past the capacity"


def test_cuda_graph_capture_and_replay():
    """The device calls never allocate or synchronise: range + compress +
    decompress (launched with programmatic dependent launch) capture into a
    CUDA graph whose replays reproduce the eager bytes and floats."""
    x_np = synth.smooth1d(300_000, seed=4, device="cpu").numpy()
    x = torch.from_numpy(x_np).to(DEV)
    n = x.numel()
    ws = cz.Workspace(n)
    out = torch.empty(cz.max_compressed_bytes(n), dtype=torch.uint8, device=DEV)
    nb = torch.zeros(1, dtype=torch.int64, device=DEV)
    y = torch.empty(n, device=DEV)
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):                      # warm-up outside capture (library init)
        cz.compress(x, 1e-4, "rel", out=out, out_bytes=nb, ws=ws, stream=s)
        cz.decompress(out, n, out=y, ws=ws, stream=s)
    s.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        cz.compress(x, 1e-4, "rel", out=out, out_bytes=nb, ws=ws, stream=s)
        cz.decompress(out, n, out=y, ws=ws, stream=s)
    st, s_o = oracle.compress(x_np, 1e-4, oracle.REL)
    st, y_o = oracle.decompress(s_o, n)
    for _ in range(3):
        out.zero_(); y.zero_()
        g.replay()
        torch.cuda.synchronize()
        assert int(nb.item()) == s_o.size
        assert np.array_equal(out[: s_o.size].cpu().numpy(), s_o)
        assert np.array_equal(y.cpu().numpy().view(np.uint32), y_o.view(np.uint32))
