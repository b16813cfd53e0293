"""World-size-2 (and 3) CPU tests of the sharded driver over gloo: slab
partitioning, the (min, max) and byte-count all-gathers, the container
header, and the end-to-end claim that shard-wise compression with the
global range decompresses to exactly the single-array result.  The
per-shard compressor is injected (the CPU oracle) because this container
has no GPU; the exchange/header code under test is the product's."""
from __future__ import annotations

import os
import pickle
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from paper_conf_sc_huangd0lc23_b200 import dist as czd


def _free_port() -> int:
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _field(n: int) -> np.ndarray:
    rng = np.random.default_rng(42)
    x = np.cumsum(rng.standard_normal(n)).astype(np.float32)
    x[n // 3: n // 3 + 5000] = 0.0       # a zero stretch (zero blocks)
    return x


def _oracle_range(x: torch.Tensor, mm: torch.Tensor):
    if x.numel() == 0:
        mm[0], mm[1] = float("inf"), float("-inf")
    else:
        lo, hi = oracle.value_range(x.numpy())
        mm[0], mm[1] = lo, hi
    return mm


def _oracle_compress(x: torch.Tensor, rel: float, mm_all: torch.Tensor):
    st, s = oracle.compress_minmax(x.numpy(), rel, mm_all.numpy())
    assert st == oracle.OK
    return torch.from_numpy(s.copy()), torch.tensor([s.size], dtype=torch.int64)


def _worker(rank, world, port, n, rel, outdir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    x = _field(n)
    s0, s1 = czd.slab_bounds(n, rank, world)
    shard_n = [b - a for a, b in (czd.slab_bounds(n, p, world) for p in range(world))]
    res = czd.compress_sharded(torch.from_numpy(x[s0:s1].copy()), rel, shard_n,
                               range_fn=_oracle_range, compress_fn=_oracle_compress)
    with open(os.path.join(outdir, f"r{rank}.pkl"), "wb") as f:
        pickle.dump(dict(bounds=(s0, s1), stream=res.stream.numpy().tobytes(), nbytes=int(res.nbytes.item()),
                         sizes=res.sizes_all.tolist(), header=res.header.tolist(),
                         mm=res.minmax_all.tolist()), f)
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,n", [(2, 100_000), (3, 70_001), (2, 33)])
def test_sharded_compress_gloo(tmp_path, world, n):
    rel = 1e-3
    port = _free_port()
    mp.spawn(_worker, args=(world, port, n, rel, str(tmp_path)), nprocs=world, join=True)
    rs = [pickle.load(open(tmp_path / f"r{p}.pkl", "rb")) for p in range(world)]
    x = _field(n)
    # slabs: disjoint, ordered, block aligned, covering [0, n)
    assert rs[0]["bounds"][0] == 0 and rs[-1]["bounds"][1] == n
    for a, b in zip(rs, rs[1:]):
        assert a["bounds"][1] == b["bounds"][0] and a["bounds"][1] % 32 == 0
    # the all-gathers agree on every rank
    for r in rs:
        assert r["sizes"] == [q["nbytes"] for q in rs]
        assert r["header"] == rs[0]["header"]
        for p, q in enumerate(rs):
            s0, s1 = q["bounds"]
            if s1 > s0:
                assert r["mm"][2 * p] == float(x[s0:s1].min()) and r["mm"][2 * p + 1] == float(x[s0:s1].max())
    # container: header -> assemble -> split round trip
    hdr = czd.parse_container_header(rs[0]["header"])
    assert hdr["P"] == world and hdr["n_total"] == n
    assert hdr["n"] == [r["bounds"][1] - r["bounds"][0] for r in rs]
    assert hdr["offsets"][0] == 0
    buf = czd.assemble_container(rs[0]["header"], [r["stream"] for r in rs])
    h2, shards = czd.split_container(buf)
    assert h2 == hdr and shards == [r["stream"] for r in rs]
    # every shard decompresses; the concatenation equals whole-array REL
    st, whole = oracle.compress(x, rel, oracle.REL)
    st, y_whole = oracle.decompress(whole, n)
    parts = []
    for s, r in zip(shards, rs):
        st, y = oracle.decompress(np.frombuffer(s, np.uint8), r["bounds"][1] - r["bounds"][0])
        assert st == oracle.OK
        parts.append(y)
    y_sharded = np.concatenate(parts)
    assert np.array_equal(y_sharded.view(np.uint32), y_whole.view(np.uint32))


def test_slab_bounds_balanced():
    for n in (0, 1, 31, 32, 1000, 1_705_544_460):
        for P in (1, 2, 4, 8):
            b = [czd.slab_bounds(n, p, P) for p in range(P)]
            assert b[0][0] == 0 and b[-1][1] == n
            nb = [(e - s + 31) // 32 for s, e in b]
            assert max(nb) - min(nb) <= 1


# ---- one concatenated container + distributed decompression

def _oracle_decompress(stream: torch.Tensor, n: int, out: torch.Tensor):
    st, y = oracle.decompress(stream.numpy(), n)
    assert st == oracle.OK
    out.copy_(torch.from_numpy(y))
    return out


def _worker_gather(rank, world, port, n, rel, outdir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    x = _field(n)
    s0, s1 = czd.slab_bounds(n, rank, world)
    shard_n = [b - a for a, b in (czd.slab_bounds(n, p, world) for p in range(world))]
    res = czd.compress_sharded(torch.from_numpy(x[s0:s1].copy()), rel, shard_n,
                               range_fn=_oracle_range, compress_fn=_oracle_compress)
    buf_all = czd.gather_container(res)                 # on every rank
    buf_root = czd.gather_container(res, dst=world - 1)  # on the last rank only
    local = czd.decompress_sharded(buf_all, decompress_fn=_oracle_decompress)
    full = czd.allgather_slabs(local, shard_n)
    with open(os.path.join(outdir, f"g{rank}.pkl"), "wb") as f:
        pickle.dump(dict(buf_all=buf_all.numpy().tobytes(),
                         buf_root=None if buf_root is None else buf_root.numpy().tobytes(),
                         stream=res.stream[: int(res.nbytes.item())].numpy().tobytes(),
                         full=full.numpy().tobytes()), f)
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,n", [(2, 100_000), (3, 70_001), (3, 40)])
def test_gather_container_and_distributed_decompress_gloo(tmp_path, world, n):
    rel = 1e-3
    port = _free_port()
    mp.spawn(_worker_gather, args=(world, port, n, rel, str(tmp_path)), nprocs=world, join=True)
    rs = [pickle.load(open(tmp_path / f"g{p}.pkl", "rb")) for p in range(world)]
    # the gathered container is identical on every rank and on the root, and
    # holds every rank's stream at a 16-byte aligned offset
    for r in rs:
        assert r["buf_all"] == rs[0]["buf_all"]
    assert rs[-1]["buf_root"] == rs[0]["buf_all"]
    assert all(r["buf_root"] is None for r in rs[:-1])
    h, shards = czd.split_container(rs[0]["buf_all"])
    assert [bytes(s) for s in shards] == [r["stream"] for r in rs]
    assert all(o % 16 == 0 for o in h["offsets"]) and czd.container_header_bytes(world) % 16 == 0
    # distributed decompression + slab all-gather == whole-array REL result, bit for bit
    x = _field(n)
    st, whole = oracle.compress(x, rel, oracle.REL)
    st, y_whole = oracle.decompress(whole, n)
    for r in rs:
        assert np.array_equal(np.frombuffer(r["full"], np.uint32), y_whole.view(np.uint32))
    # single-device decompression of the whole container agrees too
    y1 = czd.decompress_container(torch.frombuffer(bytearray(rs[0]["buf_all"]), dtype=torch.uint8),
                                  decompress_fn=_oracle_decompress)
    assert np.array_equal(y1.numpy().view(np.uint32), y_whole.view(np.uint32))
