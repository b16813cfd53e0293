"""GPU tests of SURVEY 8(f) NEXT rank 1 on one B200: a P-shard container of
one array (REL against the global range), decompressed on the device shard
by shard, equals the oracle's whole-array result bit for bit, and every
shard stream equals the oracle's compression of that slab byte for byte.
The NCCL gather path runs on a single-rank process group (the multi-rank
exchange logic is covered over gloo in tests/test_dist_gloo.py)."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist

import oracle
import paper_conf_sc_huangd0lc23_b200 as cz
import synth
from paper_conf_sc_huangd0lc23_b200 import dist as czd

pytestmark = pytest.mark.gpu
DEV = "cuda"


@pytest.mark.parametrize("P,n", [(1, 100_000), (2, 250_001), (3, 1 << 20), (8, 1_000_003), (5, 70)])
def test_container_round_trip_matches_oracle(P, n):
    x = synth.smooth1d(n, seed=P, device=DEV)
    x_np = x.cpu().numpy()
    buf = czd.compress_to_container(x, 1e-4, P)
    h, shards = czd.container_shards(buf)
    assert h["P"] == P and h["n_total"] == n and all(o % 16 == 0 for o in h["offsets"])
    lo, hi = oracle.value_range(x_np)
    mm = np.array([lo, hi], np.float32)
    for p, sh in enumerate(shards):
        s0, s1 = czd.slab_bounds(n, p, P)
        st, s_o = oracle.compress_minmax(x_np[s0:s1], 1e-4, mm)
        assert st == oracle.OK
        assert np.array_equal(sh.cpu().numpy(), s_o), p
    y = czd.decompress_container(buf)
    st, whole = oracle.compress(x_np, 1e-4, oracle.REL)
    st, y_o = oracle.decompress(whole, n)
    assert np.array_equal(y.cpu().numpy().view(np.uint32), y_o.view(np.uint32))


def test_gather_on_single_rank_nccl_group():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        x = synth.smooth1d(300_000, seed=9, device=DEV)
        res = czd.compress_sharded(x, 1e-3, [x.numel()])
        buf = czd.gather_container(res)
        buf_root = czd.gather_container(res, dst=0)
        assert torch.equal(buf, buf_root)
        local = czd.decompress_sharded(buf)
        full = czd.allgather_slabs(local, [x.numel()])
        st, s_o = oracle.compress(x.cpu().numpy(), 1e-3, oracle.REL)
        st, y_o = oracle.decompress(s_o, x.numel())
        assert np.array_equal(full.cpu().numpy().view(np.uint32), y_o.view(np.uint32))
        assert torch.equal(buf, czd.compress_to_container(x, 1e-3, 1))
    finally:
        dist.destroy_process_group()
