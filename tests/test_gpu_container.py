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


@pytest.mark.parametrize("P,n", [(1, 100_000), (3, 1 << 20), (8, 1_000_003), (5, 70)])
def test_container_put_places_shards_from_the_device_header(P, n):
    """cuszp_container_put (the one-sided gather's copy kernel) reads each
    shard's size and offset from the DEVICE-side header: P puts into one
    capacity-sized buffer (no host read of the sizes) give the container
    compress_to_container assembles on the host, byte for byte."""
    x = synth.smooth1d(n, seed=P + 10, device=DEV)
    mm = cz.value_range(x)
    streams, sizes, shard_n = [], [], []
    for p in range(P):
        s0, s1 = czd.slab_bounds(n, p, P)
        shard_n.append(s1 - s0)
        out, nb = cz.compress_minmax(x[s0:s1], 1e-4, mm)
        streams.append(out)
        sizes.append(nb.view(1).to(torch.int64))
    hdr = czd.container_header(shard_n, torch.cat(sizes))
    buf = torch.full((czd.container_capacity(shard_n),), 0xAB, dtype=torch.uint8, device=DEV)
    for p in reversed(range(P)):                       # any order
        cz.check(cz.lib().cuszp_container_put(streams[p].data_ptr(), hdr.data_ptr(), P, p, buf.data_ptr(),
                                              int(p == 0), torch.cuda.current_stream().cuda_stream), "put")
    ref = czd.compress_to_container(x, 1e-4, P)
    assert torch.equal(buf[: ref.numel()], ref)
    with pytest.raises(cz.CuszpError):
        cz.check(cz.lib().cuszp_container_put(streams[0].data_ptr(), hdr.data_ptr(), P, P, buf.data_ptr(), 0, None),
                 "put p >= P")


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
        buf_p2p = czd.gather_container_p2p(res, [x.numel()])
        assert torch.equal(buf_p2p[: buf.numel()], buf)
        local = czd.decompress_sharded(buf)
        full = czd.allgather_slabs(local, [x.numel()])
        st, s_o = oracle.compress(x.cpu().numpy(), 1e-3, oracle.REL)
        st, y_o = oracle.decompress(s_o, x.numel())
        assert np.array_equal(full.cpu().numpy().view(np.uint32), y_o.view(np.uint32))
        assert torch.equal(buf, czd.compress_to_container(x, 1e-3, 1))
    finally:
        dist.destroy_process_group()
