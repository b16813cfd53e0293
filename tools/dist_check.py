"""Multi-rank check of the sharded driver over NCCL (one GPU per rank, or
every rank on GPU 0 over gloo with CUSZP_BENCH_SHARE_GPU=1): each rank
compresses its block-aligned slab of one RTM-shaped set against the global
range, the container is gathered on every rank and on rank 0, decompressed
across the ranks, and every shard / the whole reconstruction is compared
with the CPU oracle (tests only; launched by tests/test_multi_gpu.py):

    python -m torch.distributed.run --nproc-per-node N --master-addr 127.0.0.1 tools/dist_check.py
"""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np
import torch
import torch.distributed as dist

import oracle
import synth
from paper_conf_sc_huangd0lc23_b200 import dist as czd


def main():
    world, rank = int(os.environ["WORLD_SIZE"]), int(os.environ["RANK"])
    share = os.environ.get("CUSZP_BENCH_SHARE_GPU") == "1"
    dev = torch.device("cuda", 0 if share else int(os.environ["LOCAL_RANK"]))
    torch.cuda.set_device(dev)
    dist.init_process_group("gloo" if share else "nccl", **({} if share else {"device_id": dev}))
    x = synth.field_for_config("c5_rtm", device=dev, scale=0.25)           # same bytes on every rank
    n = x.numel()
    shard_n = [b - a for a, b in (czd.slab_bounds(n, p, world) for p in range(world))]
    s0, s1 = czd.slab_bounds(n, rank, world)
    res = czd.compress_sharded(x[s0:s1].contiguous(), 1e-3, shard_n)
    buf = czd.gather_container(res)
    root = czd.gather_container(res, dst=0)
    root_p2p = czd.gather_container_p2p(res, shard_n, dst=0)          # one-sided, IPC-mapped root buffer
    root_p2p2 = czd.gather_container_p2p(res, shard_n, dst=world - 1, cache_key="last")   # another root, cached mapping
    root_p2p3 = czd.gather_container_p2p(res, shard_n, dst=world - 1, buf=root_p2p2, cache_key="last")
    local = czd.decompress_sharded(buf)
    full = czd.allgather_slabs(local, shard_n)
    x_np = x.cpu().numpy()
    lo, hi = oracle.value_range(x_np)
    st, s_p = oracle.compress_minmax(x_np[s0:s1], 1e-3, np.array([lo, hi], np.float32))
    ok = st == oracle.OK and np.array_equal(res.stream[: int(res.nbytes.item())].cpu().numpy(), s_p)
    st, whole = oracle.compress(x_np, 1e-3, oracle.REL)
    st, y_o = oracle.decompress(whole, n)
    ok &= np.array_equal(full.cpu().numpy().view(np.uint32), y_o.view(np.uint32))
    if rank == 0:
        ok &= torch.equal(buf, root)
        ok &= torch.equal(root_p2p[: buf.numel()], buf)
    if rank == world - 1:
        ok &= torch.equal(root_p2p2[: buf.numel()], buf) and torch.equal(root_p2p3[: buf.numel()], buf)
    flag = torch.tensor([1 if ok else 0], device=dev if not share else "cpu")
    dist.all_reduce(flag, op=dist.ReduceOp.MIN)
    if rank == 0:
        print(f"dist_check world={world} n={n} ok={bool(flag.item())}", flush=True)
    dist.destroy_process_group()
    sys.exit(0 if flag.item() else 1)


if __name__ == "__main__":
    main()
