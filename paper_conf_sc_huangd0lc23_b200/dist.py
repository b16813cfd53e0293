"""Sharded multi-GPU driver.

One process per GPU.  The global 1D array is split into contiguous,
32-element-block-aligned slabs (rank p owns blocks [p nb / P, (p+1) nb / P)),
so blocks never straddle ranks and the paper's per-block independence
 makes every shard an ordinary cuSZp stream.  The only
exchanges (both stream-ordered, no host synchronisation):

 1. REL: all-gather of every rank's (min, max) -- 8 B per rank over
    NVLink -- so all ranks quantise against the GLOBAL value range
    (Eq 1); the compression kernel reduces the P pairs itself.
 2. all-gather of every rank's compressed byte count (8 B per rank), from
    which the container header (per-shard n, bytes, offsets) is built.

Every shard's decompressed floats equal the single-GPU result bit for bit
(same eb_abs, block-aligned slabs).

SURVEY 8(f) NEXT rank 1 -- one concatenated stream and distributed
decompression:
 3. ``gather_container``: the shard streams are moved into ONE container
    buffer (header words + every shard at a 16-byte aligned offset) on one
    rank (NCCL point-to-point receives straight into the slices) or on every
    rank (one NCCL broadcast per shard into its slice);
    ``gather_container_p2p``: the same container on one rank with no host
    read of the sizes -- every rank's copy kernel writes its shard into the
    root's (IPC-mapped) buffer at the offset the device-side header gives;
 4. ``decompress_container``: decompresses all shards of a container on one
    GPU (one launch per shard, each writing its slab of the output), and
    ``decompress_sharded`` + ``allgather_slabs`` decompress a container
    across P GPUs, rank p taking shard p.
"""
from __future__ import annotations

import struct
from dataclasses import dataclass

import torch
import torch.distributed as dist

BLOCK = 32
CONTAINER_MAGIC = 0x544E4F43505A5343  # "CSZPCONT" little-endian
CONTAINER_VERSION = 2        # v2: shard offsets and the payload base 16-byte aligned


def slab_bounds(n_total: int, rank: int, world: int) -> tuple[int, int]:
    """Element range [start, end) of rank's block-aligned slab."""
    nb = (n_total + BLOCK - 1) // BLOCK
    b0 = (rank * nb) // world
    b1 = ((rank + 1) * nb) // world
    return min(b0 * BLOCK, n_total), min(b1 * BLOCK, n_total)


def _nccl(group) -> bool:
    return dist.get_backend(group) == "nccl"


def _allgather(dst: torch.Tensor, src: torch.Tensor, group) -> torch.Tensor:
    if _nccl(group):
        dist.all_gather_into_tensor(dst, src, group=group)
    else:
        # gloo (CPU tests; several ranks sharing one GPU): host staging
        world = dist.get_world_size(group)
        parts = [torch.empty_like(src, device="cpu") for _ in range(world)]
        dist.all_gather(parts, src.cpu(), group=group)
        dst.copy_(torch.cat(parts).view(-1))
    return dst


def _broadcast(t: torch.Tensor, src: int, group) -> None:
    if _nccl(group) or not t.is_cuda:
        dist.broadcast(t, src=src, group=group)
    else:
        tmp = t.cpu()
        dist.broadcast(tmp, src=src, group=group)
        t.copy_(tmp)


def _send(t: torch.Tensor, dst: int, group) -> None:
    dist.send(t if (_nccl(group) or not t.is_cuda) else t.cpu(), dst=dst, group=group)


def allgather_minmax(mm_local: torch.Tensor, mm_all: torch.Tensor, group=None) -> torch.Tensor:
    """(min, max) of every rank -> mm_all[2 P] (device, stream-ordered)."""
    return _allgather(mm_all, mm_local, group)


def allgather_sizes(out_bytes: torch.Tensor, group=None, sizes_all: torch.Tensor | None = None) -> torch.Tensor:
    """Compressed byte count (int64[1]) of every rank -> int64[P]."""
    world = dist.get_world_size(group)
    if sizes_all is None:
        sizes_all = torch.empty(world, dtype=torch.int64, device=out_bytes.device)
    return _allgather(sizes_all, out_bytes.view(1), group)


def container_header(shard_n: list[int], sizes_all: torch.Tensor) -> torch.Tensor:
    """u64 words: magic, version, P, n_total, n_p[P], bytes_p[P], offset_p[P]
    (offsets relative to the end of this header).  Built on the device from
    the all-gathered sizes -- no host round trip."""
    P = len(shard_n)
    dev = sizes_all.device
    n = torch.tensor(shard_n, dtype=torch.int64, device=dev)
    padded = (sizes_all.to(torch.int64) + 15) // 16 * 16    # every shard 16-byte aligned (TMA sources)
    offs = torch.cumsum(padded, 0) - padded
    head = torch.tensor([CONTAINER_MAGIC - (1 << 64) if CONTAINER_MAGIC >= 1 << 63 else CONTAINER_MAGIC,
                         CONTAINER_VERSION, P, int(sum(shard_n))], dtype=torch.int64, device=dev)
    return torch.cat([head, n, sizes_all.to(torch.int64), offs])


def container_header_bytes(P: int) -> int:
    """Bytes before the first shard: the header words, padded to 16."""
    return (8 * (4 + 3 * P) + 15) // 16 * 16


@dataclass
class ShardResult:
    stream: torch.Tensor          # this rank's cuSZp stream buffer (capacity-sized)
    nbytes: torch.Tensor          # int64[1] exact length (device)
    sizes_all: torch.Tensor       # int64[P] every rank's exact length (device)
    header: torch.Tensor          # int64 container header words (device)
    minmax_all: torch.Tensor      # float32[2P] every rank's (min, max)


def _cuda_range(x, mm):
    import paper_conf_sc_huangd0lc23_b200 as cz

    if x.numel() == 0:
        mm[0], mm[1] = float("inf"), float("-inf")
        return mm
    return cz.value_range(x, out=mm)


def _cuda_compress_minmax(x, rel, mm_all):
    import paper_conf_sc_huangd0lc23_b200 as cz

    return cz.compress_minmax(x, rel, mm_all)


def compress_sharded(x_local: torch.Tensor, rel: float, shard_n: list[int], group=None,
                     range_fn=None, compress_fn=None) -> ShardResult:
    """REL-compress this rank's slab against the global range.

    ``range_fn(x, mm_out)`` / ``compress_fn(x, rel, mm_all) -> (stream,
    nbytes)`` default to the CUDA path; tests on CPU (gloo) inject other
    implementations to exercise the exchange and header logic."""
    range_fn = range_fn or _cuda_range
    compress_fn = compress_fn or _cuda_compress_minmax
    world = dist.get_world_size(group)
    dev = x_local.device
    mm_local = torch.empty(2, dtype=torch.float32, device=dev)
    range_fn(x_local, mm_local)
    mm_all = torch.empty(2 * world, dtype=torch.float32, device=dev)
    allgather_minmax(mm_local, mm_all, group)
    stream, nbytes = compress_fn(x_local, rel, mm_all)
    sizes_all = allgather_sizes(nbytes.view(1).to(torch.int64), group)
    hdr = container_header(shard_n, sizes_all)
    return ShardResult(stream, nbytes, sizes_all, hdr, mm_all)


def parse_container_header(words) -> dict:
    w = [int(v) & ((1 << 64) - 1) for v in (words.tolist() if hasattr(words, "tolist") else words)]
    if w[0] != CONTAINER_MAGIC or w[1] != CONTAINER_VERSION:
        raise ValueError("not a cuSZp container header")
    P = w[2]
    return dict(P=P, n_total=w[3], n=w[4:4 + P], bytes=w[4 + P:4 + 2 * P], offsets=w[4 + 2 * P:4 + 3 * P])


def assemble_container(header_words, shard_streams: list[bytes]) -> bytes:
    """Host-side concatenation: container header + every shard's stream at
    its offset (what a gather of the payloads to one rank produces)."""
    h = parse_container_header(header_words)
    head = struct.pack(f"<{4 + 3 * h['P']}Q", *[int(v) & ((1 << 64) - 1) for v in
                                                (header_words.tolist() if hasattr(header_words, "tolist") else header_words)])
    head = head + bytes(container_header_bytes(h["P"]) - len(head))
    body = bytearray(container_total_bytes(h) - len(head))
    for p, s in enumerate(shard_streams):
        assert len(s) == h["bytes"][p]
        body[h["offsets"][p]:h["offsets"][p] + len(s)] = s
    return head + bytes(body)


def split_container(buf: bytes) -> tuple[dict, list[bytes]]:
    P = struct.unpack_from("<Q", buf, 16)[0]
    words = struct.unpack_from(f"<{4 + 3 * P}Q", buf, 0)
    h = parse_container_header(words)
    base = container_header_bytes(P)
    return h, [buf[base + o: base + o + b] for o, b in zip(h["offsets"], h["bytes"])]


def container_total_bytes(h: dict) -> int:
    """Length of the container described by a parsed header."""
    if h["P"] == 0:
        return container_header_bytes(0)
    return container_header_bytes(h["P"]) + h["offsets"][-1] + h["bytes"][-1]


def _header_bytes_tensor(header_words: torch.Tensor) -> torch.Tensor:
    raw = header_words.contiguous().view(torch.uint8)
    P = (header_words.numel() - 4) // 3
    pad = container_header_bytes(P) - raw.numel()
    return torch.cat([raw, torch.zeros(pad, dtype=torch.uint8, device=raw.device)]) if pad else raw


def gather_container(res: ShardResult, group=None, dst: int | None = None) -> torch.Tensor | None:
    """Materialise the concatenated container (header + every shard stream)
    from the sharded compression result.

    dst=None: on every rank (one broadcast per shard, straight into that
    shard's slice of the container); dst=r: only on rank r (point-to-point
    receives into the slices; other ranks send and return None).  One host
    read of the P all-gathered sizes (8 B each) sizes the slices."""
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    h = parse_container_header(res.header.cpu())
    base = container_header_bytes(world)
    total = container_total_bytes(h)
    dev = res.stream.device
    mine = res.stream[: h["bytes"][rank]]
    if dst is not None and rank != dst:
        if h["bytes"][rank]:
            _send(mine.contiguous(), dist.get_global_rank(group, dst) if group is not None else dst, group)
        return None
    buf = torch.zeros(total, dtype=torch.uint8, device=dev)
    buf[:base] = _header_bytes_tensor(res.header)
    views = [buf[base + o: base + o + b] for o, b in zip(h["offsets"], h["bytes"])]
    views[rank].copy_(mine)
    if dst is None:
        for p in range(world):
            if h["bytes"][p]:
                src = dist.get_global_rank(group, p) if group is not None else p
                _broadcast(views[p], src, group)
    elif _nccl(group) or not buf.is_cuda:
        ops = []
        for p in range(world):
            if p != rank and h["bytes"][p]:
                src = dist.get_global_rank(group, p) if group is not None else p
                ops.append(dist.P2POp(dist.irecv, views[p], src, group))
        if ops:
            for w in dist.batch_isend_irecv(ops):
                w.wait()
    else:
        for p in range(world):                               # gloo + CUDA buffers: host staging
            if p != rank and h["bytes"][p]:
                src = dist.get_global_rank(group, p) if group is not None else p
                tmp = torch.empty(views[p].numel(), dtype=torch.uint8)
                dist.recv(tmp, src=src, group=group)
                views[p].copy_(tmp)
    return buf


def container_capacity(shard_n: list[int]) -> int:
    """Bytes that hold a container of these shards whatever their sizes: the
    header plus every shard's align16(cuszp_max_compressed_bytes(n_p))."""
    import paper_conf_sc_huangd0lc23_b200 as cz

    return container_header_bytes(len(shard_n)) + sum((cz.max_compressed_bytes(n) + 15) // 16 * 16 for n in shard_n)


_peer_cache: dict = {}
_inflight: list = []     # (IPC view, event): mappings kept alive until the puts through them completed


def _peer_view(buf: torch.Tensor | None, dst: int, group, cache_key=None) -> torch.Tensor:
    """Every rank gets a device tensor aliasing rank dst's ``buf`` (CUDA IPC:
    the handle travels as a small host object; a rank on another GPU then
    writes it over NVLink / UVA).  With a cache_key the mapping is made once
    and reused by every later call with that key -- ALL ranks must pass the
    same keys, and dst the same buffer for a key."""
    from torch.multiprocessing.reductions import reduce_tensor

    if cache_key is not None and cache_key in _peer_cache:
        return _peer_cache[cache_key][0]
    rank = dist.get_rank(group)
    obj = [reduce_tensor(buf) if rank == dst else None]
    dist.broadcast_object_list(obj, src=dist.get_global_rank(group, dst) if group is not None else dst, group=group)
    view = buf if rank == dst else obj[0][0](*obj[0][1])
    if cache_key is not None:
        _peer_cache[cache_key] = (view, obj[0])
    return view


def gather_container_p2p(res: ShardResult, shard_n: list[int], group=None, dst: int = 0,
                         buf: torch.Tensor | None = None, cache_key=None) -> torch.Tensor | None:
    """One-sided gather of the container on rank ``dst`` with no host read
    of the sizes: every rank's copy kernel (cuszp_container_put) writes its
    shard straight into dst's buffer -- mapped by CUDA IPC, so over NVLink
    when dst is another GPU -- at the offset the DEVICE-side header gives it,
    and rank dst writes the header.  An all-reduce of one word after the put
    (stream-ordered under NCCL) orders every rank's put before dst reads the
    container.  ``buf`` (dst only): a container_capacity(shard_n)-byte device
    buffer; with ``cache_key`` (same on every rank) its IPC mapping is made
    once and reused.  Returns the buffer on dst (the container occupies its
    first container_total_bytes(header) bytes), None elsewhere."""
    import paper_conf_sc_huangd0lc23_b200 as cz

    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    dev = res.stream.device
    if rank == dst and buf is None:
        buf = torch.empty(container_capacity(shard_n), dtype=torch.uint8, device=dev)
    view = _peer_view(buf, dst, group, cache_key) if world > 1 else buf
    s = torch.cuda.current_stream(dev)
    cz.check(cz.lib().cuszp_container_put(res.stream.data_ptr(), res.header.data_ptr(), world, rank, view.data_ptr(),
                                          1 if rank == dst else 0, s.cuda_stream), "container_put")
    if world > 1:
        if _nccl(group):
            tok = torch.zeros(1, dtype=torch.int32, device=dev)
            dist.all_reduce(tok, group=group)                # after every put on every rank's stream
            if rank != dst and cache_key is None:
                # the put is still queued: keep the IPC mapping alive until it ran
                ev = torch.cuda.Event()
                ev.record(s)
                _inflight.append((view, ev))
                _inflight[:] = [(v, e) for v, e in _inflight if not e.query()]
        else:
            torch.cuda.synchronize(dev)                      # gloo (tests): host-ordered
            dist.barrier(group=group)
    return buf if rank == dst else None


def container_shards(buf: torch.Tensor) -> tuple[dict, list[torch.Tensor]]:
    """Parsed header and the shard streams (views into buf) of a container
    held in a device (or host) uint8 tensor.  Reads the header words only."""
    P = int(buf[16:24].cpu().view(torch.int64).item())
    words = buf[: 8 * (4 + 3 * P)].cpu().view(torch.int64)
    h = parse_container_header(words)
    base = container_header_bytes(P)
    return h, [buf[base + o: base + o + b] for o, b in zip(h["offsets"], h["bytes"])]


def _cuda_decompress(stream: torch.Tensor, n: int, out: torch.Tensor):
    import paper_conf_sc_huangd0lc23_b200 as cz

    return cz.decompress(stream, n, out=out, in_bytes=stream.numel())


def decompress_container(buf: torch.Tensor, out: torch.Tensor | None = None, decompress_fn=None) -> torch.Tensor:
    """Decompress every shard of a container on ONE device into the full
    array (shard p -> its block-aligned slab of ``out``)."""
    decompress_fn = decompress_fn or _cuda_decompress
    h, shards = container_shards(buf)
    if out is None:
        out = torch.empty(h["n_total"], dtype=torch.float32, device=buf.device)
    s0 = 0
    for n_p, sh in zip(h["n"], shards):
        if n_p:
            decompress_fn(sh, n_p, out[s0: s0 + n_p])
        s0 += n_p
    return out


def decompress_sharded(buf: torch.Tensor, group=None, decompress_fn=None) -> torch.Tensor:
    """Distributed decompression: rank p decompresses shard p of the
    container (present on every rank, e.g. from gather_container) into its
    slab; returns the local slab."""
    decompress_fn = decompress_fn or _cuda_decompress
    rank = dist.get_rank(group)
    h, shards = container_shards(buf)
    n_p = h["n"][rank]
    out = torch.empty(n_p, dtype=torch.float32, device=buf.device)
    if n_p:
        decompress_fn(shards[rank], n_p, out)
    return out


def allgather_slabs(local: torch.Tensor, shard_n: list[int], group=None) -> torch.Tensor:
    """Every rank's decompressed slab -> the full array on every rank
    (all-gather of equal, padded slabs, then the padding dropped)."""
    world = dist.get_world_size(group)
    m = max(shard_n) if shard_n else 0
    padded = torch.zeros(m, dtype=local.dtype, device=local.device)
    padded[: local.numel()] = local
    allp = torch.empty(world * m, dtype=local.dtype, device=local.device)
    _allgather(allp, padded, group)
    return torch.cat([allp[p * m: p * m + shard_n[p]] for p in range(world)])


def compress_to_container(x: torch.Tensor, rel: float, P: int) -> torch.Tensor:
    """Single-device construction of a P-shard container of x (REL against
    x's global range): the same bytes P ranks would produce with
    compress_sharded + gather_container."""
    import paper_conf_sc_huangd0lc23_b200 as cz

    n = x.numel()
    mm = cz.value_range(x)
    streams, sizes, shard_n = [], [], []
    for p in range(P):
        s0, s1 = slab_bounds(n, p, P)
        shard_n.append(s1 - s0)
        out, nb = cz.compress_minmax(x[s0:s1], rel, mm)    # an empty slab is a 32-byte stream (R11)
        streams.append(out)
        sizes.append(nb.view(1).to(torch.int64))
    hdr = container_header(shard_n, torch.cat(sizes))
    h = parse_container_header(hdr.cpu())
    base = container_header_bytes(P)
    buf = torch.zeros(container_total_bytes(h), dtype=torch.uint8, device=x.device)
    buf[:base] = _header_bytes_tensor(hdr)
    for p in range(P):
        buf[base + h["offsets"][p]: base + h["offsets"][p] + h["bytes"][p]] = streams[p][: h["bytes"][p]]
    return buf
