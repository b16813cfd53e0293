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
(same eb_abs, block-aligned slabs).  Moving the compressed payloads into
one concatenated buffer is SURVEY 8(f) NEXT rank 1; ``assemble_container``
does it for a gathered set of shard streams.
"""
from __future__ import annotations

import struct
from dataclasses import dataclass

import torch
import torch.distributed as dist

BLOCK = 32
CONTAINER_MAGIC = 0x544E4F43505A5343  # "CSZPCONT" little-endian
CONTAINER_VERSION = 1


def slab_bounds(n_total: int, rank: int, world: int) -> tuple[int, int]:
    """Element range [start, end) of rank's block-aligned slab."""
    nb = (n_total + BLOCK - 1) // BLOCK
    b0 = (rank * nb) // world
    b1 = ((rank + 1) * nb) // world
    return min(b0 * BLOCK, n_total), min(b1 * BLOCK, n_total)


def _allgather(dst: torch.Tensor, src: torch.Tensor, group) -> torch.Tensor:
    if dist.get_backend(group) == "nccl":
        dist.all_gather_into_tensor(dst, src, group=group)
    else:
        world = dist.get_world_size(group)
        parts = list(dst.view(world, -1).unbind(0))
        dist.all_gather(parts, src, group=group)
        dst.copy_(torch.stack(parts).view(-1))
    return dst


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
    offs = torch.cumsum(sizes_all, 0) - sizes_all
    head = torch.tensor([CONTAINER_MAGIC - (1 << 64) if CONTAINER_MAGIC >= 1 << 63 else CONTAINER_MAGIC,
                         CONTAINER_VERSION, P, int(sum(shard_n))], dtype=torch.int64, device=dev)
    return torch.cat([head, n, sizes_all.to(torch.int64), offs])


def container_header_bytes(P: int) -> int:
    return 8 * (4 + 3 * P)


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
    body = bytearray(sum(h["bytes"]))
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
