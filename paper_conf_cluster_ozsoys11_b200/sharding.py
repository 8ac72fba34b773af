"""Multi-GPU sharding of the chunked stream.

Chunks are independent units -- "the data blocks that are far enough between
each other can be treated as independent" (PAPER.md:1@30360 §V) and each
chunk decodes from "a list of block compression sizes" (PAPER.md:1@18853
§III.C) -- so the stream shards by contiguous chunk ranges with exactly one
exchange step:

  1. rank r owns chunks [floor(r C / R), floor((r+1) C / R)): a chunk-aligned
     byte slice; only the last rank's last chunk may be partial;
  2. it compresses the slice with culzss_compress_chunks (payload + u32 sizes,
     no header);
  3. an all-gather of the per-rank payload totals T_r (int64) -- over NCCL on
     B200s (NVLink 5 / NVSwitch), gloo in the CPU tests;
  4. the rank's size-table slice belongs at 32 + 4 c0 and its payload at
     32 + 4 C + sum_{r' < r} T_r' -- no further communication;
  5. optionally, the pieces are gathered on one rank (assembly; not part of
     the compression metric).

The paper's own multi-GPU attempt "could not receive any gains"
(PAPER.md:1@36682 §VII).  This module is host logic only; the per-rank
compressor is passed in (the CUDA library on GPUs; tests plug in the oracle).
"""
from __future__ import annotations

import struct
from dataclasses import dataclass
from typing import Callable, List, Sequence, Tuple

HEADER_BYTES = 32


def n_chunks(n: int, S: int) -> int:
    return (n + S - 1) // S


def chunk_range(rank: int, world: int, C: int) -> Tuple[int, int]:
    """Contiguous, balanced chunk range [c0, c1) of `rank`."""
    if not (0 <= rank < world):
        raise ValueError("rank out of range")
    return rank * C // world, (rank + 1) * C // world


def byte_range(rank: int, world: int, n: int, S: int) -> Tuple[int, int]:
    c0, c1 = chunk_range(rank, world, n_chunks(n, S))
    return min(c0 * S, n), min(c1 * S, n)


def header(n: int, S: int = 4096, W: int = 128, F: int = 128, MIN: int = 3) -> bytes:
    """32-byte little-endian stream header (include/culzss.h, reading R12)."""
    return struct.pack("<4sHHIIQHHB3x", b"CLZS", 1, HEADER_BYTES, S, n_chunks(n, S), n, W, F, MIN)


@dataclass
class RankPlacement:
    rank: int
    c0: int
    c1: int
    table_offset: int     # byte offset of this rank's u32 size-table slice
    payload_offset: int   # byte offset of this rank's first payload byte
    payload_bytes: int
    stream_bytes: int     # total length of the assembled stream


def placements(totals: Sequence[int], n: int, S: int) -> List[RankPlacement]:
    """Global placement of every rank's pieces from the all-gathered totals."""
    world = len(totals)
    C = n_chunks(n, S)
    base = HEADER_BYTES + 4 * C
    stream = base + sum(int(t) for t in totals)
    out, run = [], base
    for r in range(world):
        c0, c1 = chunk_range(r, world, C)
        out.append(RankPlacement(r, c0, c1, HEADER_BYTES + 4 * c0, run, int(totals[r]), stream))
        run += int(totals[r])
    return out


def stream_views(sizes: Sequence[int], n: int, S: int, world: int) -> List[RankPlacement]:
    """Sharded decompression of an existing stream:
    from its u32 size table (host copy, C entries), rank r decodes chunks
    [c0, c1) = chunk_range(r, world, C) -- table slice at 32 + 4 c0, payload
    at 32 + 4 C + sum(sizes[:c0]) of length sum(sizes[c0:c1]) -- into output
    bytes [c0 S, min(c1 S, n)).  No exchange is needed: the table is in the
    stream."""
    C = n_chunks(n, S)
    if len(sizes) != C:
        raise ValueError("size table length != ceil(n / S)")
    base = HEADER_BYTES + 4 * C
    prefix = [0]
    for v in sizes:
        prefix.append(prefix[-1] + int(v))
    out = []
    for r in range(world):
        c0, c1 = chunk_range(r, world, C)
        out.append(RankPlacement(r, c0, c1, HEADER_BYTES + 4 * c0, base + prefix[c0],
                                 prefix[c1] - prefix[c0], base + prefix[-1]))
    return out


def exchange_totals(my_total: int, group=None, device=None) -> List[int]:
    """The one collective: all-gather of int64 per-rank payload totals."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    t = torch.tensor([my_total], dtype=torch.int64, device=device)
    out = torch.empty(world, dtype=torch.int64, device=device)
    dist.all_gather_into_tensor(out, t, group=group)
    return [int(v) for v in out.tolist()]


def compress_rank(x_slice, n_total: int, rank: int, world: int, S: int,
                  compress_fn: Callable, group=None, device=None):
    """Compress this rank's slice and place it.  compress_fn(slice) ->
    (payload, sizes_u32) with payload/sizes as tensors or bytes/arrays."""
    payload, sizes = compress_fn(x_slice)
    plen = payload.numel() if hasattr(payload, "numel") else len(payload)
    totals = exchange_totals(plen, group, device)
    return payload, sizes, placements(totals, n_total, S)[rank]


def _global_rank(group, r: int) -> int:
    """torch.distributed point-to-point and gather roots take GLOBAL ranks;
    placements are indexed by the rank within `group`."""
    import torch.distributed as dist
    return r if group is None else dist.get_global_rank(group, r)


def assemble_on_root(payload: bytes, sizes_le: bytes, place: RankPlacement, n_total: int,
                     params: Tuple[int, int, int, int], group=None):
    """Gather every rank's (table slice, payload) on rank 0 and build the
    whole stream there (host bytes; CPU/gloo path).  Returns the stream on
    rank 0, None elsewhere."""
    import torch.distributed as dist
    world = dist.get_world_size(group)
    objs = [None] * world if dist.get_rank(group) == 0 else None
    dist.gather_object((place.rank, sizes_le, payload), objs, dst=_global_rank(group, 0), group=group)
    if dist.get_rank(group) != 0:
        return None
    S, W, F, MIN = params
    buf = bytearray(place.stream_bytes)
    buf[:HEADER_BYTES] = header(n_total, S, W, F, MIN)
    C = n_chunks(n_total, S)
    pos = HEADER_BYTES + 4 * C
    for r, tab, pay in sorted(objs):
        c0, _ = chunk_range(r, world, C)
        buf[HEADER_BYTES + 4 * c0:HEADER_BYTES + 4 * c0 + len(tab)] = tab
        buf[pos:pos + len(pay)] = pay
        pos += len(pay)
    assert pos == place.stream_bytes
    return bytes(buf)


def assemble_on_root_tensors(payload, sizes, totals: Sequence[int], n_total: int,
                             params: Tuple[int, int, int, int], group=None):
    """Assembly with point-to-point transfers of tensors:
    every rank sends its u32 size-table slice and its payload straight into
    their final byte ranges of rank 0's output tensor (NCCL send/recv over
    NVLink for CUDA tensors; gloo for CPU tensors).  `payload` is this rank's
    uint8 payload (exactly its total), `sizes` its int32 table slice,
    `totals` the all-gathered per-rank totals.  Returns the stream tensor on
    rank 0, None elsewhere."""
    import torch
    import torch.distributed as dist
    rank = dist.get_rank(group)
    world = dist.get_world_size(group)
    S, W, F, MIN = params
    pl = placements(totals, n_total, S)
    me = pl[rank]
    tab = (sizes.contiguous().view(torch.uint8) if sizes.numel()
           else torch.empty(0, dtype=torch.uint8, device=sizes.device))
    if rank != 0:
        reqs = []
        if me.c1 > me.c0:
            reqs.append(dist.isend(tab, dst=_global_rank(group, 0), group=group))
        if me.payload_bytes:
            reqs.append(dist.isend(payload.contiguous(), dst=_global_rank(group, 0), group=group))
        for r in reqs:
            r.wait()
        return None
    out = torch.empty(me.stream_bytes, dtype=torch.uint8, device=payload.device)
    out[:HEADER_BYTES] = torch.frombuffer(bytearray(header(n_total, S, W, F, MIN)), dtype=torch.uint8).to(out.device)
    reqs = []
    for p in pl:
        tsl = out[p.table_offset:p.table_offset + 4 * (p.c1 - p.c0)]
        psl = out[p.payload_offset:p.payload_offset + p.payload_bytes]
        if p.rank == 0:
            tsl.copy_(tab)
            psl.copy_(payload)
            continue
        if p.c1 > p.c0:
            reqs.append(dist.irecv(tsl, src=_global_rank(group, p.rank), group=group))
        if p.payload_bytes:
            reqs.append(dist.irecv(psl, src=_global_rank(group, p.rank), group=group))
    for r in reqs:
        r.wait()
    return out

