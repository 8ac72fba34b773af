"""Multi-process (gloo, CPU) test of the sharding + offset logic of SURVEY
§8(e): R ranks compress contiguous chunk ranges (the oracle is the per-rank
compressor here -- no GPU), all-gather their totals, and the stream
assembled on rank 0 is byte-identical to the single-process stream."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

from paper_conf_cluster_ozsoys11_b200 import datagen, sharding


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, kind, n, S, out_q):
    import torch.distributed as dist
    import oracle as O
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        x = datagen.generate(kind, n, seed=17)  # every rank derives the same input
        b0, b1 = sharding.byte_range(rank, world, n, S)
        C = sharding.n_chunks(n, S)
        c0, c1 = sharding.chunk_range(rank, world, C)

        def compress_fn(sl):
            if c1 == c0:
                return b"", np.zeros(0, np.uint32)
            pay, sizes = O.compress_range(x, c0, c1, S=S)
            return pay, sizes

        pay, sizes, place = sharding.compress_rank(x[b0:b1], n, rank, world, S, compress_fn)
        assert (place.c0, place.c1) == (c0, c1)
        stream = sharding.assemble_on_root(pay, np.asarray(sizes, "<u4").tobytes(), place, n,
                                           (S, 128, 128, 3))
        if rank == 0:
            out_q.put(stream)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,kind,n,S", [(2, "csource", 37 * 4096 + 1111, 4096),
                                            (4, "english", 9 * 4096, 4096),
                                            (2, "runs20", 3 * 4096 + 5, 4096),
                                            (3, "tarmix", 5000, 1000),
                                            (4, "random", 2 * 4096, 4096)])  # ranks with no chunks
def test_sharded_stream_equals_single(world, kind, n, S):
    import oracle as O
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, kind, n, S, q)) for r in range(world)]
    for p in procs:
        p.start()
    stream = q.get(timeout=120)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    x = datagen.generate(kind, n, seed=17)
    assert stream == O.compress(x, S=S)


def test_placements_closed_form():
    n, S = 10 * 4096 + 7, 4096
    totals = [100, 0, 250, 13]
    pl = sharding.placements(totals, n, S)
    C = 11
    assert [(p.c0, p.c1) for p in pl] == [(0, 2), (2, 5), (5, 8), (8, 11)]
    assert pl[0].payload_offset == 32 + 4 * C
    assert pl[2].payload_offset == 32 + 4 * C + 100
    assert pl[3].table_offset == 32 + 4 * 8
    assert all(p.stream_bytes == 32 + 4 * C + 363 for p in pl)
    assert sharding.header(n)[:4] == b"CLZS" and len(sharding.header(n)) == 32


def _dec_worker(rank, world, port, kind, n, S, out_q):
    """Sharded decompression on CPU: every rank decodes its own chunk range of
    the stream (a header + its table slice + its payload slice is itself a
    valid stream of the slice), rank 0 gathers the slices."""
    import torch.distributed as dist
    import oracle as O
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        x = datagen.generate(kind, n, seed=23)
        stream = O.compress(x, S=S)
        C = sharding.n_chunks(n, S)
        sizes = np.frombuffer(stream, "<u4", count=C, offset=32).tolist()
        v = sharding.stream_views(sizes, n, S, world)[rank]
        b0, b1 = sharding.byte_range(rank, world, n, S)
        mini = (sharding.header(b1 - b0, S) + stream[v.table_offset:v.table_offset + 4 * (v.c1 - v.c0)]
                + stream[v.payload_offset:v.payload_offset + v.payload_bytes])
        part = O.decompress(mini)
        objs = [None] * world if rank == 0 else None
        dist.gather_object((rank, part), objs, dst=0)
        if rank == 0:
            out_q.put(b"".join(p for _, p in sorted(objs)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,kind,n,S", [(2, "csource", 37 * 4096 + 1111, 4096),
                                            (3, "tarmix", 5000, 1000),
                                            (4, "runs20", 2 * 4096 + 7, 4096)])
def test_sharded_decompress_gloo(world, kind, n, S):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_dec_worker, args=(r, world, port, kind, n, S, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = q.get(timeout=120)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert out == datagen.generate(kind, n, seed=23).tobytes()


def test_stream_views_closed_form():
    n, S = 10 * 4096 + 7, 4096
    sizes = [10, 20, 30, 40, 50, 60, 70, 80, 90, 100, 5]
    v = sharding.stream_views(sizes, n, S, 4)
    C = 11
    assert [(p.c0, p.c1) for p in v] == [(0, 2), (2, 5), (5, 8), (8, 11)]
    assert [p.payload_offset for p in v] == [32 + 4 * C + o for o in (0, 30, 150, 360)]
    assert [p.payload_bytes for p in v] == [30, 120, 210, 195]
    assert all(p.stream_bytes == 32 + 4 * C + sum(sizes) for p in v)
    with pytest.raises(ValueError):
        sharding.stream_views(sizes[:-1], n, S, 2)


def _asm_worker(rank, world, port, kind, n, S, out_q):
    """Tensor assembly on rank 0 through point-to-point transfers (gloo here;
    NCCL send/recv on B200s)."""
    import torch
    import torch.distributed as dist
    import oracle as O
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        x = datagen.generate(kind, n, seed=31)
        C = sharding.n_chunks(n, S)
        c0, c1 = sharding.chunk_range(rank, world, C)
        if c1 > c0:
            pay, sizes = O.compress_range(x, c0, c1, S=S)
        else:
            pay, sizes = b"", np.zeros(0, np.uint32)
        pay_t = torch.frombuffer(bytearray(pay), dtype=torch.uint8) if pay else torch.empty(0, dtype=torch.uint8)
        sizes_t = torch.from_numpy(np.asarray(sizes, dtype=np.uint32).view(np.int32).copy())
        totals = sharding.exchange_totals(len(pay))
        out = sharding.assemble_on_root_tensors(pay_t, sizes_t, totals, n, (S, 128, 128, 3))
        if rank == 0:
            out_q.put(out.numpy().tobytes())
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,kind,n,S", [(2, "csource", 37 * 4096 + 1111, 4096),
                                            (3, "tarmix", 5000, 1000),
                                            (4, "random", 2 * 4096, 4096)])  # ranks with no chunks
def test_tensor_assembly_gloo(world, kind, n, S):
    import oracle as O
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_asm_worker, args=(r, world, port, kind, n, S, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = q.get(timeout=120)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert out == O.compress(datagen.generate(kind, n, seed=31), S=S)
