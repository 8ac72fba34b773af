"""GPU checks of the multi-GPU plumbing on one device:
culzss_compress_chunks_async (payload total left in device memory for the
device all-gather) equals culzss_compress_chunks, the strong-scaling chunk
ranges assemble to the one-rank stream, and the device-built rank inputs
equal the host generator's bytes."""
import numpy as np
import pytest

import oracle as O
from paper_conf_cluster_ozsoys11_b200 import datagen, sharding

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def env():
    import torch
    from paper_conf_cluster_ozsoys11_b200 import build, culzss
    build.build()
    return torch, culzss


@pytest.mark.parametrize("kind,n,S", [("csource", 9 * 4096 + 321, 4096), ("runs20", 5 * 4096, 4096),
                                      ("tarmix", 3 * 4096 + 7, 1000), ("random", 4096 * 3, 256)])
def test_compress_chunks_async_matches_sync(env, kind, n, S):
    torch, culzss = env
    x = torch.from_numpy(datagen.generate(kind, n, 3)).cuda()
    p = culzss.Params.make(S=S)
    C = (n + S - 1) // S
    cap = culzss.max_compressed_size(n, p)
    pay_a = torch.zeros(cap, dtype=torch.uint8, device="cuda")
    pay_b = torch.zeros(cap, dtype=torch.uint8, device="cuda")
    sz_a = torch.zeros(C, dtype=torch.int32, device="cuda")
    sz_b = torch.zeros(C, dtype=torch.int32, device="cuda")
    tot = torch.full((1,), -1, dtype=torch.int64, device="cuda")
    culzss.compress_chunks_async(x, pay_a, sz_a, tot, p)
    tb = culzss.compress_chunks(x, pay_b, sz_b, p)
    torch.cuda.synchronize()
    assert int(tot.item()) == tb
    assert torch.equal(sz_a, sz_b) and torch.equal(pay_a[:tb], pay_b[:tb])
    # and the pieces are the oracle's: header + table + payload = its stream
    table = sz_a.cpu().numpy().astype("<u4").tobytes()
    assert (sharding.header(n, S) + table + pay_a[:tb].cpu().numpy().tobytes()
            == O.compress(datagen.generate(kind, n, 3), S=S))


def test_async_rejects_bad_total_pointer(env):
    torch, culzss = env
    x = torch.zeros(4096, dtype=torch.uint8, device="cuda")
    pay = torch.zeros(8192, dtype=torch.uint8, device="cuda")
    sz = torch.zeros(1, dtype=torch.int32, device="cuda")
    with pytest.raises(TypeError):
        culzss.compress_chunks_async(x, pay, sz, torch.zeros(1, dtype=torch.int64))  # host total
    with pytest.raises(ValueError):
        culzss.compress_chunks_async(x, pay, torch.zeros(0, dtype=torch.int32, device="cuda"),
                                     torch.zeros(1, dtype=torch.int64, device="cuda"))


@pytest.mark.parametrize("world", [2, 3, 8])
def test_strong_scaling_ranges_assemble_to_single_stream(env, world):
    """Chunk-aligned rank ranges of one input, each compressed with the async
    call, placed by the all-gathered totals: the assembled stream is the
    one-rank stream byte for byte."""
    torch, culzss = env
    n, S = 37 * 4096 + 999, 4096
    xh = datagen.generate("tarmix", n, 8)
    C = (n + S - 1) // S
    parts, totals = [], []
    for r in range(world):
        b0, b1 = sharding.byte_range(r, world, n, S)
        c = (b1 - b0 + S - 1) // S
        xr = torch.from_numpy(xh[b0:b1].copy()).cuda() if b1 > b0 else torch.empty(0, dtype=torch.uint8, device="cuda")
        pay = torch.zeros(max(1, 2 * (b1 - b0) + 64), dtype=torch.uint8, device="cuda")
        sz = torch.zeros(max(c, 1), dtype=torch.int32, device="cuda")
        tot = torch.zeros(1, dtype=torch.int64, device="cuda")
        culzss.compress_chunks_async(xr, pay, sz, tot)
        parts.append((pay, sz[:c], c))
        totals.append(tot)
    torch.cuda.synchronize()
    tl = [int(t.item()) for t in totals]
    pl = sharding.placements(tl, n, S)
    stream = bytearray(pl[0].stream_bytes)
    stream[:32] = sharding.header(n, S, 128, 128, 3)
    for p, (pay, sz, c) in zip(pl, parts):
        stream[p.table_offset:p.table_offset + 4 * c] = sz.cpu().numpy().astype("<u4").tobytes()
        stream[p.payload_offset:p.payload_offset + p.payload_bytes] = pay[:p.payload_bytes].cpu().numpy().tobytes()
    assert bytes(stream) == O.compress(xh)


@pytest.mark.parametrize("kind,n", [("tarmix", (64 << 20) + (5 << 20) + 17), ("random", 3000001),
                                    ("runs20", 100003)])
def test_generate_range_device_equals_host(env, kind, n):
    torch, culzss = env
    for b0, b1 in [(0, min(n, 9 << 20)), (max(0, n - (7 << 20) - 3), n),
                   ((64 << 20) - 11 if n > (64 << 20) else 11, n - 5)]:
        d = datagen.generate_range_device(kind, n, 5, b0, b1, torch.device("cuda"))
        h = datagen.generate_range(kind, n, 5, b0, b1)
        assert d.numel() == h.size and np.array_equal(d.cpu().numpy(), h), (kind, b0, b1)
