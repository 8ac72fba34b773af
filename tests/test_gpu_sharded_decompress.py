"""GPU parity of sharded decompression: every rank
decodes its own contiguous chunk range with culzss_decompress_chunks -- from a
whole stream through sharding.stream_views, or straight from its
culzss_compress_chunks outputs -- and the concatenated slices equal the input.
Chunks decode independently from the size list (PAPER.md:1@18329-19204)."""
import numpy as np
import pytest

import oracle as O
from paper_conf_cluster_ozsoys11_b200 import datagen, sharding
from test_gpu_parity import dev

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def env():
    import torch
    from paper_conf_cluster_ozsoys11_b200 import build, culzss
    build.build()
    assert culzss.device_count() >= 1
    return torch, culzss


@pytest.mark.parametrize("kind,n", [("csource", 37 * 4096 + 1111), ("random", 16 * 4096),
                                    ("runs20", 5 * 4096 + 3), ("tarmix", 3 * (1 << 20) + 17)])
@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
def test_stream_views_decode(env, kind, n, world):
    torch, culzss = env
    x_np = datagen.generate(kind, n, seed=world + 3)
    s_np = np.frombuffer(O.compress(x_np), np.uint8)  # the oracle's stream
    s = dev(torch, s_np)
    S = 4096
    C = (n + S - 1) // S
    sizes = np.frombuffer(s_np.tobytes(), "<u4", count=C, offset=32)
    parts = []
    for v in sharding.stream_views(sizes.tolist(), n, S, world):
        b0, b1 = min(v.c0 * S, n), min(v.c1 * S, n)
        pay = s[v.payload_offset:v.payload_offset + v.payload_bytes]
        tab = s[v.table_offset:v.table_offset + 4 * (v.c1 - v.c0)].view(torch.int32)
        if b1 == b0:
            continue
        parts.append(culzss.decompress_chunks(pay, tab, b1 - b0).cpu().numpy())
    assert np.concatenate(parts).tobytes() == x_np.tobytes()


@pytest.mark.parametrize("world", [2, 4, 8])
def test_decode_compress_chunks_outputs(env, world):
    """The multi-GPU round trip without assembling a stream: each rank's
    payload + sizes from compress_chunks decode back to its slice."""
    torch, culzss = env
    n, S = 53 * 4096 + 999, 4096
    x = dev(torch, datagen.generate("tarmix", n, seed=44))
    C = (n + S - 1) // S
    for r in range(world):
        c0, c1 = sharding.chunk_range(r, world, C)
        sl = x[c0 * S:min(c1 * S, n)]
        pay = torch.empty(max(1, culzss.max_compressed_size(sl.numel())), dtype=torch.uint8, device="cuda")
        sizes = torch.zeros(max(1, c1 - c0), dtype=torch.int32, device="cuda")
        t = culzss.compress_chunks(sl, pay, sizes)
        y = culzss.decompress_chunks(pay[:t], sizes[:c1 - c0], sl.numel())
        assert torch.equal(y, sl), r


@pytest.mark.parametrize("S,W,F", [(1000, 64, 200), (100, 7, 9), (4096, 255, 258)])
def test_decode_chunks_params(env, S, W, F):
    torch, culzss = env
    x_np = datagen.generate("english", 20011, seed=S)
    s_np = np.frombuffer(O.compress(x_np, S=S, W=W, F=F), np.uint8)
    C = (x_np.size + S - 1) // S
    s = dev(torch, s_np)
    p = culzss.Params.make(S=S, W=W, F=F)
    sizes = np.frombuffer(s_np.tobytes(), "<u4", count=C, offset=32).tolist()
    out = []
    for v in sharding.stream_views(sizes, x_np.size, S, 3):
        b0, b1 = v.c0 * S, min(v.c1 * S, x_np.size)
        tab = s[v.table_offset:v.table_offset + 4 * (v.c1 - v.c0)].view(torch.int32)
        out.append(culzss.decompress_chunks(s[v.payload_offset:v.payload_offset + v.payload_bytes], tab,
                                            b1 - b0, params=p).cpu().numpy())
    assert np.concatenate(out).tobytes() == x_np.tobytes()


def test_decode_chunks_rejects(env):
    torch, culzss = env
    x_np = datagen.generate("csource", 5 * 4096, seed=1)
    s_np = np.frombuffer(O.compress(x_np), np.uint8)
    s = dev(torch, s_np)
    C = 5
    pay, tab = s[32 + 4 * C:], s[32:32 + 4 * C].view(torch.int32)
    assert torch.equal(culzss.decompress_chunks(pay, tab, x_np.size).cpu(), torch.from_numpy(x_np))
    st, _ = culzss.decompress_chunks_status(pay[:-1], tab, x_np.size)   # sizes sum != payload_n
    assert st == culzss.ERR_CORRUPT
    st, _ = culzss.decompress_chunks_status(pay, tab, x_np.size - 4096 + 1)  # wrong chunk count / lengths
    assert st == culzss.ERR_CORRUPT
    st, _ = culzss.decompress_chunks_status(pay, tab, 0)
    assert st == culzss.ERR_CORRUPT
    bad = pay.clone()
    bad[0] ^= 0xFF
    st, _ = culzss.decompress_chunks_status(bad, tab, x_np.size)
    ost, _ = O.decompress_status(bytes(s_np[:32 + 4 * C]) + bad.cpu().numpy().tobytes())
    assert (st == culzss.OK) == (ost == O.OK)
