"""Chunks above 4 KiB ("the decision on the length of the
blocks is a configuration parameter", PAPER.md:1@30360 §V): S in (4096,
65536] is compressed in 4096-position tiles (window history before each tile,
lookahead after it, the greedy path and the bit offset carried across tiles)
and decoded by the serial-token warp decoder.  Byte-exact against the oracle,
exact round trips, per-position (L, D) and tokens across tile borders."""
import os

import numpy as np
import pytest

import oracle as O
from paper_conf_cluster_ozsoys11_b200 import datagen

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def env():
    import torch
    from paper_conf_cluster_ozsoys11_b200 import build, culzss
    build.build()
    return torch, culzss


def dev(torch, a):
    a = np.ascontiguousarray(a, dtype=np.uint8)
    return torch.from_numpy(a.copy()).cuda() if a.size else torch.empty(0, dtype=torch.uint8, device="cuda")


def inputs(n):
    rng = np.random.default_rng(64)
    out = {k: datagen.generate(k, n, seed=5) for k in ("csource", "runs20", "tarmix", "random", "english")}
    out["period300"] = np.tile(rng.integers(0, 256, 300, dtype=np.uint8), n // 300 + 1)[:n]
    out["period64"] = np.tile(rng.integers(0, 256, 64, dtype=np.uint8), n // 64 + 1)[:n]
    out["zeros"] = np.zeros(n, np.uint8)
    return out


@pytest.mark.parametrize("S", [4097, 5000, 8192, 16384, 65536])
@pytest.mark.parametrize("W,F", [(128, 128), (256, 256), (64, 258), (16, 3)])
def test_large_chunk_streams(env, S, W, F):
    torch, culzss = env
    p = culzss.Params.make(S=S, W=W, F=F)
    n = 2 * S + 3333  # two full chunks and a partial one
    for name, x in inputs(n).items():
        s = culzss.compress(dev(torch, x), p)
        assert s.cpu().numpy().tobytes() == O.compress(x, S=S, W=W, F=F), (name, S, W, F)
        assert culzss.decompress(s).cpu().numpy().tobytes() == x.tobytes(), (name, S, W, F)


@pytest.mark.parametrize("tx", ["1000000000", "0"])
def test_large_chunks_both_walk_machines(env, tx):
    torch, culzss = env
    old = os.environ.get("CULZSS_WALK_TOKEN_SWITCH")
    os.environ["CULZSS_WALK_TOKEN_SWITCH"] = tx
    try:
        p = culzss.Params.make(S=32768)
        for name, x in inputs(3 * 32768 + 77).items():
            got = culzss.compress(dev(torch, x), p).cpu().numpy().tobytes()
            assert got == O.compress(x, S=32768), (name, tx)
    finally:
        if old is None:
            os.environ.pop("CULZSS_WALK_TOKEN_SWITCH", None)
        else:
            os.environ["CULZSS_WALK_TOKEN_SWITCH"] = old


def test_large_chunk_match_search_and_tokens(env):
    """Rows a2 / a3 across tile borders: (L, D) at every position and the
    greedy path's tokens, chunk by chunk."""
    torch, culzss = env
    S = 12000
    p = culzss.Params.make(S=S)
    for name, x in inputs(S + 4321).items():
        L, D = culzss.match_search(dev(torch, x), p)
        L, D = L.cpu().numpy(), D.cpu().numpy()
        tok = culzss.parse_tokens(dev(torch, x), p).cpu().numpy()
        for c in range((x.size + S - 1) // S):
            chunk = x[c * S:(c + 1) * S]
            eL, eD = O.match_all(chunk)
            np.testing.assert_array_equal(L[c * S:c * S + chunk.size], eL, err_msg=name)
            np.testing.assert_array_equal(D[c * S:c * S + chunk.size], eD, err_msg=name)
            exp = np.zeros(chunk.size, np.int64)
            pos = 0
            for t in O.tokens_chunk(chunk):
                if t[0] == "L":
                    exp[pos] = 1
                    pos += 1
                else:
                    exp[pos] = (t[2] << 16) | t[1]
                    pos += t[2]
            np.testing.assert_array_equal(tok[c * S:c * S + chunk.size].astype(np.int64), exp, err_msg=name)


def test_large_chunks_host_api_and_sharding(env):
    torch, culzss = env
    S = 16384
    p = culzss.Params.make(S=S)
    x = datagen.generate("tarmix", 40 * S + 999, seed=8)
    expect = O.compress(x, S=S)
    hin = torch.from_numpy(x.copy()).pin_memory()
    hout = torch.empty(culzss.max_compressed_size(x.size, p), dtype=torch.uint8).pin_memory()
    on = culzss.compress_host_ptr(hin.data_ptr(), x.size, hout.data_ptr(), hout.numel(), p)
    assert hout[:on].numpy().tobytes() == expect
    hdec = torch.empty(x.size, dtype=torch.uint8).pin_memory()
    culzss.decompress_host_ptr(hout.data_ptr(), on, hdec.data_ptr(), x.size)
    assert torch.equal(hdec, hin)
    # sharding primitives on chunk-aligned slices
    half = 20 * S
    for b0, b1 in ((0, half), (half, x.size)):
        xs = dev(torch, x[b0:b1])
        C = (b1 - b0 + S - 1) // S
        pay = torch.empty(culzss.max_compressed_size(b1 - b0, p), dtype=torch.uint8, device="cuda")
        sz = torch.empty(C, dtype=torch.int32, device="cuda")
        t = culzss.compress_chunks(xs, pay, sz, p)
        y = culzss.decompress_chunks(pay[:t], sz, b1 - b0, params=p)
        assert torch.equal(y, xs)


def test_large_chunk_limits_and_corrupt(env):
    torch, culzss = env
    x = dev(torch, datagen.generate("english", 70000, seed=1))
    for kw in (dict(S=65537), dict(S=8192, version=2)):
        with pytest.raises(culzss.CulzssError) as e:
            culzss.compress(x, culzss.Params.make(**kw))
        assert e.value.status == culzss.ERR_UNSUPPORTED, kw
    # the serial-token decoder rejects corrupt large-chunk streams like the oracle
    base = bytearray(O.compress(datagen.generate("csource", 30000, seed=3), S=8192))
    rng = np.random.default_rng(9)
    for _ in range(60):
        s = bytearray(base)
        for _ in range(int(rng.integers(1, 4))):
            i = int(rng.integers(32, len(s)))
            s[i] ^= int(rng.integers(1, 256))
        ost, oy = O.decompress_status(bytes(s))
        gst, gy = culzss.decompress_status(dev(torch, np.frombuffer(bytes(s), np.uint8)))
        if ost == O.OK:
            assert gst == culzss.OK and gy.cpu().numpy().tobytes() == oy
        else:
            assert gst in (culzss.ERR_CORRUPT, culzss.ERR_UNSUPPORTED)
