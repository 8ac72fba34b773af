"""GPU parity of params.version = 2: the paper's V2 search design (every
position, every window offset, warp-cooperative argmax; PAPER.md:1@13703-14454
§III.B, @17800) behind the paper's "version selection" parameter
(PAPER.md:1@10800 §III).  The stream is defined by the method, not by the
kernel, so version 2 must produce the oracle's bytes exactly, like version 0.
"""
import numpy as np
import pytest

import oracle as O
from paper_conf_cluster_ozsoys11_b200 import datagen
from test_gpu_parity import adversarial_inputs, dev, expand_tokens

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def env():
    import torch
    from paper_conf_cluster_ozsoys11_b200 import build, culzss
    build.build()
    assert culzss.device_count() >= 1
    return torch, culzss


def v2_stream(env, x, **kw):
    torch, culzss = env
    return culzss.compress(dev(torch, x), culzss.Params.make(version=2, **kw)).cpu().numpy().tobytes()


@pytest.mark.parametrize("name", list(adversarial_inputs().keys()))
def test_v2_stream_bit_exact_adversarial(env, name):
    x = adversarial_inputs()[name]
    assert v2_stream(env, x) == O.compress(x)


@pytest.mark.parametrize("n", [1, 2, 3, 4, 127, 128, 129, 4095, 4096, 4097, 8195, (1 << 18) + 13])
@pytest.mark.parametrize("kind", ["english", "random", "runs20", "period20"])
def test_v2_stream_bit_exact_sizes(env, n, kind):
    x = datagen.generate(kind, n, seed=n + 1)
    assert v2_stream(env, x) == O.compress(x)


@pytest.mark.parametrize("kind", datagen.GENERATORS)
def test_v2_stream_bit_exact_generators(env, kind):
    x = datagen.generate(kind, (1 << 19) + 777, seed=6)
    assert v2_stream(env, x) == O.compress(x)


@pytest.mark.parametrize("S,W,F", [(4096, 1, 3), (4096, 16, 18), (4096, 64, 200), (4096, 255, 258),
                                   (4096, 129, 129), (1, 128, 128), (100, 7, 9), (1000, 128, 128),
                                   (129, 3, 5),
                                   # the sweep's instantiations: 16-bit keys (W <= 128, F <= 254) and
                                   # 32-bit keys (F >= 255) at their border, packed chunks
                                   (4096, 128, 254), (4096, 128, 255), (4096, 100, 258), (256, 128, 254),
                                   (512, 64, 258), (4096, 255, 254), (4096, 200, 100), (2048, 255, 128)])
def test_v2_stream_params_variants(env, S, W, F):
    for kind in ("english", "runs20", "period20", "binary"):
        if kind == "binary":
            x = np.random.default_rng(S + W + F).integers(0, 2, 30000, dtype=np.uint8)
        else:
            x = datagen.generate(kind, 30000, seed=S + 2)
        assert v2_stream(env, x, S=S, W=W, F=F) == O.compress(x, S=S, W=W, F=F), kind


@pytest.mark.parametrize("kind", ["english", "csource", "runs20", "period20", "random", "tarmix"])
@pytest.mark.parametrize("W,F", [(128, 128), (255, 255), (5, 7)])
def test_v2_match_search_per_position(env, kind, W, F):
    """Row a2 in the V2 design: (L, D) at every position equals the oracle's
    definitional longest match (smallest d on ties)."""
    torch, culzss = env
    x = datagen.generate(kind, 3 * 4096 + 1234, seed=10)
    L, D = culzss.match_search(dev(torch, x), culzss.Params.make(W=W, F=F, version=2))
    L, D = L.cpu().numpy(), D.cpu().numpy()
    for c in range(4):
        chunk = x[c * 4096:(c + 1) * 4096]
        eL, eD = O.match_all(chunk, W=W, F=F)
        np.testing.assert_array_equal(L[c * 4096:c * 4096 + chunk.size], eL)
        np.testing.assert_array_equal(D[c * 4096:c * 4096 + chunk.size], eD)


@pytest.mark.parametrize("kind", ["english", "csource", "runs20", "random", "tarmix"])
def test_v2_parse_tokens(env, kind):
    """Row a3: the jump parse over the full (L, D) table is the serial greedy parse."""
    torch, culzss = env
    x = datagen.generate(kind, 4 * 4096 + 3000, seed=4)
    tok = culzss.parse_tokens(dev(torch, x), culzss.Params.make(version=2)).cpu().numpy().astype(np.int64)
    tok &= 0xFFFFFFFF
    for c in range(5):
        chunk = x[c * 4096:(c + 1) * 4096]
        np.testing.assert_array_equal(tok[c * 4096:c * 4096 + chunk.size],
                                      expand_tokens(O.tokens_chunk(chunk), chunk.size))


def test_v2_equals_v0_large(env):
    """Both versions produce the same stream on a multi-MiB mixed corpus; the
    oracle checks a spread of its chunks."""
    torch, culzss = env
    x_np = datagen.generate("tarmix", 8 << 20, seed=31)
    x = dev(torch, x_np)
    s0 = culzss.compress(x).cpu().numpy().tobytes()
    s2 = culzss.compress(x, culzss.Params.make(version=2)).cpu().numpy().tobytes()
    assert s0 == s2
    C = x_np.size // 4096
    sizes = np.frombuffer(s2[32:32 + 4 * C], "<u4").astype(np.int64)
    offs = 32 + 4 * C + np.concatenate([[0], np.cumsum(sizes)])
    for c in range(0, C, 97):
        assert s2[offs[c]:offs[c + 1]] == O.compress_chunk(x_np[c * 4096:(c + 1) * 4096]), c


def test_unsupported_versions(env):
    torch, culzss = env
    x = dev(torch, datagen.generate("english", 5000, seed=1))
    for v in (1, 3, 255):
        with pytest.raises(culzss.CulzssError) as e:
            culzss.compress(x, culzss.Params.make(version=v))
        assert e.value.status == culzss.ERR_UNSUPPORTED
