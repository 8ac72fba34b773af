"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bit-exact for every byte of the stream (integer work), per-position (L, D)
for the match search, per-position tokens for the greedy parse, and exact
round trips for the decoder.  Inputs come from the seeded generators; no
expected value comes from the CUDA path.
"""
import struct

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
    assert culzss.device_count() >= 1
    return torch, culzss


def dev(torch, a):
    a = np.ascontiguousarray(a, dtype=np.uint8)
    return torch.from_numpy(a.copy()).cuda() if a.size else torch.empty(0, dtype=torch.uint8, device="cuda")


def gpu_stream(env, x, **kw):
    torch, culzss = env
    p = culzss.Params.make(**kw) if kw else None
    return culzss.compress(dev(torch, x), p).cpu().numpy().tobytes()


def adversarial_inputs():
    rng = np.random.default_rng(123)
    cases = {
        "empty": np.zeros(0, np.uint8),
        "one": np.array([7], np.uint8),
        "zeros_64k": np.zeros(65536, np.uint8),
        "ff_5000": np.full(5000, 255, np.uint8),
        "ramp": (np.arange(10000) & 0xFF).astype(np.uint8),
        "random_100k": rng.integers(0, 256, 100000, dtype=np.uint8),
        "binary_30k": rng.integers(0, 2, 30000, dtype=np.uint8),
        "ternary_30k": rng.integers(0, 3, 30000, dtype=np.uint8),
        "figure1": np.frombuffer(b"I meant what I said\nand I said what I meant\n\nFrom there to here\n"
                                 b"from here to there\nI said what I meant", np.uint8),
    }
    for d in list(range(1, 20)) + [31, 32, 33, 63, 64, 65, 100, 126, 127, 128, 129, 130, 200, 255, 256]:
        base = rng.integers(0, 256, d, dtype=np.uint8)
        cases[f"period{d}"] = np.tile(base, 9000 // d + 1)[:9000 + d]
    runs = np.repeat(rng.integers(0, 4, 3000, dtype=np.uint8), rng.integers(1, 300, 3000))
    cases["runs_mixed"] = runs[:200000]
    return cases


@pytest.mark.parametrize("name", list(adversarial_inputs().keys()))
def test_stream_bit_exact_adversarial(env, name):
    x = adversarial_inputs()[name]
    assert gpu_stream(env, x) == O.compress(x)


@pytest.mark.parametrize("n", [1, 2, 3, 4, 5, 127, 128, 129, 4093, 4095, 4096, 4097, 8191, 8192, 8195,
                               (1 << 20) + 13])
@pytest.mark.parametrize("kind", ["english", "random", "runs20"])
def test_stream_bit_exact_sizes(env, n, kind):
    x = datagen.generate(kind, n, seed=n)
    assert gpu_stream(env, x) == O.compress(x)


@pytest.mark.parametrize("kind", datagen.GENERATORS)
def test_stream_bit_exact_generators(env, kind):
    x = datagen.generate(kind, (1 << 20) + 777, seed=5)
    assert gpu_stream(env, x) == O.compress(x)


def test_config1_english_64k_bit_exact(env):
    """BASELINE configs[0]: 64 KB English-like text, paper params, full stream."""
    for kind in ("english", "wordlist"):
        x = datagen.generate(kind, 64 << 10, seed=1)
        assert gpu_stream(env, x) == O.compress(x)


@pytest.mark.parametrize("S,W,F", [(4096, 1, 3), (4096, 2, 4), (4096, 16, 18), (4096, 64, 200),
                                   (4096, 255, 258), (4096, 128, 129), (1, 128, 128), (2, 128, 128),
                                   (100, 7, 9), (128, 128, 128), (1000, 128, 128), (4000, 100, 250),
                                   (129, 3, 5)])
def test_stream_params_variants(env, S, W, F):
    for kind in ("english", "runs20", "period20", "binary"):
        if kind == "binary":
            x = np.random.default_rng(S + W + F).integers(0, 2, 50000, dtype=np.uint8)
        else:
            x = datagen.generate(kind, 50000, seed=S)
        assert gpu_stream(env, x, S=S, W=W, F=F) == O.compress(x, S=S, W=W, F=F), kind


@pytest.mark.parametrize("S,W,F", [(4096, 1, 3), (4096, 255, 258), (4096, 16, 18), (1, 128, 128),
                                   (100, 7, 9), (129, 3, 5), (1000, 128, 128), (4000, 100, 250)])
def test_decoder_params_variants(env, S, W, F):
    """Row a6 on oracle streams of every parameter shape (lane spans vs chunk size)."""
    torch, culzss = env
    for kind in ("english", "runs20", "period20", "random"):
        x = datagen.generate(kind, 30011, seed=S + 1)
        s = O.compress(x, S=S, W=W, F=F)
        y = culzss.decompress(dev(torch, np.frombuffer(s, np.uint8)))
        assert y.cpu().numpy().tobytes() == x.tobytes(), kind


def test_decoder_unaligned_input_and_output(env):
    torch, culzss = env
    x = datagen.generate("csource", 70001, seed=9)
    s = np.frombuffer(O.compress(x), np.uint8)
    for ioff in (0, 1, 3, 7, 13):
        buf = torch.zeros(s.size + 32, dtype=torch.uint8, device="cuda")
        buf[ioff:ioff + s.size] = dev(torch, s)
        for oo in (0, 1, 2, 5):
            out = torch.zeros(x.size + 8, dtype=torch.uint8, device="cuda")
            culzss.decompress(buf[ioff:ioff + s.size], out[oo:oo + x.size])
            assert out[oo:oo + x.size].cpu().numpy().tobytes() == x.tobytes(), (ioff, oo)


@pytest.mark.parametrize("kind", ["english", "csource", "runs20", "period20", "random", "tarmix"])
def test_match_search_per_position(env, kind):
    """Row a2: (L, D) at every position of several chunks + a ragged tail."""
    torch, culzss = env
    x = datagen.generate(kind, 5 * 4096 + 1234, seed=9)
    L, D = culzss.match_search(dev(torch, x))
    L, D = L.cpu().numpy(), D.cpu().numpy()
    for c in range(6):
        chunk = x[c * 4096:(c + 1) * 4096]
        eL, eD = O.match_all(chunk)
        np.testing.assert_array_equal(L[c * 4096:c * 4096 + chunk.size], eL)
        np.testing.assert_array_equal(D[c * 4096:c * 4096 + chunk.size], eD)


@pytest.mark.parametrize("W,F", [(128, 128), (5, 7), (255, 255), (1, 3)])
def test_match_search_adversarial(env, W, F):
    torch, culzss = env
    for name, x in adversarial_inputs().items():
        x = x[:3 * 4096 + 5]
        if x.size == 0:
            continue
        L, D = culzss.match_search(dev(torch, x), culzss.Params.make(W=W, F=F))
        L, D = L.cpu().numpy(), D.cpu().numpy()
        for c in range((x.size + 4095) // 4096):
            chunk = x[c * 4096:(c + 1) * 4096]
            eL, eD = O.match_all(chunk, W=W, F=F)
            np.testing.assert_array_equal(L[c * 4096:c * 4096 + chunk.size], eL, err_msg=name)
            np.testing.assert_array_equal(D[c * 4096:c * 4096 + chunk.size], eD, err_msg=name)


def expand_tokens(toks, m):
    out = np.zeros(m, np.int64)
    p = 0
    for t in toks:
        if t[0] == "L":
            out[p] = 1
            p += 1
        else:
            out[p] = (t[2] << 16) | t[1]
            p += t[2]
    assert p == m
    return out


@pytest.mark.parametrize("kind", ["english", "csource", "runs20", "period20", "random", "tarmix",
                                  "wordlist"])
def test_parse_tokens(env, kind):
    """Row a3: the speculative segment-parallel parse equals the serial greedy parse."""
    torch, culzss = env
    x = datagen.generate(kind, 4 * 4096 + 3000, seed=3)
    tok = culzss.parse_tokens(dev(torch, x)).cpu().numpy().astype(np.int64) & 0xFFFFFFFF
    for c in range(5):
        chunk = x[c * 4096:(c + 1) * 4096]
        np.testing.assert_array_equal(tok[c * 4096:c * 4096 + chunk.size],
                                      expand_tokens(O.tokens_chunk(chunk), chunk.size))


@pytest.mark.parametrize("kind", datagen.GENERATORS)
def test_roundtrip_device(env, kind):
    torch, culzss = env
    x = dev(torch, datagen.generate(kind, 3 * (1 << 20) + 99, seed=2))
    s = culzss.compress(x)
    y = culzss.decompress(s)
    assert torch.equal(x, y)


def test_gpu_decoder_reads_oracle_streams(env):
    torch, culzss = env
    for name, x in adversarial_inputs().items():
        s = O.compress(x)
        y = culzss.decompress(dev(torch, np.frombuffer(s, np.uint8)))
        assert y.cpu().numpy().tobytes() == x.tobytes(), name


def test_gpu_decoder_rejects_corrupt(env):
    """Same malformations as the oracle pins (tests/test_oracle_pins.py)."""
    torch, culzss = env
    import test_oracle_pins as P
    for _, s in P.CORRUPT_STREAMS:
        st, _ = culzss.decompress_status(dev(torch, np.frombuffer(s, np.uint8)))
        assert st == culzss.ERR_CORRUPT, s
    # random mutations: CORRUPT or same answer as the oracle decoder
    rng = np.random.default_rng(5)
    x = datagen.generate("english", 20000, seed=4)
    base = bytearray(O.compress(x))
    for _ in range(200):
        s = bytearray(base)
        for _ in range(int(rng.integers(1, 4))):
            i = int(rng.integers(0, len(s)))
            s[i] ^= int(rng.integers(1, 256))
        ost, oout = O.decompress_status(bytes(s))
        gst, gout = culzss.decompress_status(dev(torch, np.frombuffer(bytes(s), np.uint8)))
        if ost == O.OK:
            assert gst == culzss.OK and gout.cpu().numpy().tobytes() == oout
        else:
            assert gst in (culzss.ERR_CORRUPT, culzss.ERR_UNSUPPORTED)


def test_gpu_decoder_incompressible_chunks(env):
    """Chunks of size ceil(9m/8) (PAPER.md:1@6743 §II.A.2 decoding; such a chunk
    holds only literals in a valid stream) skip the walk and decode in the literal kernel, which
    must check every flag bit and the pad bits exactly as the oracle decoder does."""
    torch, culzss = env
    S = 4096
    for n in (3 * S + 1001, 2 * S, 17, 5 * S + 8):
        x = datagen.generate("random", n, seed=n)
        s = O.compress(x)
        C = (n + S - 1) // S
        sizes = np.frombuffer(s[32:32 + 4 * C], "<u4")
        ms = [min(S, n - c * S) for c in range(C)]
        assert all(int(sz) == (9 * m + 7) // 8 for sz, m in zip(sizes, ms)), "random chunks are all-literal"
        y = culzss.decompress(dev(torch, np.frombuffer(s, np.uint8)))
        assert y.cpu().numpy().tobytes() == x.tobytes(), n
        base = 32 + 4 * C
        off = base + int(sizes[:C - 1].sum())  # the last chunk's payload
        m = ms[-1]
        for j in (0, 1, m // 2, m - 1):  # a literal's flag bit set: the oracle and the GPU reject
            b = bytearray(s)
            bit = 9 * j
            b[off + bit // 8] |= 0x80 >> (bit % 8)
            assert O.decompress_status(bytes(b))[0] == O.ERR_CORRUPT
            st, _ = culzss.decompress_status(dev(torch, np.frombuffer(bytes(b), np.uint8)))
            assert st == culzss.ERR_CORRUPT, (n, j)
        pad = 8 * int(sizes[-1]) - 9 * m
        if pad:  # a nonzero pad bit
            b = bytearray(s)
            b[off + int(sizes[-1]) - 1] |= 1
            assert O.decompress_status(bytes(b))[0] == O.ERR_CORRUPT
            st, _ = culzss.decompress_status(dev(torch, np.frombuffer(bytes(b), np.uint8)))
            assert st == culzss.ERR_CORRUPT, n


def test_gpu_decoder_mutations_mixed(env):
    """Random mutations of a stream mixing incompressible, text and run chunks (the classify /
    literal / walk / decode kernels all see malformed input): CORRUPT, or the oracle's output."""
    torch, culzss = env
    rng = np.random.default_rng(11)
    x = np.concatenate([datagen.generate("random", 2 * 4096 + 300, seed=1), datagen.generate("english", 9000, seed=2),
                        datagen.generate("runs20", 5000, seed=3), datagen.generate("random", 4096, seed=4)])
    base = bytearray(O.compress(x))
    for _ in range(200):
        s = bytearray(base)
        for _ in range(int(rng.integers(1, 4))):
            i = int(rng.integers(32, len(s)))
            s[i] ^= int(rng.integers(1, 256))
        ost, oout = O.decompress_status(bytes(s))
        gst, gout = culzss.decompress_status(dev(torch, np.frombuffer(bytes(s), np.uint8)))
        if ost == O.OK:
            assert gst == culzss.OK and gout.cpu().numpy().tobytes() == oout
        else:
            assert gst in (culzss.ERR_CORRUPT, culzss.ERR_UNSUPPORTED)


def test_unaligned_input_and_output(env):
    torch, culzss = env
    x = datagen.generate("csource", 100000, seed=8)
    buf = dev(torch, x)
    out = torch.zeros(culzss.max_compressed_size(90000) + 16, dtype=torch.uint8, device="cuda")
    for off in (1, 2, 3, 5, 15):
        expect = O.compress(x[off:off + 90000])
        for oo in (0, 1, 3):
            n = culzss.compress_into(buf[off:off + 90000], out[oo:])
            assert out[oo:oo + n].cpu().numpy().tobytes() == expect, (off, oo)


def test_buffer_too_small_and_invalid(env):
    torch, culzss = env
    x = dev(torch, datagen.generate("english", 10000, seed=1))
    out = torch.empty(100, dtype=torch.uint8, device="cuda")
    with pytest.raises(culzss.CulzssError) as e:
        culzss.compress_into(x, out)
    assert e.value.status == culzss.ERR_BUFFER_TOO_SMALL
    with pytest.raises(culzss.CulzssError) as e:
        culzss.compress(x, culzss.Params.make(MIN=2))
    assert e.value.status == culzss.ERR_INVALID_ARG
    with pytest.raises(culzss.CulzssError) as e:
        culzss.compress(x, culzss.Params.make(S=65537))  # S <= 64 KiB (tiled above 4 KiB)
    assert e.value.status == culzss.ERR_UNSUPPORTED


def test_compress_host_matches(env):
    torch, culzss = env
    x = datagen.generate("tarmix", 300000, seed=6)
    assert culzss.compress_host(x).tobytes() == O.compress(x)
    assert culzss.compress_host(x[:0]).tobytes() == O.compress(x[:0])


@pytest.mark.parametrize("kind,n", [("csource", (8 << 20) + 1), ("tarmix", 3 * (8 << 20) + 4097 * 3 + 17),
                                    ("random", 2 * (8 << 20)), ("runs20", 5 * (8 << 20) - 1)])
def test_compress_host_pipelined(env, kind, n):
    """Inputs above one 8 MiB group take the pipelined host path (groups on
    two compute streams, payload D2H placed by the earlier groups' totals):
    the host stream equals the device-API stream, whose chunks the oracle
    checks (first, last, and a spread of sampled chunks)."""
    torch, culzss = env
    x = datagen.generate(kind, n, seed=21)
    h = culzss.compress_host(x).tobytes()
    d = culzss.compress(dev(torch, x)).cpu().numpy().tobytes()
    assert h == d
    S, C = 4096, (n + 4095) // 4096
    sizes = np.frombuffer(h[32:32 + 4 * C], "<u4").astype(np.int64)
    offs = np.concatenate([[0], np.cumsum(sizes)]) + 32 + 4 * C
    for c in sorted({0, C - 1} | set(range(0, C, max(1, C // 24)))):
        ref = O.compress(x[c * S:min(n, (c + 1) * S)])
        assert h[offs[c]:offs[c + 1]] == ref[36:], c
    # pinned host buffers through the raw-pointer entry point (bench e2e path)
    xin = torch.from_numpy(x).pin_memory()
    cap = culzss.max_compressed_size(n)
    out = torch.empty(cap, dtype=torch.uint8).pin_memory()
    on = culzss.compress_host_ptr(xin.data_ptr(), n, out.data_ptr(), cap)
    assert out[:on].numpy().tobytes() == h
    # device-placed payloads land at any byte alignment of the pinned output
    out2 = torch.zeros(cap + 8, dtype=torch.uint8).pin_memory()
    on = culzss.compress_host_ptr(xin.data_ptr(), n, out2.data_ptr() + 3, cap)
    assert out2[3:3 + on].numpy().tobytes() == h


def test_sharded_assembly_equals_single(env):
    """SURVEY §8(e) on one GPU: R simulated ranks compress chunk ranges with
    culzss_compress_chunks; placing table slices at 32 + 4*c0 and payloads
    at 32 + 4C + sum of earlier totals reproduces the 1-call stream."""
    torch, culzss = env
    x_np = datagen.generate("csource", 37 * 4096 + 1111, seed=12)
    x = dev(torch, x_np)
    ref = culzss.compress(x).cpu().numpy().tobytes()
    assert ref == O.compress(x_np)
    n, S = x_np.size, 4096
    C = (n + S - 1) // S
    for R in (2, 3, 4, 8):
        parts, totals, tables = [], [], []
        for r in range(R):
            c0, c1 = r * C // R, (r + 1) * C // R
            sl = x[c0 * S:min(c1 * S, n)]
            pay = torch.empty(max(1, culzss.max_compressed_size(sl.numel()) - 32), dtype=torch.uint8, device="cuda")
            sizes = torch.zeros(max(1, c1 - c0), dtype=torch.int32, device="cuda")
            t = culzss.compress_chunks(sl, pay, sizes)
            parts.append(pay[:t])
            totals.append(t)
            tables.append(sizes[:c1 - c0])
        out = torch.empty(32 + 4 * C + sum(totals), dtype=torch.uint8, device="cuda")
        culzss.write_header(out, n)
        out[32:32 + 4 * C] = torch.cat(tables).view(torch.uint8)
        pos = 32 + 4 * C
        for r in range(R):
            out[pos:pos + totals[r]] = parts[r]
            pos += totals[r]
        assert out.cpu().numpy().tobytes() == ref, R


# ------------------------------------------------------------ full-size configs
def _sampled_chunk_check(x_np, stream: bytes, nsample: int, seed: int):
    n, S = x_np.size, 4096
    C = (n + S - 1) // S
    hdr = struct.unpack("<4sHHIIQHHB3x", stream[:32])
    assert hdr == (b"CLZS", 1, 32, S, C, n, 128, 128, 3)
    sizes = np.frombuffer(stream, dtype="<u4", count=C, offset=32).astype(np.int64)
    offs = 32 + 4 * C + np.concatenate([[0], np.cumsum(sizes)])
    assert offs[-1] == len(stream)
    rng = np.random.default_rng(seed)
    picks = set(rng.integers(0, C, nsample).tolist()) | {0, C - 1}
    for c in sorted(picks):
        chunk = x_np[c * S:(c + 1) * S]
        assert stream[offs[c]:offs[c + 1]] == O.compress_chunk(chunk), c


@pytest.mark.parametrize("cfg", ["c2_csource_128m", "c3_runs20_1g", "c4_random_1g"])
def test_full_size_configs(env, cfg):
    """BASELINE configs at full size, in the launch configuration bench.py
    times: header, table sum, >=512 oracle-checked chunks (+ first/last), and
    an exact on-device round trip of the whole input."""
    torch, culzss = env
    spec = datagen.CONFIGS[cfg]
    x_np = datagen.generate(spec["kind"], spec["n"], spec["seed"])
    x = torch.from_numpy(x_np).cuda()
    s = culzss.compress(x)
    stream = s.cpu().numpy().tobytes()
    _sampled_chunk_check(x_np, stream, 512, seed=len(stream))
    y = culzss.decompress(s)
    assert torch.equal(x, y)
    del y, s, x
    torch.cuda.empty_cache()


@pytest.mark.parametrize("S", [64, 128, 256, 512, 1024, 2048])
@pytest.mark.parametrize("W,F", [(128, 128), (32, 258), (255, 200), (1, 3)])
def test_packed_small_chunks(env, S, W, F):
    """Chunks of S = 64..2048 are packed 4096 / S to a warp pair: every
    window, lookahead and bit stream must still stop at its own chunk's
    bounds.  Ragged totals leave a partial last pair and a partial last chunk."""
    torch, culzss = env
    for kind in ("english", "runs20", "period20", "tarmix"):
        n = 3 * 4096 + 5 * S + S // 3 + 1
        x = datagen.generate(kind, n, seed=S + W)
        assert gpu_stream(env, x, S=S, W=W, F=F) == O.compress(x, S=S, W=W, F=F), kind


@pytest.mark.parametrize("S", [64, 256, 2048])
def test_packed_small_chunks_match_and_tokens(env, S):
    """Rows a2/a3 with packed chunks: per-position (L, D) and parse tokens
    per chunk, versions 0 and 2."""
    torch, culzss = env
    x = datagen.generate("csource", 2 * 4096 + 3 * S + 7, seed=S)
    for version in (0, 2):
        p = culzss.Params.make(S=S, version=version)
        L, D = culzss.match_search(dev(torch, x), p)
        L, D = L.cpu().numpy(), D.cpu().numpy()
        tok = culzss.parse_tokens(dev(torch, x), p).cpu().numpy().astype(np.int64) & 0xFFFFFFFF
        for c in range((x.size + S - 1) // S):
            chunk = x[c * S:(c + 1) * S]
            eL, eD = O.match_all(chunk)
            np.testing.assert_array_equal(L[c * S:c * S + chunk.size], eL, err_msg=f"v{version} c{c}")
            np.testing.assert_array_equal(D[c * S:c * S + chunk.size], eD, err_msg=f"v{version} c{c}")
            np.testing.assert_array_equal(tok[c * S:c * S + chunk.size],
                                          expand_tokens(O.tokens_chunk(chunk), chunk.size))


@pytest.mark.parametrize("S,version", [(256, 0), (4096, 2), (512, 2), (1000, 0)])
def test_host_api_param_combinations(env, S, version):
    """The pipelined host path (several 8 MiB groups) with packed small chunks
    and with version 2: the same bytes as the oracle."""
    torch, culzss = env
    n = 2 * (8 << 20) + 4097
    x = datagen.generate("tarmix", n, seed=S + version)
    p = culzss.Params.make(S=S, version=version)
    h = culzss.compress_host(x, params=p).tobytes()
    C = (n + S - 1) // S
    sizes = np.frombuffer(h[32:32 + 4 * C], "<u4").astype(np.int64)
    offs = np.concatenate([[0], np.cumsum(sizes)]) + 32 + 4 * C
    assert offs[-1] == len(h)
    for c in sorted({0, C - 1} | set(range(0, C, max(1, C // 40)))):
        assert h[offs[c]:offs[c + 1]] == O.compress_chunk(x[c * S:min(n, (c + 1) * S)]), c


@pytest.mark.parametrize("S", [64, 512, 2048])
def test_sharded_packed_chunks_roundtrip(env, S):
    """Sharding primitives with packed small chunks: per-rank compress_chunks
    outputs assemble into the oracle's stream and decode back per rank."""
    torch, culzss = env
    n = 40 * 4096 + 3 * S + 5
    x_np = datagen.generate("csource", n, seed=S)
    x = dev(torch, x_np)
    p = culzss.Params.make(S=S)
    C = (n + S - 1) // S
    parts, tables = [], []
    for r in range(3):
        c0, c1 = r * C // 3, (r + 1) * C // 3
        sl = x[c0 * S:min(c1 * S, n)]
        pay = torch.empty(max(1, culzss.max_compressed_size(sl.numel(), p)), dtype=torch.uint8, device="cuda")
        sizes = torch.zeros(max(1, c1 - c0), dtype=torch.int32, device="cuda")
        t = culzss.compress_chunks(sl, pay, sizes, p)
        assert torch.equal(culzss.decompress_chunks(pay[:t], sizes[:c1 - c0], sl.numel(), params=p), sl)
        parts.append(pay[:t].cpu().numpy().tobytes())
        tables.append(sizes[:c1 - c0].cpu().numpy().astype("<u4").tobytes())
    ref = O.compress(x_np, S=S)
    assert ref[32:32 + 4 * C] == b"".join(tables)
    assert ref[32 + 4 * C:] == b"".join(parts)


@pytest.mark.parametrize("kind,n,S", [("csource", (8 << 20) + 1, 4096), ("tarmix", 3 * (8 << 20) + 4097 * 3 + 17, 4096),
                                      ("random", 2 * (8 << 20), 4096), ("runs20", 5 * (8 << 20) - 1, 4096),
                                      ("english", 100_001, 4096), ("csource", 3 * (8 << 20) + 5, 512),
                                      ("english", 1, 4096)])
def test_decompress_host(env, kind, n, S):
    """Host-memory decompression of oracle streams (single and multi-group,
    packed chunk size), byte-exact."""
    torch, culzss = env
    x = datagen.generate(kind, n, seed=n % 1000)
    # small inputs: the oracle's stream; large: the GPU stream (whose chunks the
    # oracle checks in the other tests) -- the host decoder must return the input
    s = np.frombuffer(O.compress(x, S=S), np.uint8) if n < (1 << 20) else \
        culzss.compress_host(x, params=culzss.Params.make(S=S))
    y = culzss.decompress_host(s)
    assert y.tobytes() == x.tobytes()
    # pinned buffers through the raw-pointer entry point
    sin = torch.from_numpy(np.array(s, dtype=np.uint8)).pin_memory()
    out = torch.empty(n + 7, dtype=torch.uint8).pin_memory()
    on = culzss.decompress_host_ptr(sin.data_ptr(), s.size, out.data_ptr() + 3, n + 4)
    assert on == n and out[3:3 + n].numpy().tobytes() == x.tobytes()


def test_decompress_host_rejects(env):
    torch, culzss = env
    import test_oracle_pins as P
    for _, s in P.CORRUPT_STREAMS:
        st, _ = culzss.decompress_host_status(np.frombuffer(s, np.uint8))
        assert st == culzss.ERR_CORRUPT, s
    x = datagen.generate("english", 20000, seed=4)
    base = bytearray(O.compress(x))
    rng = np.random.default_rng(7)
    for _ in range(100):
        s = bytearray(base)
        for _ in range(int(rng.integers(1, 4))):
            i = int(rng.integers(0, len(s)))
            s[i] ^= int(rng.integers(1, 256))
        ost, oout = O.decompress_status(bytes(s))
        gst, gout = culzss.decompress_host_status(np.frombuffer(bytes(s), np.uint8))
        if ost == O.OK:
            assert gst == culzss.OK and gout.tobytes() == oout
        else:
            assert gst in (culzss.ERR_CORRUPT, culzss.ERR_UNSUPPORTED)
    st, _ = culzss.decompress_host_status(np.frombuffer(bytes(base), np.uint8), out=np.empty(10, np.uint8))
    assert st == culzss.ERR_BUFFER_TOO_SMALL


@pytest.mark.parametrize("cfg", ["c2_csource_128m", "c3_runs20_1g", "c4_random_1g", "c5_tarmix_1g_slice"])
def test_full_size_configs_every_chunk(env, cfg):
    """BASELINE configs at full size: EVERY chunk of the GPU stream against the
    oracle (threads over contiguous chunk ranges on the box's host cores), plus
    the header and the size table."""
    import concurrent.futures as cf
    import os
    torch, culzss = env
    if cfg == "c5_tarmix_1g_slice":  # 1 GiB of the c5 generator (its per-rank slices are 8 GiB at dp8)
        spec = dict(datagen.CONFIGS["c5_tarmix_64g"], n=1 << 30)
    else:
        spec = datagen.CONFIGS[cfg]
    x_np = datagen.generate(spec["kind"], spec["n"], spec["seed"])
    stream = culzss.compress(torch.from_numpy(x_np).cuda()).cpu().numpy().tobytes()
    n, S = x_np.size, 4096
    C = (n + S - 1) // S
    assert stream[:32] == struct.pack("<4sHHIIQHHB3x", b"CLZS", 1, 32, S, C, n, 128, 128, 3)
    k = max(1, min(len(os.sched_getaffinity(0)), 64))
    bounds = [(i * C // k, (i + 1) * C // k) for i in range(k)]
    with cf.ThreadPoolExecutor(k) as ex:
        res = list(ex.map(lambda b: O.compress_range(x_np, b[0], b[1]), bounds))
    sizes = np.concatenate([r[1] for r in res]).astype("<u4").tobytes()
    assert stream[32:32 + 4 * C] == sizes
    assert stream[32 + 4 * C:] == b"".join(r[0] for r in res)
