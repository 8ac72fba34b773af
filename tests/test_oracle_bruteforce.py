"""Brute-force and property pins of the oracle on tiny inputs.

The reference here is an independent formulation, not the oracle's loop:
  * a match (d, L) at p is *valid* iff LZ77-decoding it (byte-serial copy,
    out[i] = out[i-d], PAPER.md:1@6743 §II.A.2) after the already-known
    prefix reproduces the next L bytes;
  * L(p) = the largest valid L <= min(F, m-p) over 1 <= d <= min(W, p), with
    the smallest d among those (R7), and L < 3 means literal (R4);
  * the parse is the recursive greedy definition (R8);
  * bits are produced by string formatting (R9-R11), the container by
    struct.pack (R12).
"""
import itertools
import struct

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import oracle as O


def ref_decode_copy(prefix: bytes, d: int, L: int) -> bytes:
    buf = bytearray(prefix)
    for _ in range(L):
        buf.append(buf[-d])
    return bytes(buf[len(prefix):])


def ref_match(chunk: bytes, p: int, W: int, F: int, MIN: int = 3):
    cap = min(F, len(chunk) - p)
    best = (0, 0)
    for d in range(1, min(W, p) + 1):
        got = ref_decode_copy(chunk[:p], d, cap)
        L = 0
        while L < cap and got[L] == chunk[p + L]:
            L += 1
        if L > best[0]:
            best = (L, d)
    return best if best[0] >= MIN else (0, 0)


def ref_tokens(chunk: bytes, W: int, F: int):
    if not chunk:
        return []
    out, p = [], 0
    while p < len(chunk):
        L, d = ref_match(chunk, p, W, F)
        if L:
            out.append(("M", d, L))
            p += L
        else:
            out.append(("L", chunk[p]))
            p += 1
    return out


def ref_payload(chunk: bytes, W: int, F: int) -> bytes:
    bits = []
    for t in ref_tokens(chunk, W, F):
        bits.append("0" + format(t[1], "08b") if t[0] == "L"
                    else "1" + format(t[1] - 1, "08b") + format(t[2] - 3, "08b"))
    b = "".join(bits)
    b += "0" * (-len(b) % 8)
    return bytes(int(b[i:i + 8], 2) for i in range(0, len(b), 8))


def ref_stream(data: bytes, S: int, W: int, F: int) -> bytes:
    C = (len(data) + S - 1) // S
    pays = [ref_payload(data[c * S:(c + 1) * S], W, F) for c in range(C)]
    hdr = struct.pack("<4sHHIIQHHB3x", b"CLZS", 1, 32, S, C, len(data), W, F, 3)
    return hdr + b"".join(struct.pack("<I", len(p)) for p in pays) + b"".join(pays)


def all_strings(alphabet: bytes, maxlen: int):
    for n in range(1, maxlen + 1):
        for t in itertools.product(alphabet, repeat=n):
            yield bytes(t)


PARAMS = [(4096, 128, 128), (8, 4, 3), (16, 3, 9), (4, 8, 5), (8, 1, 4), (16, 2, 3)]


@pytest.mark.parametrize("S,W,F", PARAMS)
def test_exhaustive_ab(S, W, F):
    """Every {a,b} string of length <= 10: stream bytes and per-position
    (L, D) equal the independent definition."""
    for s in all_strings(b"ab", 10):
        assert O.compress(s, S=S, W=W, F=F) == ref_stream(s, S, W, F), s
        chunk = s[:S]
        L, D = O.match_all(chunk, W=W, F=F)
        for p in range(len(chunk)):
            assert (int(L[p]), int(D[p])) == ref_match(chunk, p, W, F), (s, p)


@pytest.mark.parametrize("S,W,F", PARAMS[:3])
def test_exhaustive_abc(S, W, F):
    for s in all_strings(b"abc", 7):
        assert O.compress(s, S=S, W=W, F=F) == ref_stream(s, S, W, F), s


def test_random_medium_vs_reference():
    """Longer strings over small alphabets, default params: several chunks and
    a ragged tail, still checked against the independent definition."""
    rng = np.random.default_rng(11)
    for trial in range(6):
        k = [2, 3, 4, 26, 256, 2][trial]
        n = int(rng.integers(300, 700))
        s = bytes(rng.integers(0, k, size=n, dtype=np.uint8).tolist())
        S = [4096, 256, 128, 4096, 200, 97][trial]
        assert O.compress(s, S=S) == ref_stream(s, S, 128, 128)


@settings(max_examples=150, deadline=None)
@given(st.binary(min_size=0, max_size=3000), st.sampled_from([1, 2, 3, 16, 256]),
       st.sampled_from([(4096, 128, 128), (64, 16, 18), (1000, 256, 258), (7, 2, 3)]))
def test_roundtrip_property(raw, k, params):
    """decompress(compress(x)) == x; stream length and per-chunk bounds."""
    S, W, F = params
    x = bytes(b % k for b in raw)
    s = O.compress(x, S=S, W=W, F=F)
    assert O.decompress(s) == x
    C = (len(x) + S - 1) // S
    sizes = struct.unpack(f"<{C}I", s[32:32 + 4 * C])
    assert len(s) == 32 + 4 * C + sum(sizes)
    for c, sz in enumerate(sizes):
        m = min(S, len(x) - c * S)
        assert sz <= (9 * m + 7) // 8


@settings(max_examples=300, deadline=None)
@given(st.binary(min_size=1, max_size=600), st.integers(0, 10 ** 6), st.integers(1, 4))
def test_mutated_streams_never_crash(raw, seed, nmut):
    """Fault injection: mutated streams decode to CORRUPT or to *some* output
    of the declared length -- never a crash or out-of-bounds access."""
    x = bytes(b % 4 for b in raw)
    s = bytearray(O.compress(x))
    rng = np.random.default_rng(seed)
    for _ in range(nmut):
        i = int(rng.integers(0, len(s)))
        s[i] ^= int(rng.integers(1, 256))
    st_, out = O.decompress_status(bytes(s))
    assert st_ in (O.OK, O.ERR_CORRUPT)
    if st_ == O.OK:
        assert len(out) == struct.unpack("<Q", bytes(s[16:24]))[0]


@pytest.mark.parametrize("S,W,F,k", [(64, 128, 128, 3), (64, 255, 258, 2), (128, 128, 20, 4), (512, 64, 128, 3)])
def test_small_chunks_window_beyond_chunk(S, W, F, k):
    """Chunks smaller than the window (the packed GPU geometry's case): the
    window never reaches before the chunk start (R5) and the lookahead stops
    at its end, against the independent definition."""
    rng = np.random.default_rng(S + W + F + k)
    for _ in range(3):
        n = int(rng.integers(3 * S, 3 * S + 200))
        s = bytes(rng.integers(0, k, size=n, dtype=np.uint8).tolist())
        assert O.compress(s, S=S, W=W, F=F) == ref_stream(s, S, W, F)
