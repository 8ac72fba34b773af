"""Pins of the CPU oracle against what the paper and the mathematics fix.

Every expected value below comes from the paper (cited), from hand work
written out in the test, or from a closed form derived in the docstring --
never from the oracle itself and never from the CUDA path.
"""
import json
import os
import struct

import numpy as np
import pytest

import oracle as O

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def bits_to_bytes(bits: str) -> bytes:
    """MSB-first bit string -> bytes, zero padded (reading R11)."""
    bits = bits + "0" * (-len(bits) % 8)
    return bytes(int(bits[i:i + 8], 2) for i in range(0, len(bits), 8))


def lit(ch) -> str:
    return "0" + format(ch if isinstance(ch, int) else ord(ch), "08b")


def mat(d, L, MIN=3) -> str:
    return "1" + format(d - 1, "08b") + format(L - MIN, "08b")


def header(n, S=4096, W=128, F=128, MIN=3):
    C = (n + S - 1) // S
    return struct.pack("<4sHHIIQHHB3x", b"CLZS", 1, 32, S, C, n, W, F, MIN)


# ---------------------------------------------------------------- Figure 1
def test_figure1_token_sequence():
    """PAPER.md:1@6051 Figure 1: 42 literals + 8 matches at the printed
    absolute offsets (R9: d = p - offset)."""
    g = json.load(open(os.path.join(GOLDEN, "figure1.json")))
    text = g["text"].encode()
    assert len(text) == g["total_characters"] == 102
    toks = O.tokens_chunk(text)
    # expand the printed encoding into the expected token list
    expect, p = [], 0
    for item in g["encoded"]:
        if isinstance(item, str):
            for ch in item.encode():
                expect.append(("L", ch))
                p += 1
        else:
            off, L = item
            expect.append(("M", p - off, L))
            p += L
    assert p == len(text)
    assert toks == expect
    assert sum(t[0] == "L" for t in toks) == g["literals"]
    assert sum(t[0] == "M" for t in toks) == g["matches"]


def test_figure1_needs_lookahead_19():
    """R2: Figure 1's (24,19) needs F >= 19; at F = 18 it must split."""
    text = json.load(open(os.path.join(GOLDEN, "figure1.json")))["text"].encode()
    toks = O.tokens_chunk(text, F=18)
    assert ("M", 59, 19) not in toks and ("M", 59, 18) in toks


# ---------------------------------------------------------------- min match 3
@pytest.mark.parametrize("s,tokens", [
    (b"abXab", [("L", 97), ("L", 98), ("L", 88), ("L", 97), ("L", 98)]),  # 2-match costs more than it saves
    (b"aaa", [("L", 97)] * 3),                      # L(1) = 2 < 3 (cap m-p = 2)
    (b"aaaa", [("L", 97), ("M", 1, 3)]),            # overlap (R6)
    (b"aaaaaaaaaa", [("L", 97), ("M", 1, 9)]),
    (b"abcabcabcabc", [("L", 97), ("L", 98), ("L", 99), ("M", 3, 9)]),
    (b"abcXabcYabc", [("L", 97), ("L", 98), ("L", 99), ("L", 88), ("M", 4, 3), ("L", 89), ("M", 4, 3)]),  # R7 smallest d
])
def test_hand_worked_tokens(s, tokens):
    """PAPER.md:1@5848: 'The minimum number of match ... in our case it is three'."""
    assert O.tokens_chunk(s) == tokens


def test_min_match_rule_bit_cost():
    """PAPER.md:1@5848-6051: a 2-byte match costs as much as two literals; 3 is
    the first length that saves bits: 17 < 27."""
    assert len(mat(1, 3)) == 17 and 3 * len(lit("a")) == 27
    # a 2-character match: 17 bits vs 18 for two literals -- both round to the
    # same number of bytes, so the paper does not code it
    assert (len(mat(1, 3)) + 7) // 8 == (2 * len(lit("a")) + 7) // 8


# ---------------------------------------------------------------- bit layout
@pytest.mark.parametrize("s,bits", [
    (b"a", lit("a")),
    (b"ab", lit("a") + lit("b")),
    (b"aaa", lit("a") * 3),
    (b"aaaa", lit("a") + mat(1, 3)),
    (b"aaaaaaaaaa", lit("a") + mat(1, 9)),
    (b"abcXabcYabc", lit("a") + lit("b") + lit("c") + lit("X") + mat(4, 3) + lit("Y") + mat(4, 3)),
])
def test_hand_built_bit_vectors(s, bits):
    """R9-R11: flag before each token, 0 literal / 1 match, MSB first,
    (d-1) and (L-3) in 8 bits each (PAPER.md:1@23049 16-bit code)."""
    assert O.compress_chunk(s) == bits_to_bytes(bits)


def test_hex_examples_written_out():
    # 'a' = 0 01100001 -> 0011 0000 1000 0000 (padded)
    assert O.compress_chunk(b"a") == bytes([0x30, 0x80])
    # 'aaaa' = 0 01100001 | 1 00000000 00000000 -> 0x30 0xC0 0x00 0x00 (26 bits)
    assert O.compress_chunk(b"aaaa") == bytes([0x30, 0xC0, 0x00, 0x00])


# ---------------------------------------------------------------- container
def test_header_layout_and_stream():
    """R12: 32-byte LE header, u32 sizes, payloads (PAPER.md:1@18853)."""
    s = O.compress(b"aaaa")
    assert s[:32] == header(4)
    assert s[32:36] == struct.pack("<I", 4)
    assert s[36:] == bits_to_bytes(lit("a") + mat(1, 3))


def test_empty_and_one_byte():
    assert O.compress(b"") == header(0)                     # R13: n=0 -> 32-byte stream
    assert O.decompress(header(0)) == b""
    assert O.compress(b"\x00") == header(1) + struct.pack("<I", 2) + bits_to_bytes(lit(0))


def test_max_compressed_size_closed_form():
    for n in [0, 1, 7, 4095, 4096, 4097, 100000]:
        C = (n + 4095) // 4096
        bound = 32 + 4 * C + (n // 4096) * 4608 + ((9 * (n % 4096) + 7) // 8 if n % 4096 else 0)
        assert O.max_compressed_size(n) == bound


# ---------------------------------------------------------------- window / cap / chunk edges
def _distinct_period(p, seed=0):
    """p <= 256 distinct byte values: x == y  iff  positions equal mod p."""
    rng = np.random.default_rng(seed + p)
    return rng.permutation(256)[:p].astype(np.uint8)


def period_size(p, m, F=128):
    """Closed form for a period-p chunk of length m with distinct bytes per
    period and p <= W: first p bytes literal; then (p, F) matches; a tail t < 3
    is literal (too short), t >= 3 one more match."""
    q, t = divmod(m - p, F)
    matches = q + (1 if t >= 3 else 0)
    literals = p + (t if t < 3 else 0)
    return (9 * literals + 17 * matches + 7) // 8


@pytest.mark.parametrize("p", [1, 2, 3, 20, 64, 100, 127, 128])
@pytest.mark.parametrize("m", [130, 1000, 4096])
def test_period_closed_form(p, m):
    if p > m:
        return
    x = np.tile(_distinct_period(p), m // p + 1)[:m]
    assert len(O.compress_chunk(x)) == period_size(p, m)


def test_period_examples_from_survey():
    assert period_size(1, 4096) == 70 and period_size(20, 4096) == 91
    assert period_size(100, 4096) == 181 and period_size(127, 4096) == 210
    assert period_size(128, 4096) == 210


def test_window_edge_128_vs_129():
    """R1: W = 128 (PAPER.md:1@22955).  Period 128 is matched at d = 128;
    period 129 is out of the window: every byte is a literal."""
    x128 = np.tile(_distinct_period(128), 40)[:4096]
    toks = O.tokens_chunk(x128)
    assert all(t[1] == 128 for t in toks if t[0] == "M") and any(t[0] == "M" for t in toks)
    x129 = np.tile(_distinct_period(129), 40)[:4096]
    assert all(t[0] == "L" for t in O.tokens_chunk(x129))
    assert len(O.compress_chunk(x129)) == 4608


def test_lookahead_cap():
    """R2: F = 128 caps a run of 300 equal bytes into 128 + 128 + 43."""
    assert O.tokens_chunk(b"z" * 300) == [("L", 122), ("M", 1, 128), ("M", 1, 128), ("M", 1, 43)]


def test_chunk_independence_and_sizes():
    """R3/R5: 5000 x 'q' -> chunks of 4096 and 904 bytes, compressed
    independently: sizes 70 and ceil((9 + 17*8)/8) = 19 (904 = 1 + 7*128 + 7)."""
    s = O.compress(b"q" * 5000)
    assert struct.unpack("<II", s[32:40]) == (70, 19)
    assert len(s) == 32 + 8 + 70 + 19
    # the second chunk's payload equals the payload of the 904-byte input alone
    assert s[32 + 8 + 70:] == O.compress_chunk(b"q" * 904)


def test_all_literal_bound_no_repeats():
    """A chunk where equal bytes are >= 256 apart has no match: 9 bits/byte."""
    x = (np.arange(4096) & 0xFF).astype(np.uint8)
    assert len(O.compress_chunk(x)) == 4608


def test_all_literal_bound_random():
    """size_c <= ceil(9 m / 8) for every chunk (invariant)."""
    rng = np.random.default_rng(7)
    x = rng.integers(0, 256, size=3 * 4096 + 100, dtype=np.uint8)
    s = O.compress(x)
    C = 4
    sizes = struct.unpack("<4I", s[32:48])
    ms = [4096, 4096, 4096, 100]
    for sz, m in zip(sizes, ms):
        assert sz <= (9 * m + 7) // 8
    assert len(s) == 32 + 4 * C + sum(sizes)


# ---------------------------------------------------------------- decoder
def test_decoder_hand_built_stream():
    payload = bits_to_bytes(lit("x") + lit("y") + mat(2, 5) + lit("!"))
    stream = header(8) + struct.pack("<I", len(payload)) + payload
    assert O.decompress(stream) == b"xyxyxyx!"


def _stream(n, payload_bits, S=4096):
    payload = bits_to_bytes(payload_bits)
    return header(n, S) + struct.pack("<I", len(payload)) + payload


CORRUPT_STREAMS = [
    ("bad magic", b"CLZX" + _stream(4, lit("a") + mat(1, 3))[4:]),
    ("d > produced", _stream(4, lit("a") + mat(2, 3))),
    ("L > remaining", _stream(3, lit("a") + mat(1, 3))),
    ("nonzero pad", _stream(1, lit("a") + "1")),
    ("size too big", header(1) + struct.pack("<I", 3) + bits_to_bytes(lit("a")) + b"\x00"),
    ("truncated", _stream(2, lit("a"))),
    ("table sum", header(1) + struct.pack("<I", 2) + bits_to_bytes(lit("a")) + b"\x00"),
    ("C mismatch", struct.pack("<4sHHIIQHHB3x", b"CLZS", 1, 32, 4096, 2, 1, 128, 128, 3)
     + struct.pack("<I", 2) + bits_to_bytes(lit("a"))),
    ("reserved", _stream(1, lit("a"))[:29] + b"\x01\x00\x00" + _stream(1, lit("a"))[32:]),
    ("bad params", struct.pack("<4sHHIIQHHB3x", b"CLZS", 1, 32, 4096, 1, 1, 0, 128, 3)
     + struct.pack("<I", 2) + bits_to_bytes(lit("a"))),
    # Each stream below is valid in every respect but ONE, so each isolates
    # one rejection branch of the decoder (DESIGN.md §3 decoder strictness;
    # PAPER.md:1@6743 §II.A.2 decode rule; readings R9, R10, R12).
    # d = 5 > W = 4, though d <= produced (5) and L = 3 <= remaining (3)
    ("d > W", header(8, W=4) + struct.pack("<I", len(bits_to_bytes("".join(lit(ch) for ch in "abcde") + mat(5, 3))))
     + bits_to_bytes("".join(lit(ch) for ch in "abcde") + mat(5, 3))),
    # L = 6 > F = 5, though L <= remaining (6) and d = 1 <= produced
    ("L > F", header(7, F=5) + struct.pack("<I", len(bits_to_bytes(lit("a") + mat(1, 6))))
     + bits_to_bytes(lit("a") + mat(1, 6))),
    # header version 2 (R12 fixes version = 1)
    ("version", _stream(1, lit("a"))[:4] + struct.pack("<H", 2) + _stream(1, lit("a"))[6:]),
    # header_bytes = 64 (R12 fixes 32)
    ("header_bytes", _stream(1, lit("a"))[:6] + struct.pack("<H", 64) + _stream(1, lit("a"))[8:]),
    # C = 1 < ceil(4097 / 4096) = 2, with a table and payload that agree with
    # C = 1 (the one chunk decodes 4096 bytes cleanly): only the C check sees it
    ("C too small", struct.pack("<4sHHIIQHHB3x", b"CLZS", 1, 32, 4096, 1, 4097, 128, 128, 3)
     + struct.pack("<I", len(bits_to_bytes(lit("z") + mat(1, 128) * 31 + mat(1, 127))))
     + bits_to_bytes(lit("z") + mat(1, 128) * 31 + mat(1, 127))),
    # C = 0 for n = 1: an empty table and no payload
    ("C zero", struct.pack("<4sHHIIQHHB3x", b"CLZS", 1, 32, 4096, 0, 1, 128, 128, 3)),
]


@pytest.mark.parametrize("name,stream", CORRUPT_STREAMS)
def test_decoder_rejects_corrupt(name, stream):
    st, _ = O.decompress_status(stream)
    assert st == O.ERR_CORRUPT, name


def test_isolating_streams_decode_once_fixed():
    """Positive controls for the isolating corrupt streams: with the one bad
    field set right, each decodes (so the rejection above is that field's)."""
    five = "".join(lit(ch) for ch in "abcde")
    ok_w = header(8, W=5) + struct.pack("<I", len(bits_to_bytes(five + mat(5, 3)))) + bits_to_bytes(five + mat(5, 3))
    assert O.decompress(ok_w) == b"abcdeabc"
    ok_f = header(7, F=6) + struct.pack("<I", len(bits_to_bytes(lit("a") + mat(1, 6)))) + bits_to_bytes(lit("a") + mat(1, 6))
    assert O.decompress(ok_f) == b"a" * 7
    pay = bits_to_bytes(lit("z") + mat(1, 128) * 31 + mat(1, 127))
    ok_c = (struct.pack("<4sHHIIQHHB3x", b"CLZS", 1, 32, 4096, 1, 4096, 128, 128, 3)
            + struct.pack("<I", len(pay)) + pay)
    assert O.decompress(ok_c) == b"z" * 4096
    assert O.decompress(_stream(1, lit("a"))) == b"a"


def test_params_validation():
    assert O.params_valid()
    assert not O.params_valid(MIN=2)
    assert not O.params_valid(W=0) and not O.params_valid(W=257)
    assert not O.params_valid(F=2) and not O.params_valid(F=259)
    assert O.params_valid(W=256, F=258)
