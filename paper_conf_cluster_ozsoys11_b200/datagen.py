"""Seeded synthetic inputs shaped like the paper's workloads.

This module holds NO compression arithmetic: it only produces bytes.  It is
the one module both the CUDA path's tests/bench and the oracle's tests read
their inputs from (DESIGN.md §4 "input recipe").

Workload shapes (PAPER.md:1@23810 §IV.B: five 128 MB sets):
  * ``csource``  -- "a collection of C files ... text based input" (@23843)
  * ``english``  -- English-like running text (64 KiB bit-exact config)
  * ``wordlist`` -- "English dictionary ... alphabetically ordered not
                    repeating words" (@24391)
  * ``runs20``   -- "highly compressible ... repeating characters in
                    substrings of 20" (@24662), reading R17: runs of 20
                    identical bytes; ``period20`` is the secondary reading
  * ``random``   -- incompressible bytes (splitmix64)
  * ``tarmix``   -- tarball-like mix (Linux kernel tarball @24533 and DE Map
                    raster data @23946)

Large inputs are built from a seeded base corpus (a few MiB produced by the
generator proper) by concatenating seeded random segments of it.  With a
128-byte window and 4 KiB chunks, repetition at distances > 4 KiB is
invisible to the method, so the per-chunk statistics are those of the base.
"""
from __future__ import annotations

import numpy as np

GENERATORS = ("english", "wordlist", "csource", "runs20", "period20", "random", "tarmix")

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)


def splitmix64(n_words: int, seed: int) -> np.ndarray:
    """splitmix64 stream of n_words uint64 (counter-based, vectorised)."""
    with np.errstate(over="ignore"):
        idx = np.arange(1, n_words + 1, dtype=np.uint64)
        z = np.uint64(seed) + idx * np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return z


def gen_random(n: int, seed: int = 4) -> np.ndarray:
    w = splitmix64((n + 7) // 8, seed)
    return w.view(np.uint8)[:n].copy()


def gen_runs20(n: int, seed: int = 3) -> np.ndarray:
    rng = np.random.Generator(np.random.PCG64(seed))
    letters = rng.integers(ord("a"), ord("z") + 1, size=(n + 19) // 20, dtype=np.uint8)
    return np.repeat(letters, 20)[:n].copy()


def _period20_base(rng) -> bytes:
    # a 20-letter string whose cyclic 3-grams are all distinct
    while True:
        s = rng.integers(ord("a"), ord("z") + 1, size=20, dtype=np.uint8).tobytes()
        grams = {(s + s[:2])[i:i + 3] for i in range(20)}
        if len(grams) == 20:
            return s


def gen_period20(n: int, seed: int = 3) -> np.ndarray:
    rng = np.random.Generator(np.random.PCG64(seed))
    base = np.frombuffer(_period20_base(rng), dtype=np.uint8)
    return np.tile(base, (n + 19) // 20)[:n].copy()


# ---------------------------------------------------------------- text
# The 100 most frequent English function/content words (public-domain
# frequency lists) carry about half of running English text.
_COMMON = (b"the of and to a in is that it was for on are as with his they i at be this "
           b"have from or one had by word but not what all were we when your can said "
           b"there use an each which she do how their if will up other about out many "
           b"then them these so some her would make like him into time has look two more "
           b"write go see number no way could people my than first water been call who "
           b"oil its now find long down day did get come made may part").split()
_ONSETS = [b"", b"b", b"c", b"d", b"f", b"g", b"h", b"l", b"m", b"n", b"p", b"r", b"s", b"t",
           b"w", b"st", b"tr", b"pr", b"ch", b"th", b"sh", b"bl", b"cr", b"gr", b"pl", b"str"]
_NUCLEI = [b"a", b"e", b"i", b"o", b"u", b"ea", b"ou", b"ai", b"ee", b"io", b"oo", b"y"]
_CODAS = [b"", b"", b"n", b"r", b"s", b"t", b"l", b"nd", b"st", b"nt", b"m", b"ck", b"ng", b"rt"]
_SUFFIXES = [b"", b"", b"", b"ing", b"ed", b"er", b"ly", b"tion", b"s", b"es", b"ment", b"ness",
             b"able", b"al", b"ous", b"ive"]


def _vocab(rng, count: int, lo: int = 1, hi: int = 3) -> list:
    """Pseudo-English words built from syllables + suffixes (unique)."""
    words, seen = [], set()
    while len(words) < count:
        nsyl = int(rng.integers(lo, hi + 1))
        w = b"".join(_ONSETS[int(rng.integers(0, len(_ONSETS)))]
                     + _NUCLEI[int(rng.integers(0, len(_NUCLEI)))]
                     + _CODAS[int(rng.integers(0, len(_CODAS)))] for _ in range(nsyl))
        w += _SUFFIXES[int(rng.integers(0, len(_SUFFIXES)))]
        if w not in seen and len(w) >= 2:
            seen.add(w)
            words.append(w)
    return words


def _zipf_indices(rng, n_items: int, size: int, s: float = 1.07) -> np.ndarray:
    w = 1.0 / np.arange(1, n_items + 1) ** s
    return rng.choice(n_items, size=size, p=w / w.sum())


def _english_base(nbytes: int, seed: int) -> bytes:
    rng = np.random.Generator(np.random.PCG64(seed))
    vocab = list(_COMMON) + _vocab(rng, 4096 - len(_COMMON), 1, 2)
    idx = _zipf_indices(rng, len(vocab), nbytes // 4 + 64, 1.15)
    out, line, k = [], 0, 0
    total = 0
    while total < nbytes:
        slen = int(rng.integers(5, 26))
        for j in range(slen):
            w = vocab[idx[k % idx.size]]
            k += 1
            if j == 0:
                w = w[:1].upper() + w[1:]
            if j == slen - 1:
                w = w + b"."
            elif rng.random() < 0.08:
                w = w + b","
            if line + len(w) + 1 > 72:
                out.append(b"\n")
                total += 1
                line = 0
            elif line > 0:
                out.append(b" ")
                total += 1
                line += 1
            out.append(w)
            total += len(w)
            line += len(w)
    return b"".join(out)[:nbytes]


def _wordlist_base(nbytes: int, seed: int) -> bytes:
    rng = np.random.Generator(np.random.PCG64(seed))
    words = sorted(_vocab(rng, max(64, nbytes // 8), 1, 4))
    return b"\n".join(words)[:nbytes]


_C_TYPES = [b"int", b"unsigned int", b"long", b"char *", b"struct device *", b"size_t",
            b"u32", b"u64", b"void *", b"const char *", b"bool", b"struct list_head *"]
_C_HEADERS = [b"linux/module.h", b"linux/kernel.h", b"linux/init.h", b"linux/slab.h",
              b"linux/fs.h", b"linux/errno.h", b"linux/types.h", b"linux/string.h",
              b"linux/device.h", b"linux/spinlock.h", b"linux/mutex.h", b"stdio.h",
              b"stdlib.h", b"string.h", b"asm/io.h", b"linux/interrupt.h"]


def _csource_base(nbytes: int, seed: int) -> bytes:
    rng = np.random.Generator(np.random.PCG64(seed))
    parts = (b"dev buf len ret priv data ctx reg val count size flags lock list node info "
             b"state irq addr base port page queue entry dma cmd hw mask status init read "
             b"write get set alloc free open close start stop reset config table index "
             b"offset name type mode id num err tmp ptr skb net card chip pci usb").split()
    parts += _vocab(rng, 200, 1, 2)
    ids, seen = [], set()
    while len(ids) < 2000:
        k = int(rng.choice([1, 2, 2, 3]))
        i = b"_".join(parts[int(j)] for j in _zipf_indices(rng, len(parts), k, 0.9))
        if i not in seen:
            seen.add(i)
            ids.append(i)
    zi = _zipf_indices(rng, len(ids), nbytes // 3 + 256)
    pos = [0]

    local = [ids[0]]

    def ident():
        pos[0] += 1
        if rng.random() < 0.7:
            return local[int(rng.integers(0, len(local)))]
        return ids[zi[pos[0] % zi.size]]

    def num():
        return str(int(rng.choice([0, 1, 2, 4, 8, 16, 32, 64, 255, 1024, int(rng.integers(0, 4096))]))).encode()

    templates = [
        lambda: b"if (%s->%s > %s) {" % (ident(), ident(), num()),
        lambda: b"for (i = 0; i < %s; i++) {" % ident(),
        lambda: b"return -EINVAL;",
        lambda: b"return 0;",
        lambda: b"%s = %s(%s, %s);" % (ident(), ident(), ident(), ident()),
        lambda: b"%s->%s = %s;" % (ident(), ident(), ident()),
        lambda: b"%s += %s;" % (ident(), num()),
        lambda: b"if (!%s)" % ident(),
        lambda: b"\tgoto out;",
        lambda: b"} else {",
        lambda: b"while (%s--) {" % ident(),
        lambda: b"%s(%s);" % (ident(), ident()),
        lambda: b"spin_lock(&%s->lock);" % ident(),
        lambda: b"spin_unlock(&%s->lock);" % ident(),
        lambda: b"%s = kmalloc(sizeof(*%s), GFP_KERNEL);" % (ident(), ident()),
        lambda: b"memset(%s, 0, sizeof(%s));" % (ident(), ident()),
        lambda: b"pr_err(\"%s: failed to %s %%d\\n\", %s);" % (ident(), ident(), ident()),
        lambda: b"/* %s the %s */" % (ident(), ident()),
        lambda: b"switch (%s) {" % ident(),
        lambda: b"case %s:" % num(),
        lambda: b"break;",
        lambda: b"%s = %s & 0x%x;" % (ident(), ident(), int(rng.integers(0, 65536))),
        lambda: b"if (%s == NULL)" % ident(),
        lambda: b"\treturn -ENOMEM;",
        lambda: b"list_for_each_entry(%s, &%s->list, node) {" % (ident(), ident()),
        lambda: b"%s %s = %s;" % (_C_TYPES[int(rng.integers(0, len(_C_TYPES)))], ident(), num()),
        lambda: b"err = %s(%s, %s);" % (ident(), ident(), num()),
        lambda: b"if (err)",
        lambda: b"\treturn err;",
        lambda: b"%s[%s] = %s;" % (ident(), ident(), num()),
        lambda: b"}",
    ]
    tw = np.array([6, 3, 2, 3, 6, 6, 3, 3, 1, 2, 1, 5, 1, 1, 1, 1, 2, 3, 1, 2, 2, 2, 2, 1, 1,
                   4, 3, 2, 2, 3, 6], dtype=float)
    tw /= tw.sum()
    out, total = [], 0
    while total < nbytes:
        f = [b"/*\n * %s.c - %s %s driver\n *\n * Copyright (C) %d %s\n */\n\n"
             % (ident(), ident(), ident(), int(rng.integers(1995, 2012)), ident())]
        for h in rng.choice(len(_C_HEADERS), size=int(rng.integers(3, 13)), replace=False):
            f.append(b"#include <%s>\n" % _C_HEADERS[h])
        f.append(b"\n")
        for _ in range(int(rng.integers(1, 6))):
            f.append(b"#define %s %s\n" % (ident().upper(), num()))
        f.append(b"\n")
        for _ in range(int(rng.integers(2, 9))):
            local[:] = [ids[zi[int(rng.integers(0, zi.size))]] for _ in range(int(rng.integers(3, 8)))]
            f.append(b"static %s %s(%s %s, %s %s)\n{\n" % (
                _C_TYPES[int(rng.integers(0, len(_C_TYPES)))], ident(),
                _C_TYPES[int(rng.integers(0, len(_C_TYPES)))], ident(),
                _C_TYPES[int(rng.integers(0, len(_C_TYPES)))], ident()))
            depth = 1
            for t in rng.choice(len(templates), size=int(rng.integers(4, 30)), p=tw):
                s = templates[t]()
                if s == b"}" or s == b"} else {":
                    if depth <= 1:
                        continue
                    depth -= 1
                f.append(b"\t" * depth + s + b"\n")
                if s.endswith(b"{"):
                    depth += 1
                if rng.random() < 0.05:
                    f.append(b"\n")
            while depth > 1:
                depth -= 1
                f.append(b"\t" * depth + b"}\n")
            f.append(b"}\n\n")
        blob = b"".join(f)
        out.append(blob)
        total += len(blob)
    return b"".join(out)[:nbytes]


def _binary_records(rng, nbytes: int) -> bytes:
    kind = int(rng.integers(0, 4))
    if kind == 0:   # little-endian u32 counters with slowly varying deltas
        start = int(rng.integers(0, 1 << 20))
        delta = np.cumsum(rng.integers(0, 3, size=nbytes // 4 + 1)) + start
        return delta.astype("<u4").tobytes()[:nbytes]
    if kind == 1:   # repeated 16-byte records with a changing field
        rec = bytearray(rng.integers(0, 256, size=16, dtype=np.uint8).tobytes())
        out = bytearray()
        i = 0
        while len(out) < nbytes:
            rec[0:2] = (i & 0xFFFF).to_bytes(2, "little")
            out += rec
            i += 1
        return bytes(out[:nbytes])
    if kind == 2:   # DE-Map-like raster: row-repeated u8 tiles with a few edits
        width = int(rng.choice([64, 100, 256, 512]))
        row = np.repeat(rng.integers(0, 8, size=width // 8 + 1, dtype=np.uint8), 8)[:width]
        rows = []
        for _ in range(nbytes // width + 1):
            if rng.random() < 0.3:
                row = row.copy()
                j = int(rng.integers(0, width))
                row[j:j + 8] = int(rng.integers(0, 8))
            rows.append(row)
        return np.concatenate(rows).tobytes()[:nbytes]
    # sparse table: mostly zero u32 with occasional values
    t = np.zeros(nbytes // 4 + 1, dtype="<u4")
    nz = rng.random(t.size) < 0.1
    t[nz] = rng.integers(0, 1 << 16, size=int(nz.sum()))
    return t.tobytes()[:nbytes]


def _tar_header(rng, name: bytes, size: int) -> bytes:
    h = bytearray(512)
    h[0:len(name[:99])] = name[:99]
    h[100:108] = b"0000644\x00"
    h[108:116] = b"0001750\x00"
    h[116:124] = b"0001750\x00"
    h[124:136] = b"%011o\x00" % size
    h[136:148] = b"%011o\x00" % int(rng.integers(1200000000, 1300000000))
    h[148:156] = b"        "
    h[156] = ord("0")
    h[257:263] = b"ustar\x00"
    h[263:265] = b"00"
    h[265:269] = b"user"
    h[297:302] = b"group"
    h[148:156] = b"%06o\x00 " % (sum(h) & 0o777777)
    return bytes(h)


def _tarmix_base(nbytes: int, seed: int) -> bytes:
    rng = np.random.Generator(np.random.PCG64(seed))
    pools = {
        "c": _csource_base(min(nbytes, 8 << 20), seed + 11),
        "e": _english_base(min(nbytes // 4 + 4096, 2 << 20), seed + 12),
    }
    out, total, k = [], 0, 0
    while total < nbytes:
        size = int(np.exp(rng.uniform(np.log(512), np.log(1 << 20))))
        r = rng.random()
        if r < 0.55:
            src = pools["c"]
            off = int(rng.integers(0, max(1, len(src) - size)))
            body = src[off:off + size]
        elif r < 0.65:
            src = pools["e"]
            off = int(rng.integers(0, max(1, len(src) - size)))
            body = src[off:off + size]
        elif r < 0.80:
            body = _binary_records(rng, size)
        elif r < 0.90:
            body = (b"\x00" if rng.random() < 0.7 else b"\xff") * size
        else:
            body = gen_random(size, int(rng.integers(0, 1 << 30))).tobytes()
        size = len(body)
        name = b"linux-2.6.38/drivers/%s/file%05d.c" % (bytes([97 + k % 26]), k)
        pad = (-size) % 512
        out += [_tar_header(rng, name, size), body, b"\x00" * pad]
        total += 512 + size + pad
        k += 1
    return b"".join(out)[:nbytes]


_BASES = {"english": _english_base, "wordlist": _wordlist_base, "csource": _csource_base,
          "tarmix": _tarmix_base}
_BASE_CAP = {"english": 4 << 20, "wordlist": 4 << 20, "csource": 16 << 20, "tarmix": 64 << 20}


def _segment_plan(base_size: int, n: int, seed: int, seg_lo: int = 1 << 16,
                  seg_hi: int = 1 << 20) -> list:
    """[(pos, off, ln)]: output bytes [pos, pos + ln) = base[off:off + ln]."""
    rng = np.random.Generator(np.random.PCG64(seed ^ 0x5EED))
    plan = []
    pos = 0
    while pos < n:
        ln = min(int(rng.integers(seg_lo, seg_hi + 1)), n - pos, base_size)
        off = int(rng.integers(0, base_size - ln + 1))
        plan.append((pos, off, ln))
        pos += ln
    return plan


def _tile_segments(base: np.ndarray, n: int, seed: int) -> np.ndarray:
    out = np.empty(n, dtype=np.uint8)
    for pos, off, ln in _segment_plan(base.size, n, seed):
        out[pos:pos + ln] = base[off:off + ln]
    return out


def _clip_plan(plan, b0: int, b1: int):
    """The plan's pieces that fall in [b0, b1), as (dst, src_off, ln) with dst
    relative to b0."""
    for pos, off, ln in plan:
        lo, hi = max(pos, b0), min(pos + ln, b1)
        if lo < hi:
            yield lo - b0, off + (lo - pos), hi - lo


def generate(kind: str, n: int, seed: int = 1) -> np.ndarray:
    """n bytes of workload ``kind`` (uint8 numpy array), deterministic in seed."""
    if n < 0:
        raise ValueError("n must be >= 0")
    if kind == "random":
        return gen_random(n, seed)
    if kind == "runs20":
        return gen_runs20(n, seed)
    if kind == "period20":
        return gen_period20(n, seed)
    if kind not in _BASES:
        raise ValueError(f"unknown generator {kind!r}; choose from {GENERATORS}")
    cap = _BASE_CAP[kind]
    base = np.frombuffer(_BASES[kind](min(n, cap), seed), dtype=np.uint8)
    if n <= cap:
        return base[:n].copy()
    return _tile_segments(base, n, seed)


def generate_range(kind: str, n: int, seed: int, b0: int, b1: int) -> np.ndarray:
    """Bytes [b0, b1) of generate(kind, n, seed) without materialising the rest
    where the generator allows it (random: counter-based; tiled corpora: only
    the segments that overlap the range)."""
    if not 0 <= b0 <= b1 <= n:
        raise ValueError("need 0 <= b0 <= b1 <= n")
    if kind == "random":
        w0 = b0 // 8
        with np.errstate(over="ignore"):
            idx = np.arange(w0 + 1, (b1 + 7) // 8 + 1, dtype=np.uint64)
            z = np.uint64(seed) + idx * np.uint64(0x9E3779B97F4A7C15)
            z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
            z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
            z = z ^ (z >> np.uint64(31))
        return z.view(np.uint8)[b0 - 8 * w0:b1 - 8 * w0].copy()
    if kind in _BASES and n > _BASE_CAP[kind]:
        base = np.frombuffer(_BASES[kind](_BASE_CAP[kind], seed), dtype=np.uint8)
        out = np.empty(b1 - b0, dtype=np.uint8)
        for dst, off, ln in _clip_plan(_segment_plan(base.size, n, seed), b0, b1):
            out[dst:dst + ln] = base[off:off + ln]
        return out
    return generate(kind, n, seed)[b0:b1].copy()


_DEV_BASE_CACHE: dict = {}


def generate_range_device(kind: str, n: int, seed: int, b0: int, b1: int, device):
    """generate_range on a CUDA device: tiled corpora upload their base corpus
    once and gather the overlapping segments with device copies (SURVEY
    §8(d): the 64 GiB config is built on the device from a host-made base);
    other kinds are made on the host and uploaded.  Returns a uint8 tensor."""
    import torch
    if kind in _BASES and n > _BASE_CAP[kind]:
        key = (kind, seed, str(device))
        if key not in _DEV_BASE_CACHE:
            base = np.frombuffer(_BASES[kind](_BASE_CAP[kind], seed), dtype=np.uint8)
            _DEV_BASE_CACHE.clear()
            _DEV_BASE_CACHE[key] = torch.from_numpy(base.copy()).to(device)
        dbase = _DEV_BASE_CACHE[key]
        out = torch.empty(b1 - b0, dtype=torch.uint8, device=device)
        for dst, off, ln in _clip_plan(_segment_plan(dbase.numel(), n, seed), b0, b1):
            out[dst:dst + ln].copy_(dbase[off:off + ln])
        return out
    return torch.from_numpy(generate_range(kind, n, seed, b0, b1)).to(device)


# BASELINE.json configs; sizes in bytes.
CONFIGS = {
    "c1_english_64k": dict(kind="english", n=64 << 10, seed=1),
    "c2_csource_128m": dict(kind="csource", n=128 << 20, seed=2),
    "c3_runs20_1g": dict(kind="runs20", n=1 << 30, seed=3),
    "c4_random_1g": dict(kind="random", n=1 << 30, seed=4),
    "c5_tarmix_64g": dict(kind="tarmix", n=64 << 30, seed=5),
}
