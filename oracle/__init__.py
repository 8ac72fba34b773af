"""CPU oracle for chunked LZSS (CULZSS, Ozsoy & Swany, CLUSTER 2011).

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  The product path (``paper_conf_cluster_ozsoys11_b200``) never
imports it and shares no code with it.

This module is argument marshalling over ``culzss_oracle.c`` (plain C, built
with gcc ``-O2``, no intrinsics).  Every definition lives in the C file, which
cites the PAPER.md passages it follows.  Parity status is listed in the C
file header and in DESIGN.md §3: every function is pinned by
``tests/test_oracle_*.py``.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import List, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "culzss_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

OK, ERR_INVALID_ARG, ERR_BUFFER_TOO_SMALL, ERR_CORRUPT = 0, 1, 3, 4
HEADER_BYTES = 32
DEFAULT = dict(S=4096, W=128, F=128, MIN=3)


def build(force: bool = False) -> str:
    """Compile culzss_oracle.c -> liboracle.so (gcc -O2, no intrinsics)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        u8p = ctypes.c_void_p
        L.oracle_match_at.argtypes = [u8p, ctypes.c_size_t, ctypes.c_size_t, ctypes.c_uint32,
                                      ctypes.c_uint32, ctypes.c_uint32,
                                      ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint32)]
        L.oracle_match_all.argtypes = [u8p, ctypes.c_size_t, ctypes.c_uint32, ctypes.c_uint32,
                                       ctypes.c_uint32, u8p, u8p]
        L.oracle_tokens_chunk.argtypes = [u8p, ctypes.c_size_t, ctypes.c_uint32, ctypes.c_uint32,
                                          ctypes.c_uint32, u8p]
        L.oracle_tokens_chunk.restype = ctypes.c_size_t
        L.oracle_compress_chunk.argtypes = [u8p, ctypes.c_size_t, ctypes.c_uint32, ctypes.c_uint32,
                                            ctypes.c_uint32, u8p]
        L.oracle_compress_chunk.restype = ctypes.c_size_t
        L.oracle_max_compressed_size.argtypes = [ctypes.c_uint64, ctypes.c_uint32]
        L.oracle_max_compressed_size.restype = ctypes.c_uint64
        L.oracle_compress.argtypes = [u8p, ctypes.c_uint64, u8p, ctypes.POINTER(ctypes.c_uint64),
                                      ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32]
        L.oracle_compress_range.argtypes = [u8p, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64,
                                            u8p, ctypes.POINTER(ctypes.c_uint64), u8p,
                                            ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32,
                                            ctypes.c_uint32]
        L.oracle_decompress.argtypes = [u8p, ctypes.c_uint64, u8p, ctypes.POINTER(ctypes.c_uint64)]
        L.oracle_decompressed_size.argtypes = [u8p, ctypes.c_uint64, ctypes.POINTER(ctypes.c_uint64)]
        L.oracle_params_valid.argtypes = [ctypes.c_uint32] * 4
        _lib = L
    return _lib


def _u8(data) -> np.ndarray:
    if isinstance(data, (bytes, bytearray, memoryview)):
        a = np.frombuffer(bytes(data), dtype=np.uint8)
    else:
        a = np.ascontiguousarray(data, dtype=np.uint8)
    if a.size == 0:
        a = np.zeros(1, dtype=np.uint8)[:0]
    return a


def _ptr(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data) if a.size else ctypes.c_void_p(0)


def max_compressed_size(n: int, S: int = 4096) -> int:
    return int(lib().oracle_max_compressed_size(n, S))


def match_at(chunk, p: int, W=128, F=128, MIN=3) -> Tuple[int, int]:
    a = _u8(chunk)
    L, D = ctypes.c_uint32(), ctypes.c_uint32()
    lib().oracle_match_at(_ptr(a), a.size, p, W, F, MIN, ctypes.byref(L), ctypes.byref(D))
    return L.value, D.value


def match_all(chunk, W=128, F=128, MIN=3) -> Tuple[np.ndarray, np.ndarray]:
    a = _u8(chunk)
    L = np.zeros(max(a.size, 1), dtype=np.uint16)
    D = np.zeros(max(a.size, 1), dtype=np.uint16)
    lib().oracle_match_all(_ptr(a), a.size, W, F, MIN, _ptr(L), _ptr(D))
    return L[: a.size], D[: a.size]


def tokens_chunk(chunk, W=128, F=128, MIN=3) -> List[tuple]:
    """Greedy-parse tokens: ('L', byte) or ('M', D, L)."""
    a = _u8(chunk)
    tok = np.zeros(max(a.size, 1), dtype=np.uint32)
    nt = lib().oracle_tokens_chunk(_ptr(a), a.size, W, F, MIN, _ptr(tok))
    out = []
    for t in tok[:nt].tolist():
        if t & 0x80000000:
            out.append(("M", (t >> 16) & 0x7FFF, t & 0xFFFF))
        else:
            out.append(("L", t & 0xFF))
    return out


def compress_chunk(chunk, W=128, F=128, MIN=3) -> bytes:
    a = _u8(chunk)
    out = np.zeros((9 * a.size + 7) // 8 + 8, dtype=np.uint8)
    sz = lib().oracle_compress_chunk(_ptr(a), a.size, W, F, MIN, _ptr(out))
    return out[:sz].tobytes()


def compress(data, S=4096, W=128, F=128, MIN=3) -> bytes:
    a = _u8(data)
    cap = max_compressed_size(a.size, S)
    out = np.zeros(cap, dtype=np.uint8)
    on = ctypes.c_uint64(cap)
    st = lib().oracle_compress(_ptr(a), a.size, _ptr(out), ctypes.byref(on), S, W, F, MIN)
    if st != OK:
        raise ValueError(f"oracle_compress status {st}")
    return out[: on.value].tobytes()


def compress_range(data, c0: int, c1: int, S=4096, W=128, F=128, MIN=3):
    """Payload bytes + u32 sizes of chunks [c0, c1) (no header / table)."""
    a = _u8(data)
    nchunks = c1 - c0
    out = np.zeros(nchunks * ((9 * S + 7) // 8) + 8, dtype=np.uint8)
    sizes = np.zeros(max(nchunks, 1), dtype=np.uint32)
    pn = ctypes.c_uint64(0)
    st = lib().oracle_compress_range(_ptr(a), a.size, c0, c1, _ptr(out), ctypes.byref(pn),
                                     _ptr(sizes), S, W, F, MIN)
    if st != OK:
        raise ValueError(f"oracle_compress_range status {st}")
    return out[: pn.value].tobytes(), sizes[:nchunks].copy()


def decompress_status(stream) -> Tuple[int, bytes]:
    a = _u8(stream)
    n = ctypes.c_uint64(0)
    st = lib().oracle_decompressed_size(_ptr(a), a.size, ctypes.byref(n))
    if st != OK:
        return st, b""
    # Memory guard only: a match token (17 bits) yields at most 258 bytes, so a
    # valid stream never expands more than 258*8/17 < 122x.
    if n.value > 122 * a.size + 1:
        return ERR_CORRUPT, b""
    out = np.zeros(max(n.value, 1), dtype=np.uint8)
    on = ctypes.c_uint64(n.value)
    st = lib().oracle_decompress(_ptr(a), a.size, _ptr(out), ctypes.byref(on))
    return st, (out[: on.value].tobytes() if st == OK else b"")


def decompress(stream) -> bytes:
    st, out = decompress_status(stream)
    if st != OK:
        raise ValueError(f"oracle_decompress status {st}")
    return out


def params_valid(S=4096, W=128, F=128, MIN=3) -> bool:
    return bool(lib().oracle_params_valid(S, W, F, MIN))
