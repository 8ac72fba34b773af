"""Thin ctypes binding over libculzss.so (include/culzss.h).

Argument marshalling only: every step of the compression path runs in the
library's CUDA kernels.  torch is used for device memory and the current
stream.  If the shared library is missing this module raises on first use --
there is no CPU fallback.
"""
from __future__ import annotations

import ctypes
import struct
import os
from typing import Optional, Tuple

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libculzss.so")

OK, ERR_INVALID_ARG, ERR_UNSUPPORTED, ERR_BUFFER_TOO_SMALL, ERR_CORRUPT, ERR_CUDA, ERR_NO_DEVICE = range(7)

EXPORTS = (
    "culzss_default_params", "culzss_max_compressed_size", "culzss_compress",
    "culzss_compress_host", "culzss_decompressed_size", "culzss_decompress",
    "culzss_compress_chunks", "culzss_compress_chunks_async", "culzss_write_header", "culzss_match_search",
    "culzss_parse_tokens", "culzss_device_count", "culzss_launch_count",
    "culzss_set_profiling", "culzss_last_kernel_ms", "culzss_status_string",
    "culzss_last_cuda_error",
)


class Params(ctypes.Structure):
    """culzss_params: S (chunk), W (window), F (max match), MIN (=3), version."""
    _fields_ = [("chunk_size", ctypes.c_uint32), ("window", ctypes.c_uint16),
                ("max_match", ctypes.c_uint16), ("min_match", ctypes.c_uint8),
                ("version", ctypes.c_uint8), ("reserved", ctypes.c_uint16)]

    @classmethod
    def make(cls, S: int = 4096, W: int = 128, F: int = 128, MIN: int = 3, version: int = 0):
        return cls(S, W, F, MIN, version, 0)


class CulzssError(RuntimeError):
    def __init__(self, status: int, what: str):
        self.status = status
        msg = _lib().culzss_status_string(status).decode()
        if status == ERR_CUDA:
            msg += f" (cudaError {_lib().culzss_last_cuda_error()})"
        super().__init__(f"{what}: {msg} [{status}]")


_L = None


def _lib():
    global _L
    if _L is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} not built; run __graft_entry__.build() "
                              "(there is no CPU fallback)")
        L = ctypes.CDLL(LIB_PATH)
        vp, sz, szp = ctypes.c_void_p, ctypes.c_size_t, ctypes.POINTER(ctypes.c_size_t)
        pp = ctypes.POINTER(Params)
        L.culzss_default_params.argtypes = [pp]
        L.culzss_max_compressed_size.argtypes = [sz, pp]
        L.culzss_max_compressed_size.restype = sz
        for name in ("culzss_compress", "culzss_compress_host"):
            getattr(L, name).argtypes = [vp, sz, vp, szp, pp, vp]
        L.culzss_decompressed_size.argtypes = [vp, sz, szp, vp]
        L.culzss_decompress.argtypes = [vp, sz, vp, szp, pp, vp]
        L.culzss_decompress_host.argtypes = [vp, sz, vp, szp, pp, vp]
        L.culzss_compress_chunks.argtypes = [vp, sz, vp, szp, vp, pp, vp]
        L.culzss_compress_chunks_async.argtypes = [vp, sz, vp, sz, vp, vp, pp, vp]
        L.culzss_decompress_chunks.argtypes = [vp, sz, vp, sz, vp, pp, vp]
        L.culzss_write_header.argtypes = [vp, sz, pp, vp]
        L.culzss_match_search.argtypes = [vp, sz, vp, pp, vp]
        L.culzss_parse_tokens.argtypes = [vp, sz, vp, pp, vp]
        L.culzss_launch_count.restype = ctypes.c_uint64
        L.culzss_set_profiling.argtypes = [ctypes.c_int]
        L.culzss_last_kernel_ms.argtypes = [ctypes.c_char_p]
        L.culzss_last_kernel_ms.restype = ctypes.c_float
        L.culzss_status_string.restype = ctypes.c_char_p
        _L = L
    return _L


def lib():
    """The loaded ctypes CDLL (raises if libculzss.so is missing)."""
    return _lib()


def _params(p: Optional[Params]):
    return ctypes.byref(p) if p is not None else None


def _stream(stream=None) -> ctypes.c_void_p:
    import torch
    s = stream if stream is not None else torch.cuda.current_stream()
    return ctypes.c_void_p(s.cuda_stream)


def _check(st: int, what: str):
    if st != OK:
        raise CulzssError(st, what)


def _dev_u8(x):
    import torch
    if not (isinstance(x, torch.Tensor) and x.is_cuda and x.dtype == torch.uint8 and x.is_contiguous()):
        raise TypeError("expected a contiguous CUDA uint8 tensor")
    return x


def max_compressed_size(n: int, params: Optional[Params] = None) -> int:
    return int(_lib().culzss_max_compressed_size(n, _params(params)))


def device_count() -> int:
    return int(_lib().culzss_device_count())


def launch_count() -> int:
    return int(_lib().culzss_launch_count())


def set_profiling(enable, call_only: bool = False) -> None:
    """enable: per-kernel + call events; call_only: events at the call's start
    and end only (no event between its kernels)."""
    _lib().culzss_set_profiling(0 if not enable else (2 if call_only else 1))


def last_kernel_ms(name: str) -> float:
    return float(_lib().culzss_last_kernel_ms(name.encode()))


def compress_into(x, out, params: Optional[Params] = None, stream=None) -> int:
    """culzss_compress(x -> out); returns the stream length out_n."""
    _dev_u8(x)
    _dev_u8(out)
    on = ctypes.c_size_t(out.numel())
    st = _lib().culzss_compress(ctypes.c_void_p(x.data_ptr()), x.numel(), ctypes.c_void_p(out.data_ptr()),
                                ctypes.byref(on), _params(params), _stream(stream))
    _check(st, "culzss_compress")
    return on.value


def compress(x, params: Optional[Params] = None, stream=None):
    """Compress a CUDA uint8 tensor; returns a CUDA uint8 tensor (the stream)."""
    import torch
    _dev_u8(x)
    out = torch.empty(max_compressed_size(x.numel(), params), dtype=torch.uint8, device=x.device)
    n = compress_into(x, out, params, stream)
    return out[:n]


def compress_host(x: np.ndarray, out: Optional[np.ndarray] = None, params: Optional[Params] = None,
                  stream=None) -> np.ndarray:
    """Host-memory form (H2D + compress + D2H inside the library)."""
    x = np.ascontiguousarray(x, dtype=np.uint8)
    if out is None:
        out = np.empty(max_compressed_size(x.size, params), dtype=np.uint8)
    on = ctypes.c_size_t(out.size)
    st = _lib().culzss_compress_host(ctypes.c_void_p(x.ctypes.data), x.size,
                                     ctypes.c_void_p(out.ctypes.data), ctypes.byref(on),
                                     _params(params), _stream(stream))
    _check(st, "culzss_compress_host")
    return out[: on.value]


def compress_host_ptr(in_ptr: int, n: int, out_ptr: int, cap: int, params: Optional[Params] = None,
                      stream=None) -> int:
    """culzss_compress_host on raw host pointers (e.g. pinned torch tensors)."""
    on = ctypes.c_size_t(cap)
    st = _lib().culzss_compress_host(ctypes.c_void_p(in_ptr), n, ctypes.c_void_p(out_ptr),
                                     ctypes.byref(on), _params(params), _stream(stream))
    _check(st, "culzss_compress_host")
    return on.value


def decompressed_size(s, stream=None) -> int:
    _dev_u8(s)
    n = ctypes.c_size_t(0)
    st = _lib().culzss_decompressed_size(ctypes.c_void_p(s.data_ptr()), s.numel(), ctypes.byref(n),
                                         _stream(stream))
    _check(st, "culzss_decompressed_size")
    return n.value


def decompress_status(s, out=None, stream=None) -> Tuple[int, object]:
    import torch
    _dev_u8(s)
    if out is None:
        st0 = ctypes.c_size_t(0)
        st = _lib().culzss_decompressed_size(ctypes.c_void_p(s.data_ptr()), s.numel(), ctypes.byref(st0),
                                             _stream(stream))
        if st != OK:
            return st, None
        if st0.value > 122 * s.numel() + 1:  # memory guard: a valid stream expands < 122x
            return ERR_CORRUPT, None
        out = torch.empty(max(st0.value, 1), dtype=torch.uint8, device=s.device)
    on = ctypes.c_size_t(out.numel())
    st = _lib().culzss_decompress(ctypes.c_void_p(s.data_ptr()), s.numel(), ctypes.c_void_p(out.data_ptr()),
                                  ctypes.byref(on), None, _stream(stream))
    return st, (out[: on.value] if st == OK else None)


def decompress_host_status(s: np.ndarray, out: Optional[np.ndarray] = None, stream=None) -> Tuple[int, object]:
    """Host-memory decompression (H2D + decode + D2H pipelined inside the library)."""
    s = np.ascontiguousarray(s, dtype=np.uint8)
    if out is None:
        n = struct.unpack_from("<Q", s.tobytes()[16:24])[0] if s.size >= 32 else 0
        if n > 122 * s.size + 1:  # memory guard: a valid stream expands < 122x
            return ERR_CORRUPT, None
        out = np.empty(max(n, 1), dtype=np.uint8)
    on = ctypes.c_size_t(out.size)
    st = _lib().culzss_decompress_host(ctypes.c_void_p(s.ctypes.data), s.size, ctypes.c_void_p(out.ctypes.data),
                                       ctypes.byref(on), None, _stream(stream))
    return st, (out[: on.value] if st == OK else None)


def decompress_host(s: np.ndarray, out: Optional[np.ndarray] = None, stream=None) -> np.ndarray:
    st, o = decompress_host_status(s, out, stream)
    _check(st, "culzss_decompress_host")
    return o


def decompress_host_ptr(in_ptr: int, in_n: int, out_ptr: int, cap: int, stream=None) -> int:
    """culzss_decompress_host on raw host pointers (e.g. pinned torch tensors)."""
    on = ctypes.c_size_t(cap)
    st = _lib().culzss_decompress_host(ctypes.c_void_p(in_ptr), in_n, ctypes.c_void_p(out_ptr), ctypes.byref(on),
                                       None, _stream(stream))
    _check(st, "culzss_decompress_host")
    return on.value


def decompress(s, out=None, stream=None):
    st, o = decompress_status(s, out, stream)
    _check(st, "culzss_decompress")
    return o


def _check_table_len(chunk_sizes, slice_n: int, params) -> None:
    """The kernels write / read ceil(slice_n / S) entries of chunk_sizes: a
    shorter tensor would be an out-of-bounds device access."""
    S = params.chunk_size if params is not None else 4096
    need = (slice_n + S - 1) // S if S else 0
    if chunk_sizes.numel() < need or not chunk_sizes.is_contiguous():
        raise ValueError(f"chunk_sizes must be a contiguous tensor of >= ceil(slice_n/S) = {need} entries")


def compress_chunks(x_slice, payload, chunk_sizes, params: Optional[Params] = None, stream=None) -> int:
    """Sharding primitive: payload only (no header/table); returns payload bytes."""
    import torch
    _dev_u8(x_slice)
    _dev_u8(payload)
    if not (chunk_sizes.is_cuda and chunk_sizes.dtype == torch.int32):
        raise TypeError("chunk_sizes must be a CUDA int32 tensor (u32 bit pattern)")
    _check_table_len(chunk_sizes, x_slice.numel(), params)
    pn = ctypes.c_size_t(payload.numel())
    st = _lib().culzss_compress_chunks(ctypes.c_void_p(x_slice.data_ptr()), x_slice.numel(),
                                       ctypes.c_void_p(payload.data_ptr()), ctypes.byref(pn),
                                       ctypes.c_void_p(chunk_sizes.data_ptr()), _params(params),
                                       _stream(stream))
    _check(st, "culzss_compress_chunks")
    return pn.value


def compress_chunks_async(x_slice, payload, chunk_sizes, dev_total, params: Optional[Params] = None,
                          stream=None) -> None:
    """Sharding primitive without a host sync: the payload total goes to the
    CUDA int64 tensor dev_total[0] (stream-ordered) for a device all-gather."""
    import torch
    _dev_u8(x_slice)
    _dev_u8(payload)
    if not (chunk_sizes.is_cuda and chunk_sizes.dtype == torch.int32):
        raise TypeError("chunk_sizes must be a CUDA int32 tensor (u32 bit pattern)")
    if not (dev_total.is_cuda and dev_total.dtype == torch.int64 and dev_total.numel() >= 1):
        raise TypeError("dev_total must be a CUDA int64 tensor")
    _check_table_len(chunk_sizes, x_slice.numel(), params)
    _check(_lib().culzss_compress_chunks_async(ctypes.c_void_p(x_slice.data_ptr()), x_slice.numel(),
                                               ctypes.c_void_p(payload.data_ptr()), payload.numel(),
                                               ctypes.c_void_p(chunk_sizes.data_ptr()),
                                               ctypes.c_void_p(dev_total.data_ptr()), _params(params),
                                               _stream(stream)), "culzss_compress_chunks_async")


def decompress_chunks_status(payload, chunk_sizes, slice_n: int, out=None, params: Optional[Params] = None,
                             stream=None) -> Tuple[int, object]:
    """Sharded decompression (inverse of compress_chunks): decode the
    ceil(slice_n/S) chunks of `payload` (CUDA uint8) sized by `chunk_sizes`
    (CUDA int32, u32 bit pattern) into `out` (CUDA uint8, slice_n bytes)."""
    import torch
    _dev_u8(payload)
    if not (chunk_sizes.is_cuda and chunk_sizes.dtype == torch.int32):
        raise TypeError("chunk_sizes must be a CUDA int32 tensor (u32 bit pattern)")
    _check_table_len(chunk_sizes, slice_n, params)
    if out is None:
        out = torch.empty(max(slice_n, 1), dtype=torch.uint8, device=payload.device)
    _dev_u8(out)
    if out.numel() < slice_n:
        raise ValueError("out is smaller than slice_n")
    st = _lib().culzss_decompress_chunks(ctypes.c_void_p(payload.data_ptr()), payload.numel(),
                                         ctypes.c_void_p(chunk_sizes.data_ptr()), slice_n,
                                         ctypes.c_void_p(out.data_ptr()), _params(params), _stream(stream))
    return st, (out[:slice_n] if st == OK else None)


def decompress_chunks(payload, chunk_sizes, slice_n: int, out=None, params: Optional[Params] = None, stream=None):
    st, o = decompress_chunks_status(payload, chunk_sizes, slice_n, out, params, stream)
    _check(st, "culzss_decompress_chunks")
    return o


def write_header(out, n_total: int, params: Optional[Params] = None, stream=None) -> None:
    _dev_u8(out)
    _check(_lib().culzss_write_header(ctypes.c_void_p(out.data_ptr()), n_total, _params(params),
                                      _stream(stream)), "culzss_write_header")


def match_search(x, params: Optional[Params] = None, stream=None):
    """Per-position (L, D) for every position of every chunk (row a2)."""
    import torch
    _dev_u8(x)
    LD = torch.zeros(2 * max(x.numel(), 1), dtype=torch.uint8, device=x.device)
    _check(_lib().culzss_match_search(ctypes.c_void_p(x.data_ptr()), x.numel(), ctypes.c_void_p(LD.data_ptr()),
                                      _params(params), _stream(stream)), "culzss_match_search")
    LD = LD[: 2 * x.numel()].view(-1, 2)
    L, D = LD[:, 0], LD[:, 1].to(torch.int16)
    return L, torch.where((L >= 3) & (D == 0), torch.full_like(D, 256), D)  # D byte 0 beside a match: D = 256


def parse_tokens(x, params: Optional[Params] = None, stream=None):
    """Per-position greedy-parse tokens (row a3): 0 inside a match, 1 literal,
    (L << 16) | D match start."""
    import torch
    _dev_u8(x)
    tok = torch.zeros(max(x.numel(), 1), dtype=torch.int32, device=x.device)
    _check(_lib().culzss_parse_tokens(ctypes.c_void_p(x.data_ptr()), x.numel(), ctypes.c_void_p(tok.data_ptr()),
                                      _params(params), _stream(stream)), "culzss_parse_tokens")
    return tok[: x.numel()]
