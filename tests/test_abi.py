"""CPU-side checks of the boundary: the C-ABI library builds, loads and
exports every symbol include/culzss.h declares; host-only entry points work
without a GPU; compute entry points fail loudly (no CPU fallback)."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "culzss.h")


@pytest.fixture(scope="module")
def culzss():
    from paper_conf_cluster_ozsoys11_b200 import build
    build.build()
    from paper_conf_cluster_ozsoys11_b200 import culzss as c
    return c


def header_symbols():
    txt = open(HEADER).read()
    return sorted(set(re.findall(r"CULZSS_API\s+[\w\s\*]*?\b(culzss_\w+)\s*\(", txt)))


def test_header_declares_expected_entry_points():
    syms = header_symbols()
    for s in ("culzss_compress", "culzss_decompress", "culzss_compress_chunks", "culzss_write_header",
              "culzss_max_compressed_size", "culzss_default_params", "culzss_status_string",
              "culzss_match_search", "culzss_parse_tokens", "culzss_compress_host",
              "culzss_decompress_chunks", "culzss_decompress_host"):
        assert s in syms


def test_library_exports_every_header_symbol(culzss):
    out = subprocess.run(["nm", "-D", "--defined-only", culzss.LIB_PATH], capture_output=True,
                         text=True, check=True).stdout
    exported = set(re.findall(r"\bT (culzss_\w+)", out))
    missing = [s for s in header_symbols() if s not in exported]
    assert not missing, missing
    assert set(culzss.EXPORTS) <= exported
    L = culzss.lib()
    for s in header_symbols():
        assert getattr(L, s) is not None


def test_sm100a_code_only(culzss):
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", culzss.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out
    assert not re.search(r"sm_(?!100a)\d+", out), out


def test_host_only_entry_points(culzss):
    p = culzss.Params()
    culzss.lib().culzss_default_params(ctypes.byref(p))
    assert (p.chunk_size, p.window, p.max_match, p.min_match, p.version) == (4096, 128, 128, 3, 0)
    import oracle
    for n in (0, 1, 4095, 4096, 4097, 1 << 20):
        assert culzss.max_compressed_size(n) == oracle.max_compressed_size(n)
    assert culzss.lib().culzss_status_string(4) == b"corrupt stream"


def test_no_cpu_fallback_without_device(culzss):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    assert culzss.device_count() == 0
    on = ctypes.c_size_t(1 << 20)
    buf = (ctypes.c_uint8 * 64)()
    st = culzss.lib().culzss_compress(ctypes.cast(buf, ctypes.c_void_p), 64, ctypes.cast(buf, ctypes.c_void_p),
                                      ctypes.byref(on), None, None)
    assert st == culzss.ERR_NO_DEVICE
    sizes = (ctypes.c_uint32 * 1)()
    st = culzss.lib().culzss_decompress_chunks(ctypes.cast(buf, ctypes.c_void_p), 8, ctypes.cast(sizes, ctypes.c_void_p),
                                               64, ctypes.cast(buf, ctypes.c_void_p), None, None)
    assert st == culzss.ERR_NO_DEVICE


def test_product_path_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_cluster_ozsoys11_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".h", ".cuh")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt, f
                assert "culzss_oracle" not in txt and "liboracle" not in txt, f
