"""GPU parity of the chunk kernel's two walk machines, each on its own and in
the default switching mode (machine 1 is the plain chain walk,
machine 2 adds the exact run-skip and chain-switch prunes; a warp switches
when one lane spends CULZSS_WALK_TOKEN_SWITCH iterations on one token).

The prunes only change which candidates are visited, never the result, so
every (L, D), every token and every stream byte must equal the oracle's under
every setting.  Inputs target the prunes: runs of equal bytes of many lengths
(around the window W, the cap F and t = the run at the parse position),
periodic records with short matches (LE counters: long chains of true
3-gram candidates), and the structured-binary part of the tarball mix.
"""
import functools
import os

import numpy as np
import pytest

import oracle as O
from paper_conf_cluster_ozsoys11_b200 import datagen

pytestmark = pytest.mark.gpu

MACHINES = {
    "machine1_only": {"CULZSS_WALK_TOKEN_SWITCH": "1000000000", "CULZSS_WALK_SWITCH": "1000000000"},
    "machine2_only": {"CULZSS_WALK_TOKEN_SWITCH": "0"},
    "switch_after_3": {"CULZSS_WALK_TOKEN_SWITCH": "3"},
    "default": {},
}


@pytest.fixture(scope="module")
def env():
    import torch
    from paper_conf_cluster_ozsoys11_b200 import build, culzss
    build.build()
    assert culzss.device_count() >= 1
    return torch, culzss


@pytest.fixture(params=sorted(MACHINES))
def machine(request):
    keys = ("CULZSS_WALK_TOKEN_SWITCH", "CULZSS_WALK_SWITCH")
    old = {k: os.environ.get(k) for k in keys}
    for k in keys:
        os.environ.pop(k, None)
    os.environ.update(MACHINES[request.param])
    yield request.param
    for k, v in old.items():
        if v is None:
            os.environ.pop(k, None)
        else:
            os.environ[k] = v


def dev(torch, a):
    a = np.ascontiguousarray(a, dtype=np.uint8)
    return torch.from_numpy(a.copy()).cuda()


@functools.lru_cache(maxsize=1)
def run_inputs():
    """Inputs aimed at the run skip and the chain switch."""
    rng = np.random.default_rng(2024)
    cases = {}
    # runs of one length from a small alphabet: earlier same-letter runs in the window
    for L in (3, 4, 5, 8, 19, 20, 21, 60, 127, 128, 129, 200, 300):
        for k in (2, 3, 26):
            letters = rng.integers(0, k, 3 * 4096 // L + 2, dtype=np.uint8) + 97
            cases[f"runs{L}_alpha{k}"] = np.repeat(letters, L)[:3 * 4096 + 77]
    # runs of random lengths (1..150), two letters
    lens = rng.integers(1, 150, 2000)
    cases["runs_rand2"] = np.repeat(rng.integers(0, 2, 2000, dtype=np.uint8), lens)[:5 * 4096]
    # runs separated by short noise
    parts = []
    for _ in range(600):
        parts.append(np.full(int(rng.integers(4, 40)), int(rng.integers(0, 3)), np.uint8))
        parts.append(rng.integers(0, 256, int(rng.integers(0, 4)), dtype=np.uint8))
    cases["runs_noise"] = np.concatenate(parts)[:4 * 4096]
    # LE u32 counters with small steps (true 3-gram chains, short matches)
    for step in (1, 2, 3):
        v = np.cumsum(rng.integers(0, step + 1, 5000)) + 0x0F2100
        cases[f"counters_step{step}"] = v.astype("<u4").view(np.uint8)[:4 * 4096]
    # 16-byte records with a changing field; 2-byte fields
    rec = rng.integers(0, 256, 16, dtype=np.uint8)
    recs = np.tile(rec, 1100).reshape(-1, 16)
    recs[:, 0] = np.arange(recs.shape[0]) & 0xFF
    cases["records16"] = recs.reshape(-1)[:4 * 4096]
    cases["u16_ramp"] = (np.arange(9000) // 3).astype("<u2").view(np.uint8)[:4 * 4096 + 9]
    # zero runs with sparse values (sparse tables)
    t = np.zeros(5000, "<u4")
    nz = rng.random(5000) < 0.1
    t[nz] = rng.integers(0, 1 << 16, int(nz.sum()))
    cases["sparse_u32"] = t.view(np.uint8)[:4 * 4096]
    # the tarball mix and runs20 as generated
    cases["tarmix"] = datagen.generate("tarmix", 6 * 4096 + 555, seed=21)
    cases["runs20"] = datagen.generate("runs20", 4 * 4096 + 13, seed=22)
    return cases


@pytest.mark.parametrize("W,F", [(128, 128), (128, 20), (64, 128), (255, 258), (16, 10)])
def test_streams_each_machine(env, machine, W, F):
    """Byte-exact streams against the oracle under each walk machine."""
    torch, culzss = env
    p = culzss.Params.make(W=W, F=F)
    for name, x in run_inputs().items():
        got = culzss.compress(dev(torch, x), p).cpu().numpy().tobytes()
        assert got == O.compress(x, W=W, F=F), (machine, name, W, F)


@pytest.mark.parametrize("W,F", [(128, 128), (64, 32), (255, 255)])
def test_match_search_each_machine(env, machine, W, F):
    """Row a2 through the production walk machines (the dump mode evaluates
    every candidate position with the same code): (L, D) at every position."""
    torch, culzss = env
    p = culzss.Params.make(W=W, F=F)
    for name, x in run_inputs().items():
        x = x[:2 * 4096 + 100]
        L, D = culzss.match_search(dev(torch, x), p)
        L, D = L.cpu().numpy(), D.cpu().numpy()
        for c in range((x.size + 4095) // 4096):
            chunk = x[c * 4096:(c + 1) * 4096]
            eL, eD = O.match_all(chunk, W=W, F=F)
            np.testing.assert_array_equal(L[c * 4096:c * 4096 + chunk.size], eL, err_msg=f"{machine} {name}")
            np.testing.assert_array_equal(D[c * 4096:c * 4096 + chunk.size], eD, err_msg=f"{machine} {name}")


def test_packed_small_chunks_each_machine(env, machine):
    """Packed chunks (S < 4096): the window limit and run queries stop at each
    small chunk's start."""
    torch, culzss = env
    for S in (64, 256, 1024):
        p = culzss.Params.make(S=S)
        for name in ("runs20", "tarmix", "counters_step1", "runs_rand2"):
            x = run_inputs()[name]
            got = culzss.compress(dev(torch, x), p).cpu().numpy().tobytes()
            assert got == O.compress(x, S=S), (machine, name, S)


@pytest.mark.parametrize("F", [3, 20, 128, 256])
def test_window_256_streams(env, machine, F):
    """W = 256 (PAPER.md:1@23151 §III.D "offsets are upto 256"): the u8 links
    hold distances <= 255 and the walk evaluates d = 256 as one extra
    candidate; byte-exact streams against the oracle, both machines."""
    torch, culzss = env
    p = culzss.Params.make(W=256, F=F)
    rng = np.random.default_rng(256)
    cases = dict(run_inputs())
    for per in (127, 128, 200, 255, 256, 257):  # matches exactly at the window edge
        base = rng.integers(0, 256, per, dtype=np.uint8)
        cases[f"period{per}"] = np.tile(base, 3 * 4096 // per + 2)[:3 * 4096 + 11]
    cases["csource"] = datagen.generate("csource", 3 * 4096 + 5, seed=31)
    cases["random"] = datagen.generate("random", 2 * 4096, seed=32)
    for name, x in cases.items():
        got = culzss.compress(dev(torch, x), p).cpu().numpy().tobytes()
        assert got == O.compress(x, W=256, F=F), (machine, name, F)


def test_window_256_match_search(env, machine):
    """Row a2 at W = 256: (L, D) at every position, including D = 256."""
    torch, culzss = env
    p = culzss.Params.make(W=256, F=200)
    rng = np.random.default_rng(257)
    xs = [np.tile(rng.integers(0, 256, 256, dtype=np.uint8), 20)[:2 * 4096 + 50],
          datagen.generate("tarmix", 2 * 4096 + 9, seed=33), run_inputs()["runs20_alpha3"][:8192]]
    seen256 = False
    for x in xs:
        L, D = culzss.match_search(dev(torch, x), p)
        L, D = L.cpu().numpy(), D.cpu().numpy()
        for c in range((x.size + 4095) // 4096):
            chunk = x[c * 4096:(c + 1) * 4096]
            eL, eD = O.match_all(chunk, W=256, F=200)
            np.testing.assert_array_equal(L[c * 4096:c * 4096 + chunk.size], eL, err_msg=machine)
            np.testing.assert_array_equal(D[c * 4096:c * 4096 + chunk.size], eD, err_msg=machine)
            seen256 |= bool((eD == 256).any())
    assert seen256  # the period-256 input exercises d = 256


def test_window_256_packed_and_roundtrip(env, machine):
    torch, culzss = env
    for S in (512, 1024, 2048, 1000):
        p = culzss.Params.make(S=S, W=256, F=256)
        for name in ("runs20", "tarmix", "counters_step2"):
            x = run_inputs()[name]
            s = culzss.compress(dev(torch, x), p)
            assert s.cpu().numpy().tobytes() == O.compress(x, S=S, W=256, F=256), (machine, name, S)
            assert culzss.decompress(s).cpu().numpy().tobytes() == x.tobytes()


def test_window_256_limits(env):
    """W = 256 with F > 256 (the 16-bit token memo's code space) and version 2
    at W = 256 are UNSUPPORTED; both stay valid parameters (INVALID_ARG is
    for W > 256 / F > 258)."""
    torch, culzss = env
    x = dev(torch, datagen.generate("english", 5000, seed=1))
    for kw in (dict(W=256, F=257), dict(W=256, F=258), dict(W=256, version=2)):
        with pytest.raises(culzss.CulzssError) as e:
            culzss.compress(x, culzss.Params.make(**kw))
        assert e.value.status == culzss.ERR_UNSUPPORTED, kw
    with pytest.raises(culzss.CulzssError) as e:
        culzss.compress(x, culzss.Params.make(W=257))
    assert e.value.status == culzss.ERR_INVALID_ARG
