"""Randomised parity sweep (GPU): random generator, size, chunk size (packed
and unpacked), window, lookahead and kernel version per case; the stream must
equal the oracle's byte for byte and decode back on the device."""
import numpy as np
import pytest

import oracle as O
from paper_conf_cluster_ozsoys11_b200 import datagen
from test_gpu_parity import dev

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def env():
    import torch
    from paper_conf_cluster_ozsoys11_b200 import build, culzss
    build.build()
    assert culzss.device_count() >= 1
    return torch, culzss


@pytest.mark.parametrize("seed", range(8))
def test_random_cases(env, seed):
    torch, culzss = env
    rng = np.random.default_rng(1000 + seed)
    for _ in range(25):
        kind = str(rng.choice(datagen.GENERATORS))
        n = int(rng.integers(1, 200_000))
        S = int(rng.choice([64, 128, 256, 512, 1024, 2048, 4096, int(rng.integers(1, 4097)),
                            int(rng.integers(4097, 65537))]))
        W = int(rng.integers(1, 257))
        F = int(rng.integers(3, 259))
        version = int(rng.choice([0, 0, 2]))
        # the GPU path's limits: version 2 up to S = 4096 and W = 255;
        # W = 256 needs F <= 256
        if version == 2 and (S > 4096 or W == 256):
            version = 0
        if W == 256:
            F = min(F, 256)
        x = datagen.generate(kind, n, seed=int(rng.integers(0, 1 << 30)))
        p = culzss.Params.make(S=S, W=W, F=F, version=version)
        s = culzss.compress(dev(torch, x), p)
        got = s.cpu().numpy().tobytes()
        assert got == O.compress(x, S=S, W=W, F=F), (kind, n, S, W, F, version)
        y = culzss.decompress(s)
        assert y.cpu().numpy().tobytes() == x.tobytes(), (kind, n, S, W, F, version)
