"""datagen.generate_range: bytes [b0, b1) of generate(kind, n, seed) made
without the rest (the bench builds per-rank slices this way; the device
variant is checked against it in tests/test_gpu_multi_rank.py)."""
import numpy as np
import pytest

from paper_conf_cluster_ozsoys11_b200 import datagen


@pytest.mark.parametrize("kind,n", [("random", 1000003), ("runs20", 100001), ("csource", 3000),
                                    ("english", 70001), ("period20", 4099)])
def test_generate_range_equals_slice(kind, n):
    full = datagen.generate(kind, n, 5)
    for b0, b1 in [(0, n), (7, n - 3), (n // 3, n // 2), (n - 1, n), (5, 5)]:
        np.testing.assert_array_equal(datagen.generate_range(kind, n, 5, b0, b1), full[b0:b1])


def test_generate_range_tiled_corpus():
    """A tiled corpus (n above its base size): only the overlapping segments
    are copied; the bytes equal the whole input's slice."""
    n = (16 << 20) + (3 << 20) + 17  # csource base is 16 MiB
    full = datagen.generate("csource", n, 2)
    for b0, b1 in [(0, n), (123, n - 7), ((16 << 20) - 5, (16 << 20) + 5), (n - 100, n)]:
        np.testing.assert_array_equal(datagen.generate_range("csource", n, 2, b0, b1), full[b0:b1])


def test_generate_range_rejects_bad_ranges():
    with pytest.raises(ValueError):
        datagen.generate_range("random", 10, 1, 5, 11)
    with pytest.raises(ValueError):
        datagen.generate_range("random", 10, 1, 6, 5)
