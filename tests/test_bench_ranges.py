"""bench.py's per-rank inputs (CPU): under strong scaling (the default: the
config's input split over the N ranks, as BASELINE.json states "1 GB ... on 1
and 8 B200", "64 GB ... sharded across 2/4/8 B200") the ranks' byte ranges are
chunk-aligned, contiguous and cover the input exactly; c5 at N = 1 is rank 0's
slice of a dp8 split; weak scaling gives every rank a config-sized input."""
import importlib.util
import os

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
spec = importlib.util.spec_from_file_location("bench", os.path.join(ROOT, "bench.py"))
bench = importlib.util.module_from_spec(spec)
spec.loader.exec_module(bench)


@pytest.mark.parametrize("cfg", ["c2_csource_128m", "c3_runs20_1g", "c4_random_1g", "c5_tarmix_64g"])
@pytest.mark.parametrize("world", [2, 3, 4, 8])
def test_strong_ranges_partition_the_input(cfg, world):
    spec = bench.datagen.CONFIGS[cfg]
    pos = 0
    for r in range(world):
        n, seed, b0, b1 = bench.rank_range(cfg, r, world, "strong")
        assert (n, seed) == (spec["n"], spec["seed"])
        assert b0 == pos and b0 % 4096 == 0 and b1 >= b0
        pos = b1
    assert pos == spec["n"]


def test_c5_single_gpu_is_rank0_of_dp8():
    n, seed, b0, b1 = bench.rank_range("c5_tarmix_64g", 0, 1, "strong")
    assert (b0, b1) == bench.rank_range("c5_tarmix_64g", 0, 8, "strong")[2:]
    assert b1 - b0 == (64 << 30) // 8


@pytest.mark.parametrize("cfg", ["c3_runs20_1g", "c4_random_1g"])
def test_weak_ranges_are_config_sized(cfg):
    spec = bench.datagen.CONFIGS[cfg]
    seeds = set()
    for r in range(4):
        n, seed, b0, b1 = bench.rank_range(cfg, r, 4, "weak")
        assert (b0, b1, n) == (0, spec["n"], spec["n"])
        seeds.add(seed)
    assert len(seeds) == 4  # independent inputs


def test_roofline_terms():
    """The compare count of a full chunk: 516,032 byte-pair tests."""
    assert bench.chunk_pairs(4096) == 516032
    assert bench.chunk_pairs(3 * 4096 + 5) == 3 * 516032 + sum(min(128, p) for p in range(5))
    rf = bench.roofline(4096 * 1000, 1000, 1000 * 600, 1.0, 18.5, 6500.0)
    assert rf["bound"] in ("alu", "hbm") and 0 < rf["frac"]
