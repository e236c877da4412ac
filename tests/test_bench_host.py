"""Host-side logic of bench.py (CPU only): the 95% confidence interval of the paper's
10-run protocol against scipy's Student t interval, the strong-scaling slices, the
configs' shapes, and the range-sharded CPU baseline on a small config."""
import numpy as np
import pytest

import bench


def test_ci95_matches_student_t():
    from scipy import stats
    rng = np.random.default_rng(1)
    for n in (2, 3, 5, 10, 16):
        xs = list(rng.normal(100, 5, n))
        m, h = bench.ci95(xs)
        lo, hi = stats.t.interval(0.95, n - 1, loc=np.mean(xs), scale=stats.sem(xs))
        assert abs(m - np.mean(xs)) < 1e-9
        assert abs(h - (hi - lo) / 2) < 1e-3 * (hi - lo)
    assert bench.ci95([3.0])[1] is None


@pytest.mark.parametrize("n,w", [(125_000_000, 8), (10, 3), (0, 4), (7, 8), (625_000, 2)])
def test_strong_scaling_slices_partition_the_batch(n, w):
    sl = bench.slices(n, w)
    assert len(sl) == w and sl[0][0] == 0 and sl[-1][1] == n
    assert all(a <= b for a, b in sl) and all(sl[i][1] == sl[i + 1][0] for i in range(w - 1))
    sizes = [b - a for a, b in sl]
    assert max(sizes) - min(sizes) <= 1


def test_configs_follow_baseline_json():
    """BASELINE.json configs[0..4] = C1 .. C5."""
    R, pre, B, nb, mix, dist, N = bench.CONFIGS["C5"]
    assert (R, pre, mix, dist) == (1_000_000_000, 500_000_000, (10, 10, 80), "uniform")
    assert B * nb == 1_000_000_000  # 1B ops
    assert bench.CONFIGS["C1"][:2] == (10_000, 5_000) and bench.CONFIGS["C1"][2] * bench.CONFIGS["C1"][3] == 100_000
    assert bench.CONFIGS["C4-16"][4] == (0, 0, 100) and bench.CONFIGS["C4-32"][6] == 32
    ins = bench.CONFIGS["INS-1M"]
    assert ins[1] == 0 and ins[2] * ins[3] == ins[0]          # R inserts from empty
    dele = bench.CONFIGS["DEL-1M"]
    assert dele[1] == dele[0] and dele[2] * dele[3] == dele[0]  # R deletes from full


def test_range_sharded_cpu_baseline_runs():
    r = bench.oracle_sample("C1", 3, 1, budget_s=5.0, threads=4)
    assert r["threads"] == 4 and r["mops"] > 0 and r["batches"] >= 1
    r1 = bench.oracle_sample("C1", 3, 1, budget_s=5.0, threads=1)
    assert r1["threads"] == 1 and r1["mops"] > 0


def test_c5_shard_configs_are_the_strong_scaled_slices():
    """C5-S<G> is what one rank of `--gpus G --config C5` holds and runs: R/G keys in its
    local key space, its share of the prefill, a 1/G slice of every global batch, the same
    mix, distribution and chunk size."""
    import bench
    R, pre, B, nb, mix, dist, N = bench.CONFIGS["C5"]
    for G in (2, 4, 8):
        r, p, b, n, m, di, c = bench.CONFIGS[f"C5-S{G}"]
        assert (r, p, b) == (R // G, pre // G, B // G)
        assert (n, m, di, c) == (nb, mix, dist, N)
