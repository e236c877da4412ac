"""The seeded generator: determinism, exact mixes, the <=1-mutation-per-key contract,
prefill permutations and Zipf skew (CPU)."""
import torch

from paper_conf_ppopp_moscovicicp17_b200.workload import (
    SEED_BASE, Workload, feistel_perm, prefill_keys, uniform_key)


def test_deterministic_and_exact_mix():
    w = Workload(100_000, 10_000, mix=(20, 20, 60))
    a = w.make_batch(3)
    b = w.make_batch(3)
    for x, y in zip(a[:3], b[:3]):
        assert torch.equal(x, y)
    op = a[0]
    assert int((op == 1).sum()) == 2000 and int((op == 2).sum()) == 2000
    c = w.make_batch(4)
    assert not torch.equal(a[1], c[1])


def test_contract_no_duplicate_mutating_keys():
    for dist in ["uniform", "zipf"]:
        w = Workload(10_000, 5_000, mix=(25, 25, 50), dist=dist)
        op, key, val, redraws = w.make_batch(0)
        mk = key[op != 0]
        assert mk.unique().numel() == mk.numel()
        assert int(key.min()) >= 0 and int(key.max()) < 10_000


def test_prefill_is_a_permutation():
    for R in [1, 2, 3, 1000, 65_537]:
        p = prefill_keys(SEED_BASE, R, R)
        assert torch.equal(p.sort().values, torch.arange(R))
    half = prefill_keys(SEED_BASE, 1000, 500)
    assert half.unique().numel() == 500


def test_uniform_key_range_and_large_R():
    idx = torch.arange(100_000)
    for R in [1, 10, 1_000_000_000, 2**32 - 2]:
        k = uniform_key(SEED_BASE, 3, idx, R)
        assert int(k.min()) >= 0 and int(k.max()) < R


def test_zipf_skew():
    w = Workload(1_000_000, 200_000, mix=(0, 0, 100), dist="zipf")
    op, key, _, _ = w.make_batch(0)
    top = feistel_perm(SEED_BASE ^ 6, torch.tensor([0]), 1_000_000)
    frac = float((key == top).float().mean())
    # p(rank 1) = 1/H_{R,0.99} ~ 0.066 at R = 1e6
    assert 0.05 < frac < 0.085
