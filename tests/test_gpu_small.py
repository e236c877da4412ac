"""GPU parity of the small-batch kernel: batches of up to GFSL_SMALL_BATCH ops (environment
at gfsl_create; 0 = never, the default) run the search phase, a grid-wide barrier (the S1
phase boundary, R1) and the update phase in ONE cooperative launch instead of a
search and an update kernel.
Every result vs Oracle-A and the same batches through the two-kernel path, the invariants
after every batch, and the launch counts that show which path ran."""
import numpy as np
import pytest
import torch

from oracle.oracle_a import OracleMap
from paper_conf_ppopp_moscovicicp17_b200.gfsl import GFSL
from tests.test_gpu_parity_r2 import check_all, to_dev

pytestmark = pytest.mark.gpu


def _handles(R, N, monkeypatch):
    monkeypatch.setenv("GFSL_SMALL_BATCH", "0")
    two = GFSL(R, chunk_entries=N)
    monkeypatch.setenv("GFSL_SMALL_BATCH", "16384")
    one = GFSL(R, chunk_entries=N)
    return one, two


@pytest.mark.parametrize("N", [16, 32])
def test_small_batch_kernel_matches_oracle_and_two_kernel_path(N, monkeypatch):
    R = 10_000
    one, two = _handles(R, N, monkeypatch)
    o = OracleMap(R)
    rng = np.random.default_rng(800 + N)
    fused = 0
    for b, n in enumerate([0, 1, 7, 100, 3000, 6250, 6250, 16384, 16385, 40000, 6250, 2]):
        # <= 1 mutation per key (R1): mutating keys drawn without replacement
        m = min(n // 5, R // 2)
        mk = rng.choice(R, m, replace=False).astype(np.uint32)
        ck = rng.integers(0, R, n - m).astype(np.uint32)
        key = np.concatenate([mk, ck])
        op = np.concatenate([rng.choice([1, 2], m), np.zeros(n - m, np.int64)]).astype(np.uint8)
        perm = rng.permutation(n)
        key, op = key[perm], op[perm]
        val = rng.integers(0, 2**32, n, dtype=np.uint64).astype(np.uint32)
        l0, l1 = one.stats()["kernel_launches"], two.stats()["kernel_launches"]
        r1 = one.batch(*to_dev(op, key, val)).cpu().numpy()
        r2 = two.batch(*to_dev(op, key, val)).cpu().numpy()
        e = o.batch(op, key, val)
        assert np.array_equal(r1, e), f"batch {b} (n={n}): fused path differs from the oracle"
        assert np.array_equal(r2, e), f"batch {b} (n={n}): two-kernel path differs from the oracle"
        d1 = one.stats()["kernel_launches"] - l0
        d2 = two.stats()["kernel_launches"] - l1
        if n == 0:
            assert d1 == d2 == 0                                        # nothing enqueued
        elif n <= 16384:
            assert d1 == d2 - 1, f"batch {b}: {d1} vs {d2} launches"   # search + update -> one kernel
            fused += 1
        else:
            assert d1 == d2
        check_all(one, o)
        rep, ks, vs = two.validate()
        ok, ov = o.export()
        assert rep.violations == 0 and np.array_equal(ks, ok) and np.array_equal(vs, ov)
    assert fused >= 8
    one.close()
    two.close()


def test_small_batch_kernel_churn_with_rebuilds(monkeypatch):
    """C1's shape (R = 10K, 6250-op batches of [10,10,80]) for 40 batches: splits, merges,
    the rebuild policy (R29) between fused batches."""
    from paper_conf_ppopp_moscovicicp17_b200.workload import SEED_BASE, Workload
    R = 10_000
    monkeypatch.setenv("GFSL_SMALL_BATCH", "16384")
    g = GFSL(R)
    o = OracleMap(R)
    k0 = np.random.default_rng(3).permutation(R)[:R // 2].astype(np.uint32)
    o.batch(np.ones(k0.size, np.uint8), k0, k0 + 1)
    g.batch(*to_dev(np.ones(k0.size, np.uint8), k0, k0 + 1))
    w = Workload(R, 6250, mix=(10, 10, 80), seed=SEED_BASE + 9)
    for b in range(40):
        op, key, val, _ = w.make_batch(b)
        op, key, val = op.numpy(), key.numpy().astype(np.uint32), val.numpy().astype(np.uint32)
        r = g.batch(*to_dev(op, key, val)).cpu().numpy()
        assert np.array_equal(r, o.batch(op, key, val)), f"batch {b}"
        if b % 5 == 4:
            check_all(g, o, cross=False)
    st = g.stats()
    assert st["splits"] > 0
    g.close()


@pytest.mark.parametrize("N", [16, 32])
def test_derived_paths_match_recorded_paths(N, monkeypatch):
    """R41: in lazy batches a directory-entered mutation writes no path and the update
    kernel recomputes its levels >= 1 from the key's directory rank when a general-path op
    (split, merge, a Delete whose key moved) needs them.  Heavy 50/50 churn with rebuilds
    between batches, derived vs recorded paths: the same results (vs Oracle-A) and valid
    structures after every batch."""
    R = 20_000
    monkeypatch.setenv("GFSL_DERIVE_PATH", "0")
    rec = GFSL(R, chunk_entries=N, rebuild_every=2)
    monkeypatch.delenv("GFSL_DERIVE_PATH")
    der = GFSL(R, chunk_entries=N, rebuild_every=2)
    o = OracleMap(R)
    rng = np.random.default_rng(900 + N)
    k0 = rng.permutation(R)[:R // 2].astype(np.uint32)
    for g in (rec, der):
        g.batch(*to_dev(np.ones(k0.size, np.uint8), k0, k0 + 3))
    o.batch(np.ones(k0.size, np.uint8), k0, k0 + 3)
    for b in range(30):
        key = rng.choice(R, 6000, replace=False).astype(np.uint32)
        op = rng.choice([0, 1, 2], key.size, p=[0.2, 0.4, 0.4]).astype(np.uint8)
        val = rng.integers(0, 2**32, key.size, dtype=np.uint64).astype(np.uint32)
        e = o.batch(op, key, val)
        for g in (rec, der):
            r = g.batch(*to_dev(op, key, val)).cpu().numpy()
            assert np.array_equal(r, e), f"batch {b}"
        check_all(der, o, cross=False)
        assert rec.check().violations == 0
    st = der.stats()
    assert st["splits"] > 0 and st["merges"] > 0
    rec.close()
    der.close()


@pytest.mark.parametrize("layout", ["dense", "clusters", "sparse"])
def test_coarse_directory_16bit_window(layout, monkeypatch):
    """With a coarse directory (C5's regime: more level-0 chunks than directory buckets,
    forced here by a 1024-bucket directory) the search kernel refines the directory's rank
    from an 8-key window of the sorted min keys (R38, R27c) and continues laterally when
    the key's chunk lies beyond it.  Dense keys, tight clusters far apart, and sparse keys:
    every result vs Oracle-A, with the directory rebuilt after every batch."""
    monkeypatch.setenv("GFSL_DIR_CAP", "1024")
    rng = np.random.default_rng({"dense": 1, "clusters": 2, "sparse": 3}[layout])
    if layout == "dense":
        R = 200_000
        keys = rng.permutation(R)[: R // 2]
    elif layout == "clusters":
        R = 1 << 30
        starts = rng.choice(R // (1 << 20), 60, replace=False) * (1 << 20)
        keys = np.unique(np.concatenate([s + rng.choice(3000, 1500, replace=False) for s in starts]))
    else:
        R = 1 << 31
        keys = np.unique(rng.integers(0, R, 60_000))
    keys = rng.permutation(keys).astype(np.uint32)
    g = GFSL(R, capacity=len(keys) * 2, rebuild_every=1)
    o = OracleMap(R)
    g.batch(*to_dev(np.ones(keys.size, np.uint8), keys, keys ^ 7))
    o.batch(np.ones(keys.size, np.uint8), keys, keys ^ 7)
    for b in range(6):
        # lookups of present keys, their neighbours, and random keys; a few mutations
        probe = np.concatenate([rng.choice(keys, 20_000), rng.choice(keys, 5_000) + 1,
                                rng.integers(0, R, 5_000).astype(np.uint32)]).astype(np.uint32)
        probe = np.minimum(probe, R - 1).astype(np.uint32)
        mut = rng.choice(keys, 2_000, replace=False)
        op = np.concatenate([np.zeros(probe.size, np.uint8), np.full(mut.size, 2, np.uint8)])
        key = np.concatenate([probe, mut]).astype(np.uint32)
        mutated = np.zeros(key.size, bool)
        mutated[probe.size:] = True
        # <= 1 mutation per key: the Contains of a mutated key may repeat (R1)
        r = g.batch(*to_dev(op, key, None)).cpu().numpy()
        e = o.batch(op, key, None)
        assert np.array_equal(r, e), f"{layout} batch {b}: {np.count_nonzero(r != e)} results differ"
        keys = np.setdiff1d(keys, mut)
        ins = rng.integers(0, R, 2_000).astype(np.uint32)
        ins = np.setdiff1d(ins, keys)[:1500]
        r = g.batch(*to_dev(np.ones(ins.size, np.uint8), ins, ins)).cpu().numpy()
        assert np.array_equal(r, o.batch(np.ones(ins.size, np.uint8), ins, ins))
        keys = np.union1d(keys, ins).astype(np.uint32)
        assert g.check().violations == 0
    g.close()


def test_host_async_zero_copy_values(monkeypatch):
    """With GFSL_ZC_VALUES=1, gfsl_batch_host_async reads the Insert values from a mapped
    pinned buffer instead of copying the value array (a pageable buffer is still copied):
    results and stored values vs Oracle-A, and the library's count of zero-copy batches."""
    R = 50_000
    monkeypatch.setenv("GFSL_ZC_VALUES", "1")
    g = GFSL(R)
    o = OracleMap(R)
    rng = np.random.default_rng(77)
    k0 = rng.permutation(R)[: R // 2].astype(np.uint32)
    g.batch(*to_dev(np.ones(k0.size, np.uint8), k0, k0 + 5))
    o.batch(np.ones(k0.size, np.uint8), k0, k0 + 5)
    outs = []
    for b in range(8):
        key = rng.choice(R, 20_000, replace=False).astype(np.uint32)
        op = rng.choice([0, 1, 2], key.size, p=[0.5, 0.3, 0.2]).astype(np.uint8)
        val = rng.integers(0, 2**32, key.size, dtype=np.uint64).astype(np.uint32)
        pinned = b % 2 == 0
        t = (torch.from_numpy(op), torch.from_numpy(key.view(np.int32)), torch.from_numpy(val.view(np.int32)))
        if pinned:
            t = tuple(x.pin_memory() for x in t)
        outs.append((g.batch_host_async(*t), o.batch(op, key, val), t))
    torch.cuda.synchronize()
    for r, e, _ in outs:
        assert np.array_equal(r.numpy(), e)
    dk, dv = g.export()
    ok, ov = o.export()
    assert np.array_equal(dk.cpu().numpy().view(np.uint32), ok)
    assert np.array_equal(dv.cpu().numpy().view(np.uint32), ov)
    assert g.stats()["zero_copy_batches"] == 4
    g.close()
