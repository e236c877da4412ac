"""GPU parity of the chunk-grouped update path (R40).

Opt-in (gfsl_config.group): in lazy concurrent batches the Insert/Delete ops that target one bottom
chunk are applied by one team in one lock session of that chunk: a merged write, a split
into several new chunks, or the paper's merge (Alg 4.12) for the last Delete.  These tests
drive every branch -- many inserts per chunk (multi-way splits), many deletes per chunk
(merges, emptied last chunks), mixed groups, out-of-contract duplicates in one group --
and check every result against Oracle-A, the exported set, and the invariants (host walk
and device check) after every batch, with grouping on and off on the same inputs.  The
out-of-contract (duplicate keys in one group) case is in test_gpu_parity_r2.
"""
import numpy as np
import pytest
import torch

from oracle.oracle_a import OracleMap
from paper_conf_ppopp_moscovicicp17_b200.gfsl import BULK_OFF, GROUP_OFF, GROUP_ON, GFSL
from tests.test_gpu_parity_r2 import check_all, run_batch, to_dev

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda")


def _pair(R, N):
    """The same map twice: grouped (opt-in) and one lock session per op (the default)."""
    return (GFSL(R, chunk_entries=N, bulk=BULK_OFF, group=GROUP_ON),
            GFSL(R, chunk_entries=N, bulk=BULK_OFF, group=GROUP_OFF))


@pytest.mark.parametrize("N", [16, 32])
def test_group_insert_heavy_multi_split(N):
    """Batches of inserts several times larger than the structure: tens of inserts per
    chunk, so a group overflows its chunk into q > 2 chunks."""
    R = 200_000
    g, g0 = _pair(R, N)
    o = OracleMap(R)
    rng = np.random.default_rng(400 + N)
    perm = rng.permutation(R).astype(np.uint32)
    s = 0
    for size in (500, 2_000, 8_000, 30_000, 60_000, 99_500):
        k = perm[s:s + size]
        s += size
        op = np.ones(k.size, np.uint8)
        r = run_batch(g, o, op, k, k ^ 0x5A5A5A5A)
        r0 = g0.batch(*to_dev(op, k, k ^ 0x5A5A5A5A)).cpu().numpy()
        assert np.array_equal(r, r0)
        check_all(g, o)
    st = g.stats()
    assert st["grouped"] > 0.5 * st["mutations"] and st["splits"] > 0
    rep, _, _ = g.validate()
    assert rep.keys == s
    g.close()
    g0.close()


@pytest.mark.parametrize("N", [16, 32])
def test_group_delete_heavy_merges_and_drain(N):
    """Fill, then drain in large delete batches: groups leave chunks below DSIZE/3 (the
    merge branch) and empty the last chunk."""
    R = 60_000
    g = GFSL(R, chunk_entries=N, bulk=BULK_OFF, group=GROUP_ON)
    o = OracleMap(R)
    rng = np.random.default_rng(500 + N)
    k = rng.permutation(R).astype(np.uint32)
    for s in range(0, R, 20_000):
        run_batch(g, o, np.ones(20_000, np.uint8), k[s:s + 20_000], k[s:s + 20_000] * 3)
    check_all(g, o)
    m0 = g.stats()["merges"]
    d = rng.permutation(R).astype(np.uint32)
    for s in range(0, R, 15_000):
        run_batch(g, o, np.full(15_000, 2, np.uint8), d[s:s + 15_000], None)
        check_all(g, o)
    assert len(o) == 0
    st = g.stats()
    assert st["merges"] > m0 and st["grouped"] > 0
    g.close()


@pytest.mark.parametrize("N", [16, 32])
def test_group_mixed_churn_small_range(N):
    """50/50 Insert/Delete over a 3000-key range, batches of ~1/3 of the range: groups
    mix inserts and deletes, splits and merges happen in the same batches."""
    R = 3000
    g, g0 = _pair(R, N)
    o = OracleMap(R)
    rng = np.random.default_rng(600 + N)
    for b in range(40):
        k = rng.choice(R, 1000, replace=False).astype(np.uint32)   # <= 1 mutation per key
        op = rng.choice([0, 1, 2], k.size, p=[0.1, 0.45, 0.45]).astype(np.uint8)
        val = rng.integers(0, 2**32, k.size, dtype=np.uint64).astype(np.uint32)
        r = run_batch(g, o, op, k, val)
        r0 = g0.batch(*to_dev(op, k, val)).cpu().numpy()
        assert np.array_equal(r, r0)
        check_all(g, o)
    st = g.stats()
    assert st["grouped"] > 0 and st["splits"] > 0 and st["merges"] > 0
    g.close()
    g0.close()


def test_group_tiny_structure_one_chunk():
    """Every op of a batch in the one chunk of a fresh map (the first chunk holds -inf and
    is also the last): the level-0 counter transitions of Alg 4.5 l.37-38 and R17."""
    R = 64
    g = GFSL(R, bulk=BULK_OFF, group=GROUP_ON)
    o = OracleMap(R)
    rng = np.random.default_rng(7)
    for b in range(30):
        k = rng.choice(R, rng.integers(1, 20), replace=False).astype(np.uint32)
        op = rng.choice([1, 2], k.size).astype(np.uint8)
        run_batch(g, o, op, k, k + 1)
        check_all(g, o)
    g.close()
