"""The level-1 directory (R27) through the C ABI: Contains enter searchDown at
level 1 in the chunk the directory names for their key's bucket.  The directory is
written by each upper-level rebuild and may be stale for the batches in between: a
chunk reached from a stale entry either leads laterally to the right chunk or holds no
key <= k, and then the traversal restarts from the top (Alg 4.2 l.25).  These tests
make it stale on purpose and check every result against Oracle-A."""
import numpy as np
import pytest

from oracle.oracle_a import OracleMap
from paper_conf_ppopp_moscovicicp17_b200.gfsl import GFSL
from paper_conf_ppopp_moscovicicp17_b200.workload import SEED_BASE, Workload

from .test_gpu_parity import check_same_set, prefill, run_batch

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("N,serial,l0", [(16, True, False), (32, True, False), (16, False, False),
                                          (32, False, False), (16, True, True), (32, False, True)])
def test_stale_directory_restarts(N, serial, l0, monkeypatch):
    """Serial mode removes deleted keys from the upper levels (Alg 4.11), so the directory
    goes stale and Contains entered at level 1 (R27) restart; concurrent batches leave them
    as separators until the next rebuild (R33), which must answer the same.  With the
    level-0 entry (R37, the default) the same batches go through the rebuild's rank order
    of level-0 chunks, which zombies and splits since the rebuild only lengthen laterally."""
    if not l0:
        monkeypatch.setenv("GFSL_NO_L0_ENTRY", "1")
    R = 40_000
    g = GFSL(R, chunk_entries=N, rebuild_every=3, serial_updates=serial)
    o = OracleMap(R)
    prefill(g, o, R, R, chunk=4096)           # several batches: a rebuild writes the directory
    check_same_set(g, o)
    rng = np.random.default_rng(N)
    r0 = g.stats()["restarts"]
    # 60% of the keys deleted in one batch: level-1 keys vanish under the directory
    keys = rng.permutation(R)[: R * 6 // 10].astype(np.uint32)
    run_batch(g, o, np.full(keys.size, 2, np.uint8), keys, None)
    # Contains of every key (and some out of range) before the next rebuild
    ck = np.concatenate([np.arange(R, dtype=np.uint32), np.array([R, R + 5], np.uint32)])
    run_batch(g, o, np.zeros(ck.size, np.uint8), ck, None)
    if serial and not l0:
        assert g.stats()["restarts"] > r0, "the stale-directory path was not exercised"
    check_same_set(g, o)
    # churn with re-inserts, then more Contains, across rebuilds
    w = Workload(R, 9_000 + 7, mix=(30, 30, 40), seed=SEED_BASE + 17)
    for b in range(8):
        op, key, val, _ = w.make_batch(b)
        run_batch(g, o, op.numpy(), key.numpy().astype(np.uint32), val.numpy().astype(np.uint32))
        check_same_set(g, o)


def test_directory_not_used_after_load():
    """gfsl_load replaces the structure: the directory is dropped until the next rebuild."""
    R = 5_000
    a = GFSL(R)
    o = OracleMap(R)
    prefill(a, o, R, R // 2, chunk=1000)
    meta, ent = a.dump()
    b = GFSL(R)
    ob = OracleMap(R)
    prefill(b, ob, R, R, chunk=700)           # b has a directory for a different structure
    b.load(meta, ent)
    ck = np.arange(R, dtype=np.uint32)
    run_batch(b, o, np.zeros(R, np.uint8), ck, None)
