"""The bulk path (R34; csrc/gfsl_bulk.cuh): a batch much larger than the
structure is applied by sorting the level-0 entries and the ops together and writing
level 0 anew.  Its results must be S1's (Oracle-A, element by element), its structure must
pass every invariant, and the per-op path must continue on it exactly."""
import time

import numpy as np
import pytest
import torch

from oracle.oracle_a import OracleMap
from paper_conf_ppopp_moscovicicp17_b200.gfsl import BULK_ALWAYS, BULK_OFF, GFSL
from paper_conf_ppopp_moscovicicp17_b200.workload import SEED_BASE, Workload
from tests.linearize import linearizable

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda")


def to_dev(op, key, val):
    return (torch.as_tensor(np.ascontiguousarray(op, np.uint8)).to(DEV),
            torch.as_tensor(np.ascontiguousarray(key, np.uint32).view(np.int32)).to(DEV),
            None if val is None else torch.as_tensor(np.ascontiguousarray(val, np.uint32).view(np.int32)).to(DEV))


def run_batch(g, o, op, key, val):
    r = g.batch(*to_dev(op, key, val)).cpu().numpy()
    e = o.batch(op, key, val)
    bad = np.flatnonzero(r != e)
    assert bad.size == 0, f"{bad.size} results differ, first {bad[:5]}: gpu={r[bad[:5]]} oracle={e[bad[:5]]}"


def same_set(g, o):
    d = g.check()
    assert d.violations == 0 and d.keys == len(o)
    rep, ks, vs = g.validate()
    ok, ov = o.export()
    assert rep.violations == 0 and np.array_equal(ks, ok) and np.array_equal(vs, ov)


@pytest.mark.parametrize("N", [16, 32])
def test_bulk_load_into_empty_map(N):
    R = 2_000_000
    g = GFSL(R, chunk_entries=N)
    o = OracleMap(R)
    k = np.random.default_rng(N).permutation(R)[:1_000_000].astype(np.uint32)
    v = (k * 3 + 1).astype(np.uint32)
    run_batch(g, o, np.ones(k.size, np.uint8), k, v)
    assert g.stats()["splits"] == 0               # no per-op path: level 0 written at once
    same_set(g, o)
    # the per-op path continues on the bulk-built structure
    w = Workload(R, 200_000, mix=(20, 20, 60), seed=SEED_BASE + 401)
    for b in range(4):
        op, key, val, _ = w.make_batch(b)
        run_batch(g, o, op.numpy(), key.numpy().astype(np.uint32), val.numpy().astype(np.uint32))
    same_set(g, o)


def test_bulk_load_rate():
    """one 1M-insert batch into an empty map (the smoke test's cold start took
    1.7 ms per 1000 inserts on the per-op path)."""
    R = 4_000_000
    k = torch.randperm(R, device=DEV)[:1_000_000].to(torch.int32)
    ones = torch.ones(k.numel(), dtype=torch.uint8, device=DEV)
    best = 1e9
    for _ in range(3):
        g = GFSL(R)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        r = g.batch(ones, k, k)
        torch.cuda.synchronize()
        best = min(best, time.perf_counter() - t0)
        assert int(r.min()) == 1
        g.close()
    print(f"bulk load: 1M inserts in {best * 1e3:.2f} ms ({1e-3 / best:.2f} G ops/s, incl. the host path)")
    assert best < 0.05


@pytest.mark.parametrize("N", [16, 12, 6])
def test_bulk_every_batch_matches_oracle(N):
    """Every batch through the bulk path (BULK_ALWAYS): mixed ops, deletes of present keys,
    inserts of present keys, invalid ops and keys."""
    R = 30_000 if N >= 12 else 3000
    g = GFSL(R, chunk_entries=N, bulk=BULK_ALWAYS)
    o = OracleMap(R)
    w = Workload(R, R // 3, mix=(35, 30, 35), seed=SEED_BASE + 402 + N)
    for b in range(10):
        op, key, val, _ = w.make_batch(b)
        op, key, val = op.numpy().copy(), key.numpy().astype(np.uint32), val.numpy().astype(np.uint32)
        if b == 3:
            op[::101] = 9
            key[::89] = R + 7
        run_batch(g, o, op, key, val)
        same_set(g, o)


def test_bulk_then_per_op_then_bulk():
    R = 200_000
    g = GFSL(R)
    o = OracleMap(R)
    rng = np.random.default_rng(9)
    k = rng.permutation(R)[:100_000].astype(np.uint32)
    run_batch(g, o, np.ones(k.size, np.uint8), k, k)          # bulk (empty map)
    for b in range(3):                                          # per-op
        kk = rng.permutation(R)[:20_000].astype(np.uint32)
        op = rng.integers(0, 3, kk.size).astype(np.uint8)
        run_batch(g, o, op, kk, kk + 5)
    g.configure(bulk=BULK_ALWAYS)
    kk = rng.permutation(R)[:150_000].astype(np.uint32)          # bulk again, mixed
    op = rng.integers(0, 3, kk.size).astype(np.uint8)
    run_batch(g, o, op, kk, kk + 9)
    same_set(g, o)


def test_bulk_out_of_contract_is_linearizable():
    R = 5000
    g = GFSL(R, bulk=BULK_ALWAYS)
    rng = np.random.default_rng(12)
    present = np.zeros(R, bool)
    value = np.zeros(R, np.uint32)
    for b in range(6):
        n = 8000
        key = rng.integers(0, R // 4, n).astype(np.uint32)
        op = rng.choice([0, 1, 2], n, p=[0.3, 0.4, 0.3]).astype(np.uint8)
        val = rng.integers(0, 2**32, n, dtype=np.uint64).astype(np.uint32)
        r = g.batch(*to_dev(op, key, val)).cpu().numpy()
        rep, ks, vs = g.validate()
        assert rep.violations == 0
        fin_p = np.zeros(R, bool)
        fin_p[ks] = True
        fin_v = np.zeros(R, np.uint32)
        fin_v[ks] = vs
        order = np.argsort(key, kind="stable")
        for grp in np.split(order, np.flatnonzero(np.diff(key[order])) + 1):
            k = int(key[grp[0]])
            assert linearizable(bool(present[k]), int(value[k]), op[grp].tolist(), r[grp].tolist(),
                                val[grp].tolist(), bool(fin_p[k]), int(fin_v[k]))
        present, value = fin_p, fin_v


def test_bulk_off_uses_the_per_op_path():
    R = 100_000
    g = GFSL(R, bulk=BULK_OFF)
    o = OracleMap(R)
    k = np.random.default_rng(3).permutation(R)[:80_000].astype(np.uint32)
    run_batch(g, o, np.ones(k.size, np.uint8), k, k)
    assert g.stats()["splits"] > 0
    same_set(g, o)
