"""GPU parity of combining mode (R26) through the C ABI.

Batches with ANY number of Insert/Delete ops per key (i.i.d. keys on tiny ranges, raw
Zipf(0.99) without the generator's redraws, hand-built chains on one key) are compared
element by element with Oracle-A's combining semantics (oracle.oracle_a oa_batch_seq:
Contains on the pre-batch map, mutations one by one in input order); after every batch
the exported (key, value) set must equal the oracle's and the invariants must hold.
"""
import numpy as np
import pytest
import torch

from oracle.oracle_a import OracleMap
from paper_conf_ppopp_moscovicicp17_b200.gfsl import GFSL
from paper_conf_ppopp_moscovicicp17_b200.workload import SEED_BASE, Workload

from .test_gpu_parity import check_same_set, prefill, to_dev

pytestmark = pytest.mark.gpu


def run_comb(g, o, op, key, val):
    r_gpu = g.batch(*to_dev(op, key, val)).cpu().numpy()
    r_ora = o.batch(op, key, val, combine=True)
    mism = np.flatnonzero(r_gpu != r_ora)
    assert mism.size == 0, (f"{mism.size} mismatches, first at {mism[:5]}: gpu={r_gpu[mism[:5]]} "
                            f"oracle={r_ora[mism[:5]]} op={op[mism[:5]]} key={key[mism[:5]]}")


def dup_batch(rng, R, B, invalid=True):
    op = rng.integers(0, 3, size=B).astype(np.uint8)
    key = rng.integers(0, R, size=B).astype(np.uint32)
    val = rng.integers(0, 2**32, size=B, dtype=np.uint64).astype(np.uint32)
    if invalid and B > 20:
        j = rng.integers(0, B, size=B // 20)
        op[j[: len(j) // 2]] = 7
        key[j[len(j) // 2:]] = R + 3
    return op, key, val


@pytest.mark.parametrize("N,serial", [(16, False), (32, False), (16, True), (12, False), (6, True)])
def test_combine_duplicates_small_range(N, serial):
    """Every key is hit by many ops per batch: long mixed chains, splits and merges."""
    R = 700
    rng = np.random.default_rng(N + 100 * serial)
    g = GFSL(R, chunk_entries=N, combine=True, serial_updates=serial)
    o = OracleMap(R)
    for b in range(12):
        B = int(rng.integers(1, 5000)) if b else 0
        if B == 0:
            continue
        run_comb(g, o, *dup_batch(rng, R, B))
        check_same_set(g, o)
    g.close()


def test_combine_chains_one_key():
    """Hand-worked chains (tests/test_oracle_a.py::test_oracle_seq_per_key_automaton) on the GPU."""
    I, D, C = 1, 2, 0
    g = GFSL(10, combine=True)
    o = OracleMap(10)
    for ops, vals in [([I, I, D, I, C], [5, 6, 0, 7, 0]), ([D, D, I, I], [0, 0, 8, 9]),
                      ([I, D, C], [1, 0, 0]), ([I, I, I], [3, 4, 5]), ([D, I, D, I], [0, 6, 0, 7]),
                      ([I, D, I, D, I], [1, 2, 3, 4, 5])]:
        op = np.array(ops, np.uint8)
        run_comb(g, o, op, np.full(op.size, 4, np.uint32), np.array(vals, np.uint32))
        check_same_set(g, o)


@pytest.mark.parametrize("mix", [(10, 10, 80), (50, 50, 0)])
def test_combine_raw_zipf(mix):
    """Zipf(0.99) with the mutating keys i.i.d. (no redraws): hot keys carry long chains."""
    R = 200_000
    g = GFSL(R, combine=True)
    o = OracleMap(R)
    prefill(g, o, R, R // 2)
    w = Workload(R, 60_000 + 11, mix=mix, dist="zipf", seed=SEED_BASE + 5, dedup=False)
    for b in range(5):
        op, key, val, red = w.make_batch(b)
        assert red == 0
        kn = key.numpy().astype(np.uint32)
        mut = op.numpy() != 0
        assert np.unique(kn[mut]).size < mut.sum()  # duplicates really occur
        run_comb(g, o, op.numpy(), kn, val.numpy().astype(np.uint32))
        check_same_set(g, o)


def test_combine_equals_contract_mode_under_contract():
    """Inside the contract the two modes give the same results and the same map."""
    R = 50_000
    a, b = GFSL(R), GFSL(R, combine=True)
    o = OracleMap(R)
    w = Workload(R, 20_000 + 5, mix=(30, 20, 50), seed=SEED_BASE + 9)
    for i in range(6):
        op, key, val, _ = w.make_batch(i)
        d = to_dev(op.numpy(), key.numpy().astype(np.uint32), val.numpy().astype(np.uint32))
        ra, rb = a.batch(*d).cpu().numpy(), b.batch(*d).cpu().numpy()
        ro = o.batch(op.numpy(), key.numpy().astype(np.uint32), val.numpy().astype(np.uint32))
        assert np.array_equal(ra, ro) and np.array_equal(rb, ro)
    check_same_set(a, o)
    check_same_set(b, o)


def test_combine_host_entry_and_toggle():
    """gfsl_batch_host in combining mode; switching the mode on a live handle."""
    R = 5_000
    rng = np.random.default_rng(3)
    g = GFSL(R)
    o = OracleMap(R)
    op, key, val = dup_batch(rng, R, 3000)
    op[key < R] = np.where(op[key < R] == 2, 0, op[key < R])  # inserts only ...
    _, first = np.unique(key, return_index=True)
    keep = np.zeros(op.size, bool)
    keep[first] = True
    op[~keep & (op == 1)] = 0                                 # ... at most one per key
    run_comb(g, o, op, key, val)
    g.configure(combine=1)
    for _ in range(4):
        op, key, val = dup_batch(rng, R, 4000)
        r = g.batch_host(torch.from_numpy(op), torch.from_numpy(key.view(np.int32)),
                         torch.from_numpy(val.view(np.int32))).numpy()
        assert np.array_equal(r, o.batch(op, key, val, combine=True))
        check_same_set(g, o)
