"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times
(same configs, generator, prefill, chunk size and default launch shape).

* C2 (R = 1M, 625K-op batches): every result of every batch vs the direct-address-table
  checker (oracle/dat.py, pinned to Oracle-A), the exported final set, the invariants.
* C3 (R = 10M, 6.25M-op batches): the same, for 4 batches.
* C2 raw Zipf in combining mode (R26): every result vs Oracle-A's combining semantics.
* C4-16 (100M keys, 50M Contains per batch): every lookup of a key of the full structure
  answers true (a property at any size), and the invariants hold.
* C5 (R = 1B, 500M live keys, 125M-op batches): sampled -- present and absent keys of the
  prefill answer true / false, and one full 10/10/80 batch keeps #true inserts and
  deletes equal to the closed forms |I \\ M| and |D & M| on its sampled keys.
"""
import numpy as np
import pytest
import torch

from oracle.dat import DirectAddressMap
from oracle.oracle_a import OracleMap
from paper_conf_ppopp_moscovicicp17_b200.gfsl import GFSL
from paper_conf_ppopp_moscovicicp17_b200.workload import (
    SEED_BASE, Workload, prefill_keys, prefill_values)

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda")


def cfg(name):
    import bench
    return bench.CONFIGS[name]


def prefill_both(g, ref, R, count):
    import bench
    bench.prefill_gpu(g, R, count, DEV)
    if ref is not None and count:
        k = prefill_keys(SEED_BASE, R, count).numpy().astype(np.uint32)
        ref.batch(np.ones(k.size, np.uint8), k, prefill_values(SEED_BASE, torch.from_numpy(k.astype(np.int64))).numpy().astype(np.uint32))


def run_and_compare(g, ref, w, b, combine=False):
    op, key, val, _ = w.make_batch(b, device=DEV)
    r = g.batch(op.contiguous(), key.to(torch.int32).contiguous(), val.to(torch.int32).contiguous()).cpu().numpy()
    on, kn, vn = op.cpu().numpy(), key.cpu().numpy().astype(np.uint32), val.cpu().numpy().astype(np.uint32)
    e = ref.batch(on, kn, vn, combine=True) if combine else ref.batch(on, kn, vn)
    bad = np.flatnonzero(r != e)
    assert bad.size == 0, f"batch {b}: {bad.size} results differ, first {bad[:5]}"


def check_set(g, ref):
    rep, ks, vs = g.validate()
    ek, ev = ref.export()
    assert rep.violations == 0
    assert np.array_equal(ks, ek) and np.array_equal(vs, ev)


@pytest.mark.parametrize("name,nb", [("C2", 19), ("C3", 4)])
def test_fullsize_every_result(name, nb):
    R, pre, B, _, mix, dist, N = cfg(name)
    g = GFSL(R, capacity=R, chunk_entries=N)
    ref = DirectAddressMap(R)
    prefill_both(g, ref, R, pre)
    w = Workload(R, B, mix=mix, dist=dist, seed=SEED_BASE + 1)
    for b in range(nb):
        run_and_compare(g, ref, w, b)
    check_set(g, ref)
    g.close()


def test_fullsize_raw_zipf_combining():
    R, pre, B, _, mix, dist, N = cfg("C2-zipf-raw")
    g = GFSL(R, capacity=R, chunk_entries=N, combine=True)
    ref = OracleMap(R)
    prefill_both(g, ref, R, pre)
    w = Workload(R, B, mix=mix, dist=dist, seed=SEED_BASE + 1, dedup=False)
    for b in range(4):
        run_and_compare(g, ref, w, b, combine=True)
    check_set(g, ref)
    g.close()


def test_fullsize_c4_contains_all_true():
    R, pre, B, _, mix, dist, N = cfg("C4-16")
    g = GFSL(R, capacity=R, chunk_entries=N)
    prefill_both(g, None, R, pre)
    w = Workload(R, B, mix=mix, dist=dist, seed=SEED_BASE + 1)
    for b in range(2):
        op, key, val, _ = w.make_batch(b, device=DEV)
        assert int(op.max()) == 0
        r = g.batch(op.contiguous(), key.to(torch.int32).contiguous(), None)
        assert int(r.min()) == 1 and int(r.max()) == 1
    rep, _, _ = g.validate(export=False)
    assert rep.violations == 0 and rep.keys == R
    g.close()


def test_fullsize_c5_sampled():
    R, pre, B, _, mix, dist, N = cfg("C5")
    g = GFSL(R, capacity=R, chunk_entries=N)
    prefill_both(g, None, R, pre)
    present = prefill_keys(SEED_BASE, R, 1 << 20, start=0, device=DEV)
    absent = prefill_keys(SEED_BASE, R, 1 << 20, start=pre, device=DEV)
    zeros = torch.zeros(1 << 20, dtype=torch.uint8, device=DEV)
    assert int(g.batch(zeros, present.to(torch.int32)).min()) == 1
    assert int(g.batch(zeros, absent.to(torch.int32)).max()) == 0
    # one full batch; its mutating keys on the sampled present / absent sets obey the
    # closed forms of S1 (an Insert succeeds iff absent, a Delete iff present)
    w = Workload(R, B, mix=mix, dist=dist, seed=SEED_BASE + 1)
    op, key, val, _ = w.make_batch(0, device=DEV)
    r = g.batch(op.contiguous(), key.to(torch.int32).contiguous(), val.to(torch.int32).contiguous())
    ps = torch.zeros(R, dtype=torch.bool, device=DEV)
    ps[present] = True
    ab = torch.zeros(R, dtype=torch.bool, device=DEV)
    ab[absent] = True
    k = key.to(torch.int64)
    ins, dele = op == 1, op == 2
    assert bool((r[ins & ps[k]] == 0).all()) and bool((r[ins & ab[k]] == 1).all())
    assert bool((r[dele & ps[k]] == 1).all()) and bool((r[dele & ab[k]] == 0).all())
    assert bool((r[(op == 0) & ps[k]] == 1).all()) and bool((r[(op == 0) & ab[k]] == 0).all())
    assert int((ins & (ps[k] | ab[k])).sum()) > 1000
    g.close()
