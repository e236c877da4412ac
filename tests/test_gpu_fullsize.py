"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times
(same configs, generator, prefill, chunk size and default launch shape).

* C2 (R = 1M, 625K-op batches): every result of every batch vs the direct-address-table
  checker (oracle/dat.py, pinned to Oracle-A), the exported final set, the invariants.
* C3 (R = 10M, 6.25M-op batches): the same, for 4 batches.
* C2 raw Zipf in combining mode (R26): every result vs Oracle-A's combining semantics.
* C4-16 (100M keys, 50M Contains per batch): every lookup of a key of the full structure
  answers true, the device export is exactly (k, prefill value of k) for every k, and the
  device check passes.
* C5 (R = 1B, 500M live keys, 125M-op batches): every result of 2 full batches vs the DAT
  (5 GB of host memory), then the exported set (device export, 500M pairs) vs the DAT and
  the device check (gfsl_check: V1-V5, V7-V9, V12, V14, chain shape; V6 / V11 across the
  batches).
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
    d = g.check()
    assert d.violations == 0 and d.keys == R
    ks, vs = g.export()
    assert ks.numel() == R
    assert bool((ks.to(torch.int64) == torch.arange(R, device=DEV)).all())
    exp_v = prefill_values(SEED_BASE, torch.arange(R, device=DEV)).to(torch.int32)
    assert bool((vs == exp_v).all())
    g.close()


def test_fullsize_c5_every_result():
    R, pre, B, _, mix, dist, N = cfg("C5")
    g = GFSL(R, capacity=R, chunk_entries=N)
    ref = DirectAddressMap(R)
    import bench
    bench.prefill_gpu(g, R, pre, DEV)
    for s0 in range(0, pre, 1 << 26):  # the same prefill into the DAT, in slices
        k = prefill_keys(SEED_BASE, R, min(1 << 26, pre - s0), start=s0, device=DEV)
        v = prefill_values(SEED_BASE, k)
        ref.load(k.cpu().numpy(), v.cpu().numpy().astype(np.uint32))
    d = g.check(snapshot=True)
    assert d.violations == 0 and d.keys == pre
    w = Workload(R, B, mix=mix, dist=dist, seed=SEED_BASE + 1)
    for b in range(2):
        op, key, val, _ = w.make_batch(b, device=DEV)
        r = g.batch(op.contiguous(), key.to(torch.int32).contiguous(), val.to(torch.int32).contiguous())
        r = r.cpu().numpy()
        e = ref.batch(op.cpu().numpy(), key.cpu().numpy().astype(np.uint32), val.cpu().numpy().astype(np.uint32))
        bad = np.flatnonzero(r != e)
        assert bad.size == 0, f"batch {b}: {bad.size} of {B} results differ, first {bad[:5]}"
        d = g.check(snapshot=True, cross=True)
        assert d.violations == 0
    ks, vs = g.export()
    ek, ev = ref.export()
    assert ks.numel() == ek.size
    assert np.array_equal(ks.cpu().numpy().view(np.uint32), ek)
    assert np.array_equal(vs.cpu().numpy().view(np.uint32), ev)
    g.close()
