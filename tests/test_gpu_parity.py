"""GPU parity: the CUDA path (through the C ABI) vs Oracle-A, element by element.

Every test runs seeded batches through ``gfsl_batch`` and through the oracle on the same
inputs, compares every per-op result bit-exactly, and after every batch checks the
structural invariants (``gfsl_validate``) and that the exported (key, value) set equals
the oracle's.  Sizes span many chunks and levels plus ragged tails.
"""
import numpy as np
import pytest
import torch

from oracle.oracle_a import OracleMap
from paper_conf_ppopp_moscovicicp17_b200.gfsl import GFSL
from paper_conf_ppopp_moscovicicp17_b200.workload import (
    SEED_BASE, Workload, prefill_keys, prefill_values)

pytestmark = pytest.mark.gpu


def to_dev(op, key, val):
    dev = torch.device("cuda")
    op_d = torch.as_tensor(np.ascontiguousarray(op, np.uint8)).to(dev)
    key_d = torch.as_tensor(np.ascontiguousarray(key, np.uint32).view(np.int32)).to(dev)
    val_d = None if val is None else torch.as_tensor(
        np.ascontiguousarray(val, np.uint32).view(np.int32)).to(dev)
    return op_d, key_d, val_d


def check_same_set(g: GFSL, o: OracleMap):
    rep, ks, vs = g.validate()
    ok, ov = o.export()
    assert rep.violations == 0
    assert rep.keys == len(o)
    assert np.array_equal(ks, ok)
    assert np.array_equal(vs, ov)
    return rep


def run_batch(g, o, op, key, val):
    r_gpu = g.batch(*to_dev(op, key, val)).cpu().numpy()
    torch.cuda.synchronize()
    r_ora = o.batch(op, key, val)
    mism = np.flatnonzero(r_gpu != r_ora)
    assert mism.size == 0, f"{mism.size} mismatches, first at {mism[:5]}: gpu={r_gpu[mism[:5]]} oracle={r_ora[mism[:5]]} op={op[mism[:5]]} key={key[mism[:5]]}"
    return r_gpu


def prefill(g, o, R, count, seed=SEED_BASE, chunk=1 << 20):
    for s in range(0, count, chunk):
        c = min(chunk, count - s)
        k = prefill_keys(seed, R, c, start=s)
        v = prefill_values(seed, k)
        op = np.ones(c, np.uint8)
        run_batch(g, o, op, k.numpy().astype(np.uint32), v.numpy().astype(np.uint32))


def workload_batches(R, B, nb, mix, dist="uniform", seed=SEED_BASE + 1):
    w = Workload(R, B, mix=mix, dist=dist, seed=seed)
    for b in range(nb):
        op, key, val, _ = w.make_batch(b)
        yield op.numpy(), key.numpy().astype(np.uint32), val.numpy().astype(np.uint32)


@pytest.mark.parametrize("N,team", [(32, 8), (32, 16), (32, 32), (16, 4), (16, 8), (16, 16)])
def test_mixed_batches(N, team):
    R = 20_000
    g = GFSL(R, chunk_entries=N, contains_team=team)
    o = OracleMap(R)
    prefill(g, o, R, R // 2)
    check_same_set(g, o)
    for op, key, val in workload_batches(R, 4_000 + 37, 6, (20, 20, 60)):
        run_batch(g, o, op, key, val)
        check_same_set(g, o)


@pytest.mark.parametrize("N", [32, 16, 12, 6])
def test_serial_mode_churn(N):
    """One team applies the updates in op order: the deterministic mode."""
    R = 3_000
    g = GFSL(R, chunk_entries=N, serial_updates=True)
    o = OracleMap(R)
    prefill(g, o, R, R // 2)
    check_same_set(g, o)
    for op, key, val in workload_batches(R, 1_500, 8, (30, 30, 40)):
        run_batch(g, o, op, key, val)
        check_same_set(g, o)


@pytest.mark.parametrize("N", [32, 16])
def test_heavy_churn_small_range(N):
    """Tiny key range, 50/50 updates: contention, splits, merges and zombies everywhere."""
    R = 600
    g = GFSL(R, chunk_entries=N)
    o = OracleMap(R)
    for op, key, val in workload_batches(R, 300, 40, (50, 50, 0)):
        run_batch(g, o, op, key, val)
        check_same_set(g, o)
    st = g.stats()
    assert st["splits"] > 0 and st["merges"] > 0


@pytest.mark.parametrize("N", [32, 16])
def test_fill_then_drain(N):
    """Insert-only of every key from empty, then Delete-only of every key."""
    R = 50_000
    g = GFSL(R, chunk_entries=N)
    o = OracleMap(R)
    perm = np.random.default_rng(5).permutation(R).astype(np.uint32)
    for s in range(0, R, 12_345):
        k = perm[s:s + 12_345]
        run_batch(g, o, np.ones(k.size, np.uint8), k, k * 3)
    rep = check_same_set(g, o)
    assert rep.keys == R and rep.height >= 2
    perm2 = np.random.default_rng(6).permutation(R).astype(np.uint32)
    for s in range(0, R, 9_999):
        k = perm2[s:s + 9_999]
        run_batch(g, o, np.full(k.size, 2, np.uint8), k, None)
        check_same_set(g, o)
    rep = check_same_set(g, o)
    assert rep.keys == 0


def test_edge_cases():
    R = 1000
    g = GFSL(R)
    o = OracleMap(R)
    # empty batch
    out = g.batch(*to_dev(np.zeros(0, np.uint8), np.zeros(0, np.uint32), None))
    assert out.numel() == 0
    # everything on an empty map
    run_batch(g, o, np.array([0, 2, 1, 0], np.uint8), np.array([5, 5, 7, 7], np.uint32),
              np.array([0, 0, 9, 0], np.uint32))
    # invalid op codes and keys >= key_range get 0xFF and change nothing
    op = np.array([3, 255, 1, 0, 2, 1], np.uint8)
    key = np.array([1, 2, R, R + 5, 0xFFFFFFFF, 999], np.uint32)
    r = run_batch(g, o, op, key, np.arange(6, dtype=np.uint32))
    assert r.tolist() == [255, 255, 255, 255, 255, 1]
    # largest and smallest valid keys
    run_batch(g, o, np.array([1, 1], np.uint8), np.array([0, R - 1], np.uint32),
              np.array([1, 2], np.uint32))
    run_batch(g, o, np.array([0, 0, 2, 0], np.uint8), np.array([0, R - 1, 0, 1], np.uint32), None)
    check_same_set(g, o)


def test_contains_only_full_structure():
    """Contains-only on a structure holding every key (C4 shape, small)."""
    R = 200_000
    for N in (32, 16):
        g = GFSL(R, chunk_entries=N)
        o = OracleMap(R)
        prefill(g, o, R, R)
        for op, key, val in workload_batches(R, 100_003, 2, (0, 0, 100)):
            r = run_batch(g, o, op, key, val)
            assert r.all()


def test_zipf_batches():
    R = 100_000
    g = GFSL(R)
    o = OracleMap(R)
    prefill(g, o, R, R // 2)
    for op, key, val in workload_batches(R, 20_000, 4, (10, 10, 80), dist="zipf"):
        run_batch(g, o, op, key, val)
    check_same_set(g, o)


def test_batch_host_matches_device_path():
    R = 10_000
    g1, g2 = GFSL(R), GFSL(R)
    o = OracleMap(R)
    for op, key, val in workload_batches(R, 3_000, 5, (10, 10, 80)):
        r1 = run_batch(g1, o, op, key, val)
        r2 = g2.batch_host(torch.from_numpy(op), torch.from_numpy(key.view(np.int32)),
                           torch.from_numpy(val.view(np.int32))).numpy()
        assert np.array_equal(r1, r2)
    _, k1, v1 = g1.validate()
    _, k2, v2 = g2.validate()
    assert np.array_equal(k1, k2) and np.array_equal(v1, v2)


def test_batch_host_async_pipelined():
    """Many gfsl_batch_host_async calls in flight (two staging slots reused in turn, the
    copy-in of batch b+1 overlapping batch b) give the oracle's answers for every batch."""
    R = 30_000
    g = GFSL(R)
    o = OracleMap(R)
    batches = list(workload_batches(R, 7_001, 9, (20, 20, 60)))
    host = [tuple(torch.from_numpy(np.ascontiguousarray(a).view(np.int32) if a.dtype == np.uint32 else a).pin_memory()
                  for a in b) for b in batches]
    outs = [torch.empty(7_001, dtype=torch.uint8).pin_memory() for _ in batches]
    for h, out in zip(host, outs):
        g.batch_host_async(*h, out=out)
    torch.cuda.synchronize()
    for (op, key, val), out in zip(batches, outs):
        assert np.array_equal(out.numpy(), o.batch(op, key, val))
    check_same_set(g, o)


def test_batch_host_async_interleaved_on_caller_stream():
    """Async host batches (kernels on the library's exec stream, copy-out on its d2h
    stream) interleaved with device batches, all issued on a caller stream: batches apply
    in issue order, and synchronising only the caller stream makes every async result
    visible in host memory (the contract of gfsl_batch_host_async in include/gfsl.h)."""
    R = 20_000
    g = GFSL(R)
    o = OracleMap(R)
    batches = list(workload_batches(R, 5_003, 8, (20, 20, 60)))
    side = torch.cuda.Stream()
    outs, keep = [], []  # inputs stay referenced until the stream is synchronised
    with torch.cuda.stream(side):
        for i, (op, key, val) in enumerate(batches):
            if i % 3 == 1:  # device entry point on the same handle and stream
                d = [torch.from_numpy(np.ascontiguousarray(a).view(np.int32) if a.dtype == np.uint32 else a).cuda()
                     for a in (op, key, val)]
                keep.append(d)
                outs.append(g.batch(*d, stream=side))
            else:
                h = [torch.from_numpy(np.ascontiguousarray(a).view(np.int32) if a.dtype == np.uint32 else a).pin_memory()
                     for a in (op, key, val)]
                keep.append(h)
                outs.append(g.batch_host_async(*h, out=torch.empty(len(op), dtype=torch.uint8).pin_memory(),
                                               stream=side))
    side.synchronize()
    for (op, key, val), out in zip(batches, outs):
        assert np.array_equal(out.cpu().numpy(), o.batch(op, key, val))
    check_same_set(g, o)


@pytest.mark.parametrize("p", [0.25, 0.5])
def test_p_chunk_concurrent(p):
    """p_chunk < 1 with the concurrent update kernel and the paper's structure dynamics."""
    from paper_conf_ppopp_moscovicicp17_b200.gfsl import REBUILD_NEVER
    R = 30_000
    g = GFSL(R, p_chunk=p, rebuild_every=REBUILD_NEVER)
    o = OracleMap(R)
    prefill(g, o, R, R // 2, chunk=5000)
    for op, key, val in workload_batches(R, 6_000 + 3, 6, (20, 20, 60)):
        run_batch(g, o, op, key, val)
        check_same_set(g, o)


def test_long_churn_reclaims_and_stays_exact():
    """Concurrent 50/50 churn for many batches with rebuild + reclamation every batch:
    results stay bit-exact and the level-0 pool stops growing."""
    R = 20_000
    g = GFSL(R, rebuild_every=1)
    o = OracleMap(R)
    prefill(g, o, R, R // 2)
    used = []
    for i, (op, key, val) in enumerate(workload_batches(R, 4_000, 60, (50, 50, 0))):
        run_batch(g, o, op, key, val)
        if i % 10 == 9:
            rep = check_same_set(g, o)
            used.append(rep.pool_used[0])
    assert used[-1] <= used[1] * 1.02 + 8


def test_pool_exhaustion_is_sticky():
    """Inserting far more keys than `capacity` sizes the pool for exhausts it: the next
    call reports GFSL_EPOOL, and so does every later one (the structure is undefined)."""
    from paper_conf_ppopp_moscovicicp17_b200.gfsl import GFSLError, GFSL_EPOOL
    R = 100_000
    g = GFSL(R, capacity=100)
    keys = np.random.default_rng(3).permutation(R)[:20_000].astype(np.uint32)
    with pytest.raises(GFSLError) as ei:
        for s in range(0, keys.size, 2_000):
            k = keys[s:s + 2_000]
            g.batch(*to_dev(np.ones(k.size, np.uint8), k, k))
            torch.cuda.synchronize()
    assert ei.value.status == GFSL_EPOOL
    with pytest.raises(GFSLError):
        g.batch(*to_dev(np.zeros(1, np.uint8), np.zeros(1, np.uint32), None))
