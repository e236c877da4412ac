"""Pins of Oracle-B (oracle/oracle_b.py), the step-by-step GFSL model (CPU only).

* the paper's worked examples on the fixtures of SURVEY Appendix B (tests/gfsl_fixtures.py):
  Fig 4.1 Contains 17 / 52 / 70 with the exact chunks read;
  Fig 4.2/4.3 Insert 15 without a split;
  Fig 4.4 Insert 22 with a split, key 20's down pointer redirected, 22 raised (P:705-707,
  P:740); Fig 4.5 Delete 13 with a merge; Fig 4.6
  Delete without a merge, incl. the max-field update;
* results and final sets equal Oracle-A's on random batch sequences (N = 6, 12, 16, 32),
  with the model's own invariant check after every batch;
* a special case: while every key fits one chunk, level 0 is one sorted array.
"""
import numpy as np
import pytest

from oracle.oracle_a import OracleMap
from oracle.oracle_b import GFSLModel, INF, NEG_INF, NULL, ZOMBIE, K, V
from paper_conf_ppopp_moscovicicp17_b200.workload import Workload, SEED_BASE
from tests import gfsl_fixtures as fx


def internal(keys):
    return [k + 1 for k in keys]


def level0_keys(m, c):
    return [k for k in m.keys(c) if k != INF]


def test_fig41_contains_paths():
    m, n = fx.build(fx.FC, 6)
    f, path, top = m.search(17 + 1)
    assert f and m.trace == [n["A"], n["B"], n["E"]]
    assert m.eq_idx(n["E"], 18) == 2                               # "T2 sees key 17"
    f, path, top = m.search(52 + 1)
    assert not f and m.trace == [n["A"], n["B"], n["C"], n["H"], n["I"]]
    f, path, top = m.search(70 + 1)
    assert not f and m.trace == [n["A"], n["C"], n["J"]]           # P:429 (no injection)


def test_fig42_insert_15_shifts_right():
    m, n = fx.build(fx.FI, 6)
    res = m.batch([1], [15], [777])
    assert res == [1]
    assert level0_keys(m, n["E"]) == internal([10, 15, 17, 21])   # Fig 4.3
    assert m.mx(n["E"]) == 21 + 1                                   # max untouched
    assert m.bump == [1 + 8, 5 + 1]                                 # no allocation: no split
    assert m.check_invariants() == []


def test_fig44_split_on_insert_22():
    m, n = fx.build(fx.FS, 6)
    b = n["B"]
    res = m.batch([1], [22], [5])
    assert res == [1]
    d = m.nxt(b)                                                     # the new chunk D
    assert level0_keys(m, b) == [NEG_INF] + internal([12])          # B keeps -inf, 12
    assert m.mx(b) == 12 + 1
    assert level0_keys(m, d) == internal([20, 22, 25])             # 20, 25 moved; 22 in D
    assert m.mx(d) == INF and m.nxt(d) == NULL                      # D is the last chunk
    a = n["A"]
    up = {K(e): V(e) for e in m.pool[a][: m.DSIZE] if K(e) != INF}
    assert up[20 + 1] == d                                          # caption: 20's pointer -> D
    assert up[22 + 1] == d                                          # raised max(22, 20)
    assert m.counter[0] == 2
    assert m.check_invariants() == []


def test_fig45_delete_13_with_merge():
    m, n = fx.build(fx.FD, 12)
    res = m.batch([2], [13])
    assert res == [1]
    e, f, b = n["E"], n["F"], n["B"]
    assert m.zombie(e)                                               # E marked zombie
    assert level0_keys(m, e) == internal([13, 17, 21])             # contents kept
    assert level0_keys(m, f) == internal([17, 21, 24, 26])         # merged into F (Fig 4.5c)
    assert [K(x) for x in m.pool[b][: m.DSIZE] if K(x) != INF] == [NEG_INF, 24 + 1]  # B: 13 gone
    assert m.counter[0] == 2                                        # one chunk less
    assert m.check_invariants() == []
    assert m.batch([0, 0, 0], [17, 13, 26]) == [1, 0, 1]            # 17 via the zombie's NEXT


def test_fig46_delete_without_merge_and_max_update():
    m, n = fx.build(fx.FDN, 12)
    assert m.batch([2], [13]) == [1]
    e = n["E"]
    assert not m.zombie(e)
    assert level0_keys(m, e) == internal([17, 21, 22])             # shift left (Fig 4.6)
    m2, n2 = fx.build(fx.FDN, 12)
    assert m2.batch([2], [22]) == [1]                               # remove a non-last max
    assert level0_keys(m2, n2["E"]) == internal([13, 17, 21])
    assert m2.mx(n2["E"]) == 21 + 1                                 # max follows
    assert m2.check_invariants() == []


def test_single_chunk_is_a_sorted_array():
    m = GFSLModel(32, 1000, 64, 64)
    rng = np.random.default_rng(1)
    keys = rng.choice(1000, 30 - 1, replace=False)
    for k in keys:
        m.batch([1], [int(k)], [int(k)])
    assert level0_keys(m, m.head[0]) == [NEG_INF] + sorted(int(k) + 1 for k in keys)
    assert m.height() == 0 and m.bump == [1, 31]


@pytest.mark.parametrize("N", [6, 12, 16, 32])
def test_model_matches_oracle_a(N):
    R = 400 if N <= 12 else 2000
    m = GFSLModel(N, R, cap_bottom=4000, cap_upper=1000)
    m.check_each_op = True          # V1-V5, V7-V9, V12 after every Insert / Delete
    o = OracleMap(R)
    w = Workload(R, 150, mix=(35, 35, 30), seed=SEED_BASE + N)
    snap = m.snapshot()
    for b in range(30):
        op, key, val, _ = w.make_batch(b)
        opn, kn, vn = op.numpy(), key.numpy().astype(np.uint32), val.numpy().astype(np.uint32)
        r = m.batch(opn.tolist(), kn.tolist(), vn.tolist())
        e = o.batch(opn, kn, vn)
        assert r == e.tolist()
        ks, vs = m.export()
        ok, ov = o.export()
        assert ks == ok.tolist() and vs == ov.tolist()
        assert m.check_invariants(prev=snap) == []   # + V6 / V11 across the batch
        snap = m.snapshot()
    assert m.restarts == 0


@pytest.mark.parametrize("N,every", [(6, 1), (12, 2), (16, 1), (32, 3)])
def test_model_with_rebuild_matches_oracle_a(N, every):
    """R24: rebuilding the upper levels between batches changes no result and keeps
    every invariant; after a rebuild every level-0 chunk is the target of a level-1 key."""
    R = 400 if N <= 12 else 2000
    m = GFSLModel(N, R, cap_bottom=4000, cap_upper=1000, rebuild_every=every)
    m.check_each_op = True
    o = OracleMap(R)
    w = Workload(R, 150, mix=(35, 35, 30), seed=SEED_BASE + 3 * N)
    for b in range(24):
        snap = m.snapshot()
        op, key, val, _ = w.make_batch(b)
        opn, kn, vn = op.numpy(), key.numpy().astype(np.uint32), val.numpy().astype(np.uint32)
        assert m.batch(opn.tolist(), kn.tolist(), vn.tolist()) == o.batch(opn, kn, vn).tolist()
        ks, vs = m.export()
        ok, ov = o.export()
        assert ks == ok.tolist() and vs == ov.tolist()
        assert m.check_invariants(prev=snap) == []
        if (b + 1) % every == 0:
            l0 = [c for c in m.level_chain(0) if not m.zombie(c)][1:]
            targets = {V(e) for c in m.level_chain(1) for e in m.pool[c][: m.DSIZE] if K(e) != INF}
            assert all(c in targets for c in l0 if m.keys(c)[0] != INF)


def test_reclaimed_chunks_bound_the_pool():
    """R25: with zombies recycled after each rebuild, sustained 50/50 churn stops growing
    the level-0 pool; without reclamation (no rebuild) every merge leaks a chunk."""
    R, N = 600, 16
    o = OracleMap(R)
    runs = {}
    for every in (1, 0):
        m = GFSLModel(N, R, cap_bottom=20000, cap_upper=4000, rebuild_every=every)
        w = Workload(R, 200, mix=(50, 50, 0), seed=SEED_BASE + 99)
        used = []
        for b in range(120):
            op, key, val, _ = w.make_batch(b)
            m.batch(op.numpy().tolist(), key.numpy().astype(np.uint32).tolist(),
                    val.numpy().astype(np.uint32).tolist())
            used.append(m.bump[0])
        assert m.check_invariants() == []
        runs[every] = used
    assert runs[1][-1] == runs[1][60]          # plateau with reclamation
    assert runs[0][-1] > runs[0][60] + 20      # keeps leaking without it


@pytest.mark.parametrize("N,p", [(6, 0.5), (16, 0.25), (32, 0.5)])
def test_model_with_p_chunk_matches_oracle_a(N, p):
    """p_chunk < 1 (R28): results, final set and invariants unchanged; fewer
    keys reach the upper levels than at p_chunk = 1 (the raise is a coin flip per split)."""
    R = 400 if N <= 12 else 2000
    q = int(p * 2**32)
    m = GFSLModel(N, R, cap_bottom=4000, cap_upper=1000, p_chunk_q32=q)
    m1 = GFSLModel(N, R, cap_bottom=4000, cap_upper=1000)
    o = OracleMap(R)
    w = Workload(R, 150, mix=(45, 25, 30), seed=SEED_BASE + 7 * N)
    for b in range(30):
        op, key, val, _ = w.make_batch(b)
        opn, kn, vn = op.numpy(), key.numpy().astype(np.uint32), val.numpy().astype(np.uint32)
        r = m.batch(opn.tolist(), kn.tolist(), vn.tolist())
        m1.batch(opn.tolist(), kn.tolist(), vn.tolist())
        assert r == o.batch(opn, kn, vn).tolist()
        assert m.check_invariants() == []
    ks, vs = m.export()
    ok, ov = o.export()
    assert ks == ok.tolist() and vs == ov.tolist()
    upper = lambda mm: sum(len(mm.level_keys(l)) for l in range(1, mm.N))  # noqa: E731
    assert upper(m) < upper(m1)


def test_raise_draw_is_uniform():
    """The draw of R28 is a fixed bijective mix of its input: about p of all (key, level)
    pairs are raised, and the fraction is monotone in p."""
    from oracle.oracle_b import raise_draw
    d = np.array([raise_draw(k, lv) for k in range(1, 20001) for lv in range(3)], np.uint64)
    for p in (0.25, 0.5, 0.75):
        assert abs(float((d < int(p * 2**32)).mean()) - p) < 0.01
