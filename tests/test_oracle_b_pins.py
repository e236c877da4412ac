"""Pins of Oracle-B that do not go through its own code (CPU only).

Each test fixes one function of oracle/oracle_b.py against something other than itself:
a worked example or a printed intermediate state of the paper, a hand-worked fixture, or
a plain re-derivation written here from the definition (SURVEY 8(c) "What pins each part").

* restart of Contains(70) when Deletes of 59 and 68 run between its down-step A -> C and
  the read of C (Alg 4.2 l.25)                       -> search()
* write orders: Insert right to left (Alg 4.7 l.7-10), Delete without merge left to
  right with the max first, split copy -> link -> EMPTY (Alg 4.9 l.27-32,
  P:705), merge in descending index with F = [24, 26, EMPTY, 26] after the first write
  (P:947-951), zombie mark before F's unlock (Alg 4.12 l.21-25)     -> execute_*, split
* a hand-worked splitRemove (Alg 4.12 l.16-19)             -> remove_from_chunk
* the lazy zombie redirect and head-array update (Alg 4.6 l.10-20)
                                                                    -> redirect_zombie
* searchDown to a level (Alg 4.10 l.4) against a brute-force enclosing chunk
                                                                    -> search_down_to_level
* the upper-level rebuild (R24) against a plain re-derivation from the level-0 chain
                                                                    -> rebuild
* the between-batch zombie unlinking (R23) and reclamation (R25) by their defining
  properties                                                        -> upkeep, reclaim
* the invariant checker itself: each of V5 / V6 / V11 / V12 fires on a planted fault
"""
import numpy as np
import pytest

from oracle.oracle_a import OracleMap
from oracle.oracle_b import (E, EMPTY, FREE, HELD, INF, K, NEG_INF, NULL, V, ZOMBIE,
                             GFSLModel)
from paper_conf_ppopp_moscovicicp17_b200.workload import SEED_BASE, Workload
from tests import gfsl_fixtures as fx


def ukeys(m, c):
    """User keys of a chunk's DATA entries in slot order (None = EMPTY, '-inf')."""
    out = []
    for e in m.pool[c][: m.DSIZE]:
        k = K(e)
        out.append(None if k == INF else ("-inf" if k == NEG_INF else k - 1))
    return out


def churned_model(N=16, R=2000, batches=20, mix=(40, 40, 20), rebuild_every=0, seed=0):
    m = GFSLModel(N, R, cap_bottom=4000, cap_upper=1000, rebuild_every=rebuild_every)
    w = Workload(R, 200, mix=mix, seed=SEED_BASE + 500 + seed)
    for b in range(batches):
        op, key, val, _ = w.make_batch(b)
        m.batch(op.numpy().tolist(), key.numpy().astype(np.uint32).tolist(),
                val.numpy().astype(np.uint32).tolist())
    return m


# ---------------------------------------------------------------- WE-C70r

def test_contains_70_restarts_when_59_and_68_are_deleted_mid_traversal():
    m, n = fx.build(fx.FC, 6)
    fired = []

    def hook(c):
        # the team has stepped down from A to C and stalls before reading C
        if c == n["C"] and not fired:
            fired.append(True)
            assert m.batch([2, 2], [59, 68]) == [1, 1]   # a concurrent team's Deletes
    found, path, top = m.search(70 + 1, hook=hook)
    assert fired and m.restarts == 1                  # backtrack with no prevKv -> restart
    assert not found
    # after the restart: 59 left level 2 (A holds only -inf: height 1), so the traversal
    # starts at B, steps laterally to C (75, 80), backtracks to 47 -> H, and walks level 0
    assert m.trace == [n["B"], n["C"], n["H"], n["I"], n["J"]]
    assert m.height() == 1
    assert ukeys(m, n["C"])[:2] == [75, 80]
    # on the quiescent structure the same search does not restart (R1)
    r0 = m.restarts
    assert m.search(70 + 1)[0] is False and m.restarts == r0


# ---------------------------------------------------------------- write orders

def test_insert_15_writes_right_to_left():
    """Alg 4.7 l.7-10: lanes DSIZE-1 .. insertIdx, each writes its left neighbour's entry;
    the first write duplicates 21 (a key may appear twice, higher lanes win)."""
    m, n = fx.build(fx.FI, 6)
    e = n["E"]
    m.wtrace = []
    assert m.batch([1], [15], [777]) == [1]
    data = [(i, K(x) - 1) for c, i, x in m.wtrace if c == e and i < m.DSIZE]
    assert data == [(3, 21), (2, 17), (1, 15)]


def test_delete_no_merge_writes_left_to_right_max_first():
    m, n = fx.build(fx.FDN, 12)
    e = n["E"]
    m.wtrace = []
    assert m.batch([2], [13]) == [1]                  # Fig 4.6
    data = [(i, None if K(x) == INF else K(x) - 1) for c, i, x in m.wtrace
            if c == e and i < m.DSIZE]
    assert data == [(0, 17), (1, 21), (2, 22), (3, None)]
    m2, n2 = fx.build(fx.FDN, 12)
    e2 = n2["E"]
    m2.wtrace = []
    assert m2.batch([2], [22]) == [1]                 # the max goes first
    ws = [(i, x) for c, i, x in m2.wtrace if c == e2 and i != m2.LOCK]
    assert ws[0] == (m2.NEXT, E(21 + 1, n2["F"]))
    assert ws[1:] == [(3, EMPTY)]


def test_split_copy_then_link_then_empty():
    m, n = fx.build(fx.FS, 6)
    b = n["B"]
    m.wtrace = []
    assert m.batch([1], [22], [5]) == [1]
    d = m.nxt(b)
    ws = [(c, i) for c, i, _ in m.wtrace if i != m.LOCK]
    link = ws.index((b, m.NEXT))
    copies = [j for j, (c, i) in enumerate(ws) if c == d and i < m.DSIZE]
    empties = [j for j, (c, i) in enumerate(ws) if c == b and i in (2, 3) and j < len(ws)]
    assert ws.index((d, m.NEXT)) < copies[0]          # preSplit: new chunk -> next first
    assert max(copies[:2]) < link                      # splitCopy before the link (l.27-30)
    assert all(j > link for j in empties[:2])          # setMovedValsEmpty after it (l.32)


def test_merge_fig45_descending_order_and_printed_state():
    m, n = fx.build(fx.FD, 12)
    e, f = n["E"], n["F"]
    m.wtrace = []
    assert m.batch([2], [13]) == [1]
    fw = [(j, i, x) for j, (c, i, x) in enumerate(m.wtrace) if c == f and i < m.DSIZE]
    assert [i for _, i, _ in fw] == [3, 2, 1, 0]       # descending index
    # replay the first write onto F as it was: [24, 26, EMPTY, 26]
    before = [24, 26, None, None]
    j0, i0, x0 = fw[0]
    before[i0] = K(x0) - 1
    assert before == [24, 26, None, 26]
    assert ukeys(m, f)[:4] == [17, 21, 24, 26]
    zmark = [j for j, (c, i, x) in enumerate(m.wtrace) if c == e and i == m.LOCK and K(x) == ZOMBIE]
    funlock = [j for j, (c, i, x) in enumerate(m.wtrace) if c == f and i == m.LOCK and K(x) == FREE]
    assert zmark and funlock and fw[-1][0] < zmark[0] < funlock[-1]   # Alg 4.12 l.21-25


# ---------------------------------------------------------------- splitRemove

# N = 12 (DSIZE 10, merge threshold floor(10/3) = 3, split move from index DSIZE/2 = 5).
# Level 1: B = [-inf -> E0, 13 -> E, 24 -> F, 36 -> F]; level 0: E0 = [-inf, 5, 8],
# E = [13, 17, 21], F = [24, 26, 28, 30, 32, 34, 36, 38, 40] (9 keys, the last chunk).
FSR = {
    1: [("B", [("-inf", "E0"), (13, "E"), (24, "F"), (36, "F")])],
    0: [("E0", [5, 8]), ("E", [13, 17, 21]), ("F", [24, 26, 28, 30, 32, 34, 36, 38, 40])],
}


def test_split_remove_hand_worked():
    """Delete 13, worked by hand from Alg 4.11-4.12:
    level 1: B holds 4 entries (> 3): shift left -> B = [-inf, 24, 36];
    level 0: E holds 3 entries (<= 3): merge into F; 9 + 3 - 1 = 11 > DSIZE, so F is
    split first (splitRemove, no key inserted, no raise): F keeps [24 .. 32] (max 32), the
    new chunk G gets [34, 36, 38, 40] (max inf, the last chunk: F was last), counter+1;
    then E's 17, 21 move into F -> [17, 21, 24, 26, 28, 30, 32]; E a zombie keeping
    [13, 17, 21] and NEXT = F; counter-1; updateDownPtrs moves 36's pointer to G (Alg
    4.10); upkeep (R23) then points E0 past the zombie to F."""
    m, n = fx.build(FSR, 12)
    b, e0, e, f = n["B"], n["E0"], n["E"], n["F"]
    assert m.counter[0] == 3 and m.counter[1] == 1
    assert m.batch([2], [13]) == [1]
    assert ukeys(m, b)[:3] == ["-inf", 24, 36] and ukeys(m, b)[3] is None
    g = m.nxt(f)
    assert g != NULL and g >= m.cap_upper
    assert ukeys(m, f)[:8] == [17, 21, 24, 26, 28, 30, 32, None]
    assert m.mx(f) == 32 + 1
    assert ukeys(m, g)[:5] == [34, 36, 38, 40, None]
    assert m.mx(g) == INF and m.nxt(g) == NULL
    assert m.zombie(e) and ukeys(m, e)[:4] == [13, 17, 21, None] and m.nxt(e) == f
    ptr = {K(x) - 1: V(x) for x in m.pool[b][: m.DSIZE] if K(x) not in (INF, NEG_INF)}
    assert ptr == {24: f, 36: g}
    assert m.nxt(e0) == f                             # upkeep (R23)
    assert m.counter[0] == 3                          # +1 split, -1 merge
    assert m.level_keys(1) == [25, 37]
    assert m.check_invariants() == []


# ---------------------------------------------------------------- zombie redirect

def test_find_and_lock_enclosing_unlinks_a_zombie_chain_and_fixes_the_head():
    """Alg 4.6 l.10-20 / R15: a team that steps laterally into a zombie redirects the
    previous chunk past the whole zombie chain (try-lock succeeds when sequential); a
    zombie first chunk is replaced in the head array."""
    m, n = fx.build(fx.FC, 6)
    h, i, j, k = n["H"], n["I"], n["J"], n["K"]
    for z in (i, j):                                  # I and J zombies, as after merges
        m.pool[z][m.LOCK] = E(ZOMBIE, 1)
    zbytes = [list(m.pool[z]) for z in (i, j)]
    c = m.find_and_lock_enclosing(h, 76, 0)           # 75 + 1: encloses in K
    assert c == k and m.state(k) == HELD
    assert m.nxt(h) == k                              # H -> K, past I and J
    assert [list(m.pool[z]) for z in (i, j)] == zbytes   # zombies untouched
    assert m.state(h) == FREE
    m.unlock(k)
    e0 = m.head[0]                                    # now the first chunk: a zombie
    m.pool[e0][m.LOCK] = E(ZOMBIE, 1)
    c = m.find_and_lock_enclosing(e0, 4, 0)           # 3 + 1
    assert m.head[0] == n["E"] and c == n["E"]        # updateHeadArray (Alg 4.6 l.15)


# ---------------------------------------------------------------- searchDown to a level

def brute_enclosing(m, level, k):
    """The first non-zombie chunk of the level (in chain order) with max >= k."""
    for c in m.level_chain(level):
        if not m.zombie(c) and m.mx(c) >= k:
            return c
    raise AssertionError


@pytest.mark.parametrize("N", [6, 16])
def test_search_down_to_level_reaches_the_enclosing_chunk(N):
    m = churned_model(N=N, R=600 if N == 6 else 3000, batches=15, seed=N)
    H = m.height()
    assert H >= 2
    for L in range(0, H):
        for key in range(0, m.key_range, 7):
            k = key + 1
            c = m.search_down_to_level(L, k)
            enc = brute_enclosing(m, L, k)
            hops = 0
            while c != enc:                            # only lateral steps past chunks
                assert m.zombie(c) or m.mx(c) < k      # that cannot enclose k
                c, hops = m.nxt(c), hops + 1
                assert c != NULL and hops < 10_000


# ---------------------------------------------------------------- rebuild (R24)

def plain_upper_levels(m):
    """R24 written out from its definition, without the model's closed form: level 1 =
    -inf + the min key of every live level-0 chunk after the first (in chain order),
    F = N - 4 per chunk; level l+1 = -inf + the first key of every chunk of level l after
    its first; stop when a level fits one chunk or level N-1 (MAX_LEVEL = N) is
    reached.  Returns [(keys, targets)] per level,
    targets as ("L0", chunk) for level 1 and ("chunk", j) (chunk j of the level below)."""
    F = m.N - 4
    l0 = [c for c in m.level_chain(0) if not m.zombie(c)]
    live = [(m.keys(c)[0], c) for c in l0[1:] if m.keys(c)[0] != INF]
    levels = [[(NEG_INF, ("L0", l0[0]))] + [(k, ("L0", c)) for k, c in live]]
    while len(levels[-1]) > F and len(levels) < m.N - 1:
        prev = levels[-1]
        groups = [prev[i:i + F] for i in range(0, len(prev), F)]
        levels.append([(NEG_INF, ("chunk", 0))] + [(g[0][0], ("chunk", j))
                                                   for j, g in enumerate(groups) if j > 0])
    return levels


@pytest.mark.parametrize("N,seed", [(6, 1), (12, 2), (16, 3), (32, 4)])
def test_rebuild_matches_a_plain_rederivation(N, seed):
    m = churned_model(N=N, R=500 if N <= 12 else 6000, batches=12, seed=seed,
                      mix=(50, 30, 20))
    m.rebuild()
    exp = plain_upper_levels(m)
    F = m.N - 4
    for l, want in enumerate(exp, start=1):
        chain = m.level_chain(l)
        got = [(K(x), V(x)) for c in chain for x in m.pool[c][: m.DSIZE] if K(x) != INF]
        assert [k for k, _ in got] == [k for k, _ in want], f"level {l} keys"
        sizes = [sum(1 for x in m.pool[c][: m.DSIZE] if K(x) != INF) for c in chain]
        assert all(s == F for s in sizes[:-1]) and 1 <= sizes[-1] <= F
        below = m.level_chain(l - 1)
        for (k, tgt), (_, (kind, ref)) in zip(got, want):
            assert tgt == (ref if kind == "L0" else below[ref]), f"level {l} key {k}"
        assert m.counter[l] == (len(chain) if len(want) > 1 else 0)   # R9
    top = len(exp) if len(exp[-1]) > 1 else len(exp) - 1
    assert m.height() == top
    for l in range(len(exp) + 1, m.N):                 # levels above: only -inf
        assert m.level_keys(l) == [] and m.counter[l] == 0
    assert m.check_invariants() == []


# ---------------------------------------------------------------- upkeep (R23), reclaim (R25)

def test_upkeep_unlinks_zombies_and_changes_nothing_else():
    R, N = 800, 12
    m = GFSLModel(N, R, cap_bottom=4000, cap_upper=1000)
    real_upkeep = m.upkeep
    m.upkeep = lambda: None                           # run the batch without it
    w = Workload(R, 300, mix=(30, 70, 0), seed=SEED_BASE + 71)
    seen_zombie_link = False
    for b in range(10):
        op, key, val, _ = w.make_batch(b)
        m.batch(op.numpy().tolist(), key.numpy().astype(np.uint32).tolist(),
                val.numpy().astype(np.uint32).tolist())
        live = {l: [c for c in m.level_chain(l) if not m.zombie(c)] for l in range(N)}
        used = list(range(m.bump[1])) + [m.cap_upper + i for i in range(m.bump[0])]
        seen_zombie_link |= any(not m.zombie(c) and m.nxt(c) != NULL and m.zombie(m.nxt(c))
                                for c in used)
        before = [list(ch) for ch in m.pool]
        real_upkeep()
        for c in used:
            if m.zombie(c):
                assert m.pool[c] == before[c]          # zombies untouched
            else:
                assert m.pool[c][: m.NEXT] == before[c][: m.NEXT]
                assert m.mx(c) == K(before[c][m.NEXT])
                assert m.nxt(c) == NULL or not m.zombie(m.nxt(c))
        for l in range(N):
            assert not m.zombie(m.head[l])
            assert m.level_chain(l) == live[l]         # same live chunks, no zombie left
        assert m.check_invariants() == []
    assert seen_zombie_link


def test_reclaim_recycles_exactly_the_unreachable_zombies():
    m = churned_model(N=12, R=500, batches=12, mix=(30, 60, 10), seed=9)
    zombies = sorted(m.cap_upper + i for i in range(m.bump[0]) if m.zombie(m.cap_upper + i))
    assert zombies
    m.rebuild()
    assert not (set(zombies) & m.reachable())         # nothing points at them any more
    m.reclaim()
    assert m.free[m.free_taken:] == zombies           # ascending, all of them
    for c in zombies:
        assert m.pool[c] == [EMPTY] * (m.N - 1) + [E(HELD, 0)]   # P:237 allocated state
    bump0 = m.bump[0]
    got = [m.alloc(0) for _ in range(len(zombies))]
    assert got == zombies and m.bump[0] == bump0      # allocation takes them first
    assert m.alloc(0) == m.cap_upper + bump0          # then the bump counter


# ---------------------------------------------------------------- the checker fires

def test_invariant_checker_detects_planted_faults():
    m = churned_model(N=12, R=500, batches=10, mix=(40, 40, 20), seed=5)
    assert m.check_invariants() == []
    snap = m.snapshot()
    # V5: a level-1 down pointer aimed to the right of its key's chunk
    c1 = [c for c in m.level_chain(1) if not m.zombie(c)][0]
    i = next(i for i, x in enumerate(m.pool[c1][: m.DSIZE]) if K(x) not in (INF, NEG_INF))
    saved = m.pool[c1][i]
    last0 = m.level_chain(0)[-1]
    m.pool[c1][i] = E(K(saved), last0)
    assert any(v.startswith("V5") for v in m.check_invariants())
    m.pool[c1][i] = saved
    # V6: a max field that grew
    c0 = [c for c in m.level_chain(0) if not m.zombie(c) and m.nxt(c) != NULL][0]
    saved = m.pool[c0][m.NEXT]
    m.pool[c0][m.NEXT] = E(K(saved) + 1, V(saved))
    assert any(v.startswith("V6") for v in m.check_invariants(prev=snap))
    m.pool[c0][m.NEXT] = saved
    # V11: a zombie whose bytes changed
    z = next(c for c in snap["zombie"])
    saved = m.pool[z][0]
    m.pool[z][0] = E(K(saved) ^ 1, V(saved))
    assert any(v.startswith("V11") for v in m.check_invariants(prev=snap))
    m.pool[z][0] = saved
    # V12: a reachable index beyond the bump counter
    saved = m.pool[c0][m.NEXT]
    m.pool[c0][m.NEXT] = E(K(saved), m.cap_upper + m.bump[0] + 3)
    assert any(v.startswith("V12") for v in m.check_invariants())
    m.pool[c0][m.NEXT] = saved
    assert m.check_invariants(prev=snap) == []


def test_paper_delete_checks_every_level_from_the_height():
    """Alg 4.11 l.12-20: a key raised since the snapshot (as minK of a split) is
    still removed from the level it reached; results and sets equal Oracle-A's."""
    R, N = 300, 6
    m = GFSLModel(N, R, cap_bottom=4000, cap_upper=1000)
    m.check_each_op = True
    o = OracleMap(R)
    rng = np.random.default_rng(3)
    for b in range(40):
        keys = rng.choice(R, 60, replace=False).astype(np.uint32)
        ops = rng.choice([0, 1, 2], 60, p=[0.2, 0.5, 0.3]).astype(np.uint8)
        vals = rng.integers(0, 2**32, 60, dtype=np.uint64).astype(np.uint32)
        assert m.batch(ops.tolist(), keys.tolist(), vals.tolist()) == o.batch(ops, keys, vals).tolist()
    ks, vs = m.export()
    ok, ov = o.export()
    assert ks == ok.tolist() and vs == ov.tolist()
