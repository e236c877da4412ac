"""Pins of Oracle-A (oracle/oracle_a.c) against things other than itself (CPU only).

* brute force: a Python dict on tiny key ranges (every op kind, invalid ops, values);
* a direct-address table (numpy presence bitmap + value array) on medium ranges;
* closed forms of S1 batches: #true inserts = |I \\ M|, #true deletes = |D & M|,
  |M'| = |M| + #true inserts - #true deletes; permutation fill / full drain;
* the paper's Contains examples (Fig 4.1) on the key set of the
  worked-example fixture (tests/golden/fig41_contains.txt);
* the contract check (two mutating ops on one key) and invalid-op handling.
"""
import os

import numpy as np
import pytest

from oracle.oracle_a import OracleMap, INVALID

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def brute_batch(M: dict, op, key, val, R):
    """The plain definition of an S1 batch over a Python dict (R1)."""
    res = []
    for o, k in zip(op, key):
        if o > 2 or k >= R:
            res.append(INVALID)
        elif o == 0:
            res.append(int(k in M))
        elif o == 1:
            res.append(int(k not in M))
        else:
            res.append(int(k in M))
    for o, k, v, r in zip(op, key, val, res):
        if r == 1 and o == 1:
            M[k] = v
        elif r == 1 and o == 2:
            del M[k]
    return np.array(res, dtype=np.uint8)


def random_batch(rng, R, B, allow_invalid=True):
    op = rng.integers(0, 3, size=B).astype(np.uint8)
    key = rng.integers(0, R, size=B).astype(np.uint32)
    val = rng.integers(0, 2**32, size=B, dtype=np.uint64).astype(np.uint32)
    # contract: at most one mutating op per key -> turn later duplicates into Contains
    seen = set()
    for i in range(B):
        if op[i] != 0:
            if key[i] in seen:
                op[i] = 0
            seen.add(key[i])
    if allow_invalid and B:
        j = rng.integers(0, B, size=max(1, B // 20))
        op[j[: len(j) // 2]] = rng.integers(3, 256, size=len(j[: len(j) // 2]))
        key[j[len(j) // 2:]] = rng.integers(R, 2**32, size=len(j) - len(j) // 2,
                                            dtype=np.uint64).astype(np.uint32)
    return op, key, val


@pytest.mark.parametrize("R", [1, 2, 7, 64])
def test_oracle_vs_dict_tiny(R):
    rng = np.random.default_rng(R)
    o = OracleMap(R, seed=3)
    M = {}
    for _ in range(400):
        B = int(rng.integers(0, 24))
        op, key, val = random_batch(rng, R, B)
        r = o.batch(op, key, val)
        e = brute_batch(M, op.tolist(), key.tolist(), val.tolist(), R)
        assert np.array_equal(r, e)
        ks, vs = o.export()
        assert ks.tolist() == sorted(M)
        assert vs.tolist() == [M[k] for k in sorted(M)]


def test_oracle_vs_direct_address_table():
    R, B = 100_000, 20_000
    rng = np.random.default_rng(7)
    o = OracleMap(R)
    present = np.zeros(R, dtype=bool)
    value = np.zeros(R, dtype=np.uint32)
    for _ in range(12):
        op, key, val = random_batch(rng, R, B, allow_invalid=False)
        r = o.batch(op, key, val)
        pre = present[key]
        exp = np.where(op == 1, ~pre, pre).astype(np.uint8)
        assert np.array_equal(r, exp)
        ins = (op == 1) & (r == 1)
        dele = (op == 2) & (r == 1)
        present[key[ins]] = True
        value[key[ins]] = val[ins]
        present[key[dele]] = False
        ks, vs = o.export()
        assert np.array_equal(ks, np.flatnonzero(present).astype(np.uint32))
        assert np.array_equal(vs, value[ks])


def test_closed_forms():
    R, B = 5000, 3000
    rng = np.random.default_rng(11)
    o = OracleMap(R)
    # empty start + a permutation of all R keys inserted: every result true, |M| = R
    perm = rng.permutation(R).astype(np.uint32)
    r = o.batch(np.ones(R, np.uint8), perm, perm)
    assert r.all() and len(o) == R
    # |M'| = |M| + #true inserts - #true deletes; #true delete = |D & M|
    for _ in range(10):
        op, key, val = random_batch(rng, R, B, allow_invalid=False)
        before = set(o.export()[0].tolist())
        n0 = len(o)
        r = o.batch(op, key, val)
        ti = int(((op == 1) & (r == 1)).sum())
        td = int(((op == 2) & (r == 1)).sum())
        I = {int(k) for k, p in zip(key, op) if p == 1}
        D = {int(k) for k, p in zip(key, op) if p == 2}
        assert ti == len(I - before)
        assert td == len(D & before)
        assert len(o) == n0 + ti - td
    # full drain
    ks = o.export()[0]
    r = o.batch(np.full(ks.size, 2, np.uint8), ks, None)
    assert r.all() and len(o) == 0


def test_insert_does_not_overwrite_and_contract():
    o = OracleMap(100)
    o.batch(np.array([1], np.uint8), np.array([5], np.uint32), np.array([111], np.uint32))
    r = o.batch(np.array([1], np.uint8), np.array([5], np.uint32), np.array([222], np.uint32))
    assert r.tolist() == [0] and o.get(5) == 111
    with pytest.raises(ValueError):
        o.batch(np.array([1, 2], np.uint8), np.array([9, 9], np.uint32), np.array([1, 2], np.uint32))
    assert len(o) == 1  # a violating batch applies nothing
    # Contains + one mutation of the same key is inside the contract; S1 answers "before"
    r = o.batch(np.array([0, 2, 0], np.uint8), np.array([5, 5, 5], np.uint32), None)
    assert r.tolist() == [1, 1, 1] and len(o) == 0


def _read_golden(name):
    rows = {}
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.split("#", 1)[0].strip()
            if not line:
                continue
            k, v = line.split(":", 1)
            rows[k.strip()] = [int(x) for x in v.split()]
    return rows


def test_paper_contains_examples():
    """Fig 4.1: on the fixture's key set, Contains(17) is true and
    Contains(52), Contains(70) are false."""
    g = _read_golden("fig41_contains.txt")
    keys = np.array(g["keys"], np.uint32)
    o = OracleMap(100)
    o.batch(np.ones(keys.size, np.uint8), keys, keys)
    q = np.array(g["query"], np.uint32)
    r = o.batch(np.zeros(q.size, np.uint8), q, None)
    assert r.tolist() == g["expect"]


# ---- combining semantics (R26) ----

def brute_batch_seq(M: dict, op, key, val, R):
    """Plain definition of R26 over a Python dict: Contains against the pre-batch map,
    then every Insert/Delete one at a time in input order."""
    pre = set(M)
    res = []
    for o, k in zip(op, key):
        res.append(INVALID if (o > 2 or k >= R) else (int(k in pre) if o == 0 else None))
    for i, (o, k, v) in enumerate(zip(op, key, val)):
        if res[i] is not None:
            continue
        if o == 1:
            res[i] = int(k not in M)
            if k not in M:
                M[k] = v
        else:
            res[i] = int(k in M)
            M.pop(k, None)
    return np.array(res, dtype=np.uint8)


@pytest.mark.parametrize("R", [1, 3, 16, 200])
def test_oracle_seq_vs_dict_with_duplicates(R):
    rng = np.random.default_rng(100 + R)
    o = OracleMap(R, seed=5)
    M = {}
    for _ in range(300):
        B = int(rng.integers(0, 40))
        op = rng.integers(0, 3, size=B).astype(np.uint8)
        key = rng.integers(0, R + 1, size=B).astype(np.uint32)  # R = invalid
        val = rng.integers(0, 2**32, size=B, dtype=np.uint64).astype(np.uint32)
        r = o.batch(op, key, val, combine=True)
        e = brute_batch_seq(M, op.tolist(), key.tolist(), val.tolist(), R)
        assert np.array_equal(r, e)
        ks, vs = o.export()
        assert ks.tolist() == sorted(M)
        assert vs.tolist() == [M[k] for k in sorted(M)]


def test_oracle_seq_equals_s1_under_contract():
    R, B = 3000, 2000
    rng = np.random.default_rng(21)
    a, b = OracleMap(R), OracleMap(R)
    for _ in range(10):
        op, key, val = random_batch(rng, R, B)
        assert np.array_equal(a.batch(op, key, val), b.batch(op, key, val, combine=True))
    assert np.array_equal(a.export()[0], b.export()[0])
    assert np.array_equal(a.export()[1], b.export()[1])


def test_oracle_seq_per_key_automaton():
    """Hand-worked chains on one key (Insert false iff present, Delete false iff absent,
    Alg 4.5 l.2-4 / Alg 4.11 l.3-5; a present key's value is never overwritten)."""
    I, D, C = 1, 2, 0
    o = OracleMap(10)
    # absent: I(5) I(6) D I(7) C -> 1 0 1 1 | C sees the pre-batch map -> 0; final 7
    r = o.batch(np.array([I, I, D, I, C], np.uint8), np.full(5, 4, np.uint32),
                np.array([5, 6, 0, 7, 0], np.uint32), combine=True)
    assert r.tolist() == [1, 0, 1, 1, 0] and o.get(4) == 7
    # present (7): D D I(8) I(9) -> 1 0 1 0; final 8
    r = o.batch(np.array([D, D, I, I], np.uint8), np.full(4, 4, np.uint32),
                np.array([0, 0, 8, 9], np.uint32), combine=True)
    assert r.tolist() == [1, 0, 1, 0] and o.get(4) == 8
    # present: I(1) D C -> 0 1 1; final absent
    r = o.batch(np.array([I, D, C], np.uint8), np.full(3, 4, np.uint32),
                np.array([1, 0, 0], np.uint32), combine=True)
    assert r.tolist() == [0, 1, 1] and o.get(4) is None and len(o) == 0
