"""Pin of the per-key linearizability checker (tests/linearize.py) by brute force: for every
small list of ops on one key, every start state and every result vector, the checker says
yes iff some order of the ops, run sequentially, gives exactly those results and final
state (CPU only)."""
import itertools

from tests.linearize import linearizable


def sequential(p, v, ops, vals, order):
    res = [None] * len(ops)
    for i in order:
        o = ops[i]
        if o == 0:
            res[i] = int(p)
        elif o == 1:
            res[i] = int(not p)
            if not p:
                p, v = True, vals[i]
        else:
            res[i] = int(p)
            p = False
    return res, p, v


def test_checker_equals_brute_force():
    cases = 0
    for n in range(1, 5):
        for ops in itertools.product([0, 1, 2], repeat=n):
            vals = [10 + i for i in range(n)]
            for p0 in (False, True):
                reachable = set()
                for order in itertools.permutations(range(n)):
                    r, p, v = sequential(p0, 7, list(ops), vals, order)
                    reachable.add((tuple(r), p, v if p else None))
                for res in itertools.product([0, 1], repeat=n):
                    for fp in (False, True):
                        for fv in ([7] + vals if fp else [None]):
                            want = (tuple(res), fp, fv) in reachable
                            got = linearizable(p0, 7, list(ops), list(res), vals, fp,
                                               fv if fv is not None else 0)
                            assert got == want, (ops, p0, res, fp, fv)
                            cases += 1
    assert cases > 1000
