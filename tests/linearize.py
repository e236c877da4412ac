"""Per-key linearizability of one batch's results (test helper; no GPU, no oracle code).

The sequential definitions are the paper's: Contains(k) -> k present (Alg 4.1), Insert(k, v)
-> false iff present, no overwrite (Alg 4.5 l.2-4), Delete(k) -> false iff absent
(Alg 4.11 l.3-5).  Pinned against brute force over every order of small op lists in
tests/test_linearize.py.
"""


def linearizable(p0, v0, ops, res, vals, final_present, final_value):
    """Is there an order of one key's ops (Contains / Insert / Delete with their results)
    consistent with the sequential definitions (Alg 4.1 / 4.5 l.2-4 / 4.11 l.3-5) that
    starts in (p0, v0) and ends in (final_present, final_value)?  The successful Inserts
    and Deletes alternate from p0; failed ops and Contains need an interval of the state
    they saw; the final value is that of the last successful Insert (or v0)."""
    ti = sum(1 for o, r in zip(ops, res) if o == 1 and r == 1)
    td = sum(1 for o, r in zip(ops, res) if o == 2 and r == 1)
    if p0 and not (td == ti or td == ti + 1):
        return False
    if not p0 and not (ti == td or ti == td + 1):
        return False
    present_ok = p0 or ti >= 1
    absent_ok = (not p0) or td >= 1
    for o, r in zip(ops, res):
        if o == 0 and r == 1 and not present_ok:
            return False
        if o == 0 and r == 0 and not absent_ok:
            return False
        if o == 1 and r == 0 and not present_ok:
            return False
        if o == 2 and r == 0 and not absent_ok:
            return False
    if final_present != (p0 ^ ((ti + td) % 2 == 1)):
        return False
    if final_present:
        ins_vals = {v for o, r, v in zip(ops, res, vals) if o == 1 and r == 1}
        if (ti == 0 and final_value != v0) or (ti > 0 and final_value not in ins_vals):
            return False
    return True
