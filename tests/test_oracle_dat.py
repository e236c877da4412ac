"""Pins of the direct-address-table checker (oracle/dat.py), CPU only: the same results
and final set as Oracle-A (the Pugh skiplist) and as a Python dict, batch by batch."""
import numpy as np
import pytest

from oracle.dat import DirectAddressMap
from oracle.oracle_a import OracleMap

from .test_oracle_a import brute_batch, random_batch


@pytest.mark.parametrize("R", [1, 7, 64, 5000])
def test_dat_vs_oracle_a_and_dict(R):
    rng = np.random.default_rng(R + 11)
    d, o, M = DirectAddressMap(R), OracleMap(R), {}
    for _ in range(60):
        op, key, val = random_batch(rng, R, int(rng.integers(0, 3000)))
        r = d.batch(op, key, val)
        assert np.array_equal(r, o.batch(op, key, val))
        assert np.array_equal(r, brute_batch(M, op.tolist(), key.tolist(), val.tolist(), R))
    ks, vs = d.export()
    ok, ov = o.export()
    assert np.array_equal(ks, ok) and np.array_equal(vs, ov)


def test_dat_contract_check():
    d = DirectAddressMap(10)
    with pytest.raises(ValueError):
        d.batch(np.array([1, 2], np.uint8), np.array([3, 3], np.uint32), None)


def test_load_equals_an_insert_batch():
    """DirectAddressMap.load (the full-size prefill) = an S1 batch of distinct Inserts."""
    rng = np.random.default_rng(11)
    R = 5000
    k = rng.permutation(R)[:2000].astype(np.uint32)
    v = rng.integers(0, 2**32, k.size, dtype=np.uint64).astype(np.uint32)
    a = DirectAddressMap(R)
    b = DirectAddressMap(R)
    a.batch(np.ones(k.size, np.uint8), k, v)
    b.load(k, v)
    ka, va = a.export()
    kb, vb = b.export()
    assert np.array_equal(ka, kb) and np.array_equal(va, vb)
    import pytest
    with pytest.raises(ValueError):
        b.load(k[:3], v[:3])
