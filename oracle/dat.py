"""Direct-address table (DAT) -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

The brute-force definition of an S1 batch (R1) over a bounded key universe
[0, R): a presence bitmap and a value array indexed by key (SURVEY 8(c) "DAT", the
checker for the full-size configs, where the Pugh skiplist of Oracle-A would take
minutes).  Vectorised with numpy; under the <=1-mutation-per-key contract the order of
the mutations does not matter, so they are applied as one scatter.

  contains(k) -> present[k]                 (Alg 4.1)
  insert(k,v) -> not present[k]; no overwrite (Alg 4.5 l.2-4)
  delete(k)   -> present[k]                 (Alg 4.11 l.3-5)
  invalid op (code > 2 or key >= R) -> 0xFF, no effect (R5)

Pinned by tests/test_oracle_dat.py against Oracle-A and a Python dict.
"""
from __future__ import annotations

import numpy as np


class DirectAddressMap:
    def __init__(self, key_range: int, values: bool = True):
        self.R = int(key_range)
        self.present = np.zeros(self.R, dtype=bool)
        self.value = np.zeros(self.R, dtype=np.uint32) if values else None

    def __len__(self):
        return int(self.present.sum())

    def batch(self, op, key, val=None) -> np.ndarray:
        op = np.asarray(op, dtype=np.uint8)
        key = np.asarray(key, dtype=np.uint32)
        res = np.full(op.shape[0], 0xFF, dtype=np.uint8)
        valid = (op <= 2) & (key.astype(np.int64) < self.R)
        k = key[valid].astype(np.int64)
        o = op[valid]
        pre = self.present[k]                       # every result from the pre-batch map
        res[valid] = np.where(o == 1, ~pre, pre).astype(np.uint8)
        mut = valid & (op != 0)
        mk = key[mut]
        if np.unique(mk).size != mk.size:
            raise ValueError("batch violates the <=1-mutating-op-per-key contract")
        ins = mut & (op == 1) & (res == 1)
        dele = mut & (op == 2) & (res == 1)
        self.present[key[ins].astype(np.int64)] = True
        if self.value is not None and val is not None:
            self.value[key[ins].astype(np.int64)] = np.asarray(val, dtype=np.uint32)[ins]
        elif self.value is not None:
            self.value[key[ins].astype(np.int64)] = 0
        self.present[key[dele].astype(np.int64)] = False
        return res

    def load(self, keys, vals=None):
        """Insert DISTINCT keys absent from the map (a prefill): the same as an S1 batch of
        Inserts, without the batch's contract check (its sort costs minutes at 500M keys)."""
        k = np.asarray(keys).astype(np.int64)
        if self.present[k].any():
            raise ValueError("load: a key is already present")
        self.present[k] = True
        if self.value is not None:
            self.value[k] = 0 if vals is None else np.asarray(vals, dtype=np.uint32)
        return self

    def export(self):
        ks = np.flatnonzero(self.present).astype(np.uint32)
        return ks, (self.value[ks] if self.value is not None else None)
