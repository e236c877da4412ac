"""ctypes loader for Oracle-A (``oracle_a.c``) -- TEST INFRASTRUCTURE ONLY.

See ``oracle_a.c`` for what is computed and the passages it follows.  Only tests/,
``__graft_entry__.smoke()`` and bench.py's cpu_baseline / reference legs use this.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle_a.c")
_LIB = os.path.join(_HERE, "liboracle_a.so")

OA_OK, OA_ECONTRACT, OA_ENOMEM = 0, 1, 2
CONTAINS, INSERT, DELETE = 0, 1, 2
FALSE, TRUE, INVALID = 0, 1, 0xFF


def build(force: bool = False) -> str:
    """Compile oracle_a.c with plain gcc -O2 (building the checker is not using it)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(
            ["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-o", _LIB, _SRC])
    return _LIB


_lib = None


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        vp, u64, u32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32
        lib.oa_create.restype = vp
        lib.oa_create.argtypes = [u64]
        lib.oa_destroy.argtypes = [vp]
        lib.oa_size.restype = u64
        lib.oa_size.argtypes = [vp]
        lib.oa_contains.restype = ctypes.c_int
        lib.oa_contains.argtypes = [vp, u32]
        lib.oa_get.restype = ctypes.c_int
        lib.oa_get.argtypes = [vp, u32, ctypes.POINTER(u32)]
        lib.oa_insert.restype = ctypes.c_int
        lib.oa_insert.argtypes = [vp, u32, u32]
        lib.oa_erase.restype = ctypes.c_int
        lib.oa_erase.argtypes = [vp, u32]
        lib.oa_export.restype = u64
        lib.oa_export.argtypes = [vp, vp, vp, u64]
        lib.oa_batch.restype = ctypes.c_int
        lib.oa_batch.argtypes = [vp, vp, vp, vp, vp, u64, u64]
        lib.oa_batch_seq.restype = ctypes.c_int
        lib.oa_batch_seq.argtypes = [vp, vp, vp, vp, vp, u64, u64]
        _lib = lib
    return _lib


def _ptr(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data) if a is not None else None


class OracleMap:
    """A sequential ordered map (Pugh skiplist) with S1 batch semantics."""

    def __init__(self, key_range: int, seed: int = 1):
        self.lib = _load()
        self.key_range = int(key_range)
        self.h = self.lib.oa_create(seed)
        if not self.h:
            raise MemoryError("oa_create failed")

    def close(self):
        if self.h:
            self.lib.oa_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __len__(self):
        return int(self.lib.oa_size(self.h))

    def contains(self, k: int) -> bool:
        return bool(self.lib.oa_contains(self.h, k))

    def get(self, k: int):
        v = ctypes.c_uint32()
        return int(v.value) if self.lib.oa_get(self.h, k, ctypes.byref(v)) else None

    def insert(self, k: int, v: int) -> bool:
        r = self.lib.oa_insert(self.h, k, v)
        if r < 0:
            raise MemoryError
        return bool(r)

    def erase(self, k: int) -> bool:
        return bool(self.lib.oa_erase(self.h, k))

    def batch(self, op: np.ndarray, key: np.ndarray, val: np.ndarray | None,
              combine: bool = False) -> np.ndarray:
        """S1 batch (R1; contract enforced), or with combine=True the combining
        semantics of R26 (Contains on the pre-batch map, mutations in input order)."""
        op = np.ascontiguousarray(op, dtype=np.uint8)
        key = np.ascontiguousarray(key, dtype=np.uint32)
        val = None if val is None else np.ascontiguousarray(val, dtype=np.uint32)
        res = np.empty(op.shape[0], dtype=np.uint8)
        fn = self.lib.oa_batch_seq if combine else self.lib.oa_batch
        rc = fn(self.h, _ptr(op), _ptr(key), _ptr(val), _ptr(res), op.shape[0], self.key_range)
        if rc == OA_ECONTRACT:
            raise ValueError("batch violates the <=1-mutating-op-per-key contract")
        if rc != OA_OK:
            raise MemoryError("oa_batch failed")
        return res

    def export(self):
        n = len(self)
        keys = np.empty(n, dtype=np.uint32)
        vals = np.empty(n, dtype=np.uint32)
        c = self.lib.oa_export(self.h, _ptr(keys), _ptr(vals), n)
        assert c == n
        return keys, vals
