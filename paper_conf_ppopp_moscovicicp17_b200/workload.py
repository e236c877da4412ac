"""Seeded, counter-based synthetic workloads (SURVEY 8(d) "Generator").

This module holds NO arithmetic of the method: it only draws op types, keys and values.
Both the CUDA path (bench.py, tests) and the oracle side (tests, cpu_baseline) consume
its arrays, so it is the one piece of code they share.  It runs on any torch device
(CPU for the oracle side, CUDA for the bench) with identical results: everything is
int64 integer arithmetic, except the Zipf inverse-CDF table (float64, computed once).

Recipe (the paper's workloads):
* ``h(seed, stream, i) = splitmix64(seed ^ stream*PHI ^ i)``; streams PREFILL, TYPE, KEY,
  VAL, ZIPF, PERM.
* uniform key = ``(h mod 2^32) * R >> 32``.
* op types: exact per-batch counts round(i%*B), round(d%*B), rest Contains, placed by a
  keyed shuffle (argsort of h over the batch).  The paper draws i.i.d.; exact counts keep
  the mix exact.
* mutating keys of one batch are drawn WITHOUT replacement (the <=1-mutating-op-per-key
  contract, R2): a colliding draw is redrawn from the next counter value, up to
  64 tries, then uniformly.  ``dedup=False`` keeps the i.i.d. draws (for combining mode,
  DESIGN.md R26, which has no contract).
* value = ``h(seed, VAL, i) mod 2^32`` (the paper inserts NULL; random values make
  the export check meaningful).
* prefill = the first P elements of a keyed Feistel permutation of [0, R) (cycle walking),
  inserted in that random order ("a random set of keys, exactly half the size of
  the key range"; all R keys for Contains-only).
* Zipf(s): rank from the inverse CDF of ``1/r^s`` over R ranks (binary search of u in
  [0,1)), key = Feistel(rank) so hot keys are scattered over the key space.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import torch

SEED_BASE = 20170204
PREFILL, TYPE, KEY, VAL, ZIPF, PERM = 1, 2, 3, 4, 5, 6
PHI = 0x9E3779B97F4A7C15

CONTAINS, INSERT, DELETE = 0, 1, 2

_M64 = (1 << 64) - 1


def _s64(x: int) -> int:
    """Python int -> the int64 with the same 64 bits."""
    x &= _M64
    return x - (1 << 64) if x >= (1 << 63) else x


def _srl(x: torch.Tensor, s: int) -> torch.Tensor:
    """Logical right shift of int64 tensors holding uint64 bit patterns."""
    return (x >> s) & ((1 << (64 - s)) - 1)


_C1 = _s64(0x9E3779B97F4A7C15)
_C2 = _s64(0xBF58476D1CE4E5B9)
_C3 = _s64(0x94D049BB133111EB)


def splitmix64(x: torch.Tensor) -> torch.Tensor:
    z = x + _C1
    z = (z ^ _srl(z, 30)) * _C2
    z = (z ^ _srl(z, 27)) * _C3
    return z ^ _srl(z, 31)


def h(seed: int, stream: int, idx: torch.Tensor) -> torch.Tensor:
    """Counter-based hash: int64 tensor of uint64 bit patterns."""
    base = _s64(seed ^ ((stream * PHI) & _M64))
    return splitmix64(idx ^ base)


def uniform_u32(seed: int, stream: int, idx: torch.Tensor) -> torch.Tensor:
    return h(seed, stream, idx) & 0xFFFFFFFF


def uniform_key(seed: int, stream: int, idx: torch.Tensor, R: int) -> torch.Tensor:
    u = uniform_u32(seed, stream, idx)
    if R <= (1 << 31):
        return (u * R) >> 32
    # (u * R) may need 64 unsigned bits: split R
    hi, lo = R >> 16, R & 0xFFFF
    return ((u * hi) + ((u * lo) >> 16)) >> 16


def feistel_perm(seed: int, x: torch.Tensor, R: int, rounds: int = 4) -> torch.Tensor:
    """A keyed bijection of [0, R): balanced Feistel over 2*hb bits + cycle walking."""
    bits = max(2, (max(R - 1, 1)).bit_length())
    bits += bits & 1
    hb = bits // 2
    mask = (1 << hb) - 1

    def enc(v):
        left, right = _srl(v, hb) & mask, v & mask
        for r in range(rounds):
            f = splitmix64(right ^ _s64(seed * 0x100000001B3 + r * PHI)) & mask
            left, right = right, left ^ f
        return (left << hb) | right

    y = enc(x)
    bad = y >= R
    while bool(bad.any()):
        y = torch.where(bad, enc(y), y)
        bad = y >= R
    return y


def prefill_keys(seed: int, R: int, count: int, start: int = 0, device="cpu") -> torch.Tensor:
    """Elements [start, start+count) of the keyed permutation of [0, R)."""
    idx = torch.arange(start, start + count, dtype=torch.int64, device=device)
    return feistel_perm(_s64(seed ^ PREFILL), idx, R)


def prefill_values(seed: int, keys: torch.Tensor) -> torch.Tensor:
    return uniform_u32(seed, VAL, keys | (1 << 52))


class ZipfTable:
    """Inverse CDF of P(rank r) ~ 1/r^s over r = 1..R, float64 (computed once)."""

    def __init__(self, R: int, s: float = 0.99, device="cpu"):
        r = torch.arange(1, R + 1, dtype=torch.float64, device=device)
        w = r.pow(-s)
        self.cdf = torch.cumsum(w, 0)
        self.cdf /= self.cdf[-1].clone()
        self.R = R

    def rank(self, u53: torch.Tensor) -> torch.Tensor:
        u = u53.to(torch.float64) * (2.0 ** -53)
        return torch.searchsorted(self.cdf, u, right=True).clamp_max(self.R - 1)


@dataclass
class Workload:
    """One config's op stream; batch b is a pure function of (seed, b)."""
    key_range: int
    batch: int
    mix: tuple = (10, 10, 80)      # insert %, delete %, contains %
    dist: str = "uniform"          # "uniform" | "zipf"
    zipf_s: float = 0.99
    seed: int = SEED_BASE
    dedup: bool = True             # False: mutating keys i.i.d. too (combining mode, R26)
    _zipf: ZipfTable | None = field(default=None, repr=False)

    def n_ins_del(self):
        ni = int(round(self.mix[0] * self.batch / 100.0))
        nd = int(round(self.mix[1] * self.batch / 100.0))
        return ni, nd

    def _draw(self, stream_idx: torch.Tensor, device) -> torch.Tensor:
        if self.dist == "uniform":
            return uniform_key(self.seed, KEY, stream_idx, self.key_range)
        if self._zipf is None or self._zipf.cdf.device != torch.device(device):
            self._zipf = ZipfTable(self.key_range, self.zipf_s, device=device)
        u53 = _srl(h(self.seed, ZIPF, stream_idx), 11)
        rk = self._zipf.rank(u53)
        return feistel_perm(_s64(self.seed ^ PERM), rk, self.key_range)

    def make_batch(self, b: int, device="cpu"):
        """Returns (op u8, key int64 in [0,R), val int64 in [0,2^32), redraws)."""
        B = self.batch
        gidx = torch.arange(B, dtype=torch.int64, device=device) + b * B
        # op types: exact counts placed by a keyed shuffle
        order = torch.argsort(h(self.seed, TYPE, gidx))
        ni, nd = self.n_ins_del()
        op = torch.zeros(B, dtype=torch.uint8, device=device)
        op[order[:ni]] = INSERT
        op[order[ni:ni + nd]] = DELETE
        key = self._draw(gidx, device)
        val = uniform_u32(self.seed, VAL, gidx)
        redraws = 0
        mut = (op != CONTAINS).nonzero().flatten()
        if mut.numel() and self.dedup:
            key, redraws = self._dedup_mutating(key, mut, gidx, device)
        return op, key, val, redraws

    def _dedup_mutating(self, key, mut, gidx, device):
        """Without replacement among the batch's mutating ops (first in index order keeps)."""
        R = self.key_range
        taken = torch.zeros(R, dtype=torch.bool, device=device)
        pending = mut                     # op indices still needing a key, ascending
        cand = key[pending]
        redraws = 0
        attempt = 0
        while pending.numel():
            # first occurrence of each candidate among pending (ascending index order)
            srt, perm = torch.sort(cand, stable=True)
            first = torch.ones_like(srt, dtype=torch.bool)
            first[1:] = srt[1:] != srt[:-1]
            ok_sorted = first & ~taken[srt]
            ok = torch.empty_like(ok_sorted)
            ok[perm] = ok_sorted
            acc = pending[ok]
            key[acc] = cand[ok]
            taken[cand[ok]] = True
            pending = pending[~ok]
            if not pending.numel():
                break
            attempt += 1
            redraws += int(pending.numel())
            sidx = gidx[pending] + (attempt << 40)
            if attempt <= 64:
                cand = self._draw(sidx, device)
            else:
                cand = uniform_key(self.seed, KEY, sidx, R)
        return key, redraws
