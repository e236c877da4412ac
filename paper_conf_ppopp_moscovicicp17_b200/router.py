"""Range-partitioned multi-GPU GFSL.

Shard g owns keys [g*ceil(R/G), min(R, (g+1)*ceil(R/G))) in its own GFSL (keys stay
global; no rebasing).  Every rank calls ``batch`` collectively with its own slice of the
global batch, like an NCCL collective.  One batch is:

  route_plan (CUDA: per-op destination, per-tile histogram, scan, stable scatter)
  -> all_to_all of the per-destination counts
  -> route_pack (CUDA) -> all_to_all of ops, keys, values (NCCL over NVLink)
  -> the local gfsl_batch (S1 on the shard)
  -> all_to_all of the 1-byte results back -> route_unpack (CUDA) into the caller's order.

A key's state lives on exactly one shard and every op touches one key, so the S1
semantics and the results are those of one global GFSL.  torch.distributed is the
plumbing for the exchange; every step that touches ops runs in libgfsl kernels.  The
plan/pack/local/unpack steps are injectable so that the exchange logic is tested on CPU
with the gloo backend (tests/test_router_gloo.py).
"""
from __future__ import annotations

import torch
import torch.distributed as dist

from . import gfsl as G


def shard_bounds(key_range: int, world: int, rank: int):
    span = -(-key_range // world)
    lo = min(key_range, rank * span)
    hi = min(key_range, (rank + 1) * span)
    return lo, hi, span


class CudaRouteKernels:
    """The production steps: libgfsl route kernels and a local GFSL."""

    def __init__(self, local: "G.GFSL"):
        self.local = local

    def plan(self, op, key, key_range, world):
        return G.route_plan(op, key, key_range, world)

    def pack(self, perm, op, key, val):
        return G.route_pack(perm, op, key, val)

    def local_batch(self, op, key, val):
        return self.local.batch(op, key, val)

    def unpack(self, perm, res_routed, n):
        out = torch.empty(n, dtype=torch.uint8, device=res_routed.device)
        return G.route_unpack(perm, res_routed, out)


class ShardedGFSL:
    def __init__(self, key_range: int, rank: int, world: int, capacity: int = 0, group=None,
                 kernels=None, **gfsl_kw):
        self.key_range = int(key_range)
        self.rank, self.world, self.group = rank, world, group
        self.key_lo, self.key_hi, self.span = shard_bounds(self.key_range, world, rank)
        if kernels is None:
            cap = capacity if capacity else max(1, self.key_hi - self.key_lo)
            self.local = G.GFSL(self.key_range, capacity=cap, **gfsl_kw)
            kernels = CudaRouteKernels(self.local)
        else:
            self.local = getattr(kernels, "local", None)
        self.k = kernels
        self.last_counts = None

    def _a2a(self, out, inp, out_splits, in_splits):
        if out.is_cuda and dist.get_backend(self.group) == "gloo":
            # gloo has no CUDA all-to-all: stage through host memory (test path only)
            tmp = torch.empty(out.shape, dtype=out.dtype)
            dist.all_to_all_single(tmp, inp.cpu(), out_splits, in_splits, group=self.group)
            out.copy_(tmp)
            return out
        dist.all_to_all_single(out, inp, out_splits, in_splits, group=self.group)
        return out

    def batch(self, op, key, val=None):
        """Collective.  op uint8[n], key 32-bit[n], val 32-bit[n] (this rank's slice);
        returns uint8[n] results in the slice's order."""
        n = op.numel()
        if val is None:
            val = torch.zeros_like(key)
        counts, perm = self.k.plan(op, key, self.key_range, self.world)
        so, sk, sv = self.k.pack(perm, op, key, val)
        recv_counts = torch.empty_like(counts)
        self._a2a(recv_counts, counts, None, None)
        send_split = counts.tolist()
        recv_split = recv_counts.tolist()
        m = int(sum(recv_split))
        ro = torch.empty(m, dtype=op.dtype, device=op.device)
        rk = torch.empty(m, dtype=key.dtype, device=key.device)
        rv = torch.empty(m, dtype=val.dtype, device=val.device)
        self._a2a(ro, so, recv_split, send_split)
        self._a2a(rk, sk, recv_split, send_split)
        self._a2a(rv, sv, recv_split, send_split)
        rr = self.k.local_batch(ro, rk, rv) if m else torch.empty(0, dtype=torch.uint8, device=op.device)
        back = torch.empty(n, dtype=torch.uint8, device=op.device)
        self._a2a(back, rr, send_split, recv_split)
        self.last_counts = (send_split, recv_split)
        return self.k.unpack(perm, back, n)
