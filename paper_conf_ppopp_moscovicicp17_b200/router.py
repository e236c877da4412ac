"""Range-partitioned multi-GPU GFSL.

Shard g owns keys [g*ceil(R/G), min(R, (g+1)*ceil(R/G))) in its own GFSL, created over
its LOCAL key space [0, hi - lo): the route kernels rebase every key on its way in
(key - lo), so each shard's bitmaps and directory are sized for its own range, and the
export adds lo back.  Every rank calls ``batch`` collectively with its own slice of the
global batch, like an NCCL collective.  One batch is:

  route_plan (CUDA: per-op destination, per-tile histogram, scan, stable scatter)
  -> all_to_all of the per-destination counts
  -> route_pack (CUDA, keys rebased) -> all_to_all of ops, keys, values (NCCL over NVLink)
  -> the local gfsl_batch (S1 on the shard)
  -> all_to_all of the 1-byte results back -> route_unpack (CUDA) into the caller's order.

A key's state lives on exactly one shard and every op touches one key, so the S1
semantics and the results are those of one global GFSL.  torch.distributed is the
plumbing for the exchange; every step that touches ops runs in libgfsl kernels.  The
plan/pack/local/unpack steps are injectable so that the exchange logic is tested on CPU
with the gloo backend (tests/test_router_gloo.py).
"""
from __future__ import annotations

import numpy as np
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

    def pack(self, perm, op, key, val, key_range, world):
        return G.route_pack(perm, op, key, val, key_range, world)

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
            width = max(1, self.key_hi - self.key_lo)
            self.local = G.GFSL(width, capacity=capacity or width, **gfsl_kw)
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
        so, sk, sv = self.k.pack(perm, op, key, val, self.key_range, self.world)
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

    def export(self):
        """This shard's validated (report, global keys, values)."""
        return export_global(self.local, self.key_lo)


def export_global(local: "G.GFSL", key_lo: int):
    rep, ks, vs = local.validate()
    if ks is not None:
        ks = (ks.astype(np.uint64) + key_lo).astype(np.uint32)
    return rep, ks, vs


class PeerShardedGFSL:
    """Range-partitioned GFSL with the fused peer-memory exchange (gfsl_xr_*; SURVEY 8(f)
    NEXT-3): one rank per process and GPU.  Same partition and the same collective
    ``batch`` contract as ShardedGFSL, but no NCCL on the data path: the route kernels
    store every op straight into its destination's window and load every result straight
    back (CUDA IPC mappings over NVLink).  torch.distributed only exchanges the windows'
    IPC handles once, at construction."""

    def __init__(self, key_range: int, rank: int, world: int, max_slice: int, capacity: int = 0,
                 group=None, timeout_ms: int = 0, **gfsl_kw):
        self.key_range = int(key_range)
        self.rank, self.world, self.group = rank, world, group
        self.key_lo, self.key_hi, self.span = shard_bounds(self.key_range, world, rank)
        width = max(1, self.key_hi - self.key_lo)
        self.local = G.GFSL(width, capacity=capacity or width, **gfsl_kw)
        self.xr = G.XRoute(rank, world, self.key_range, max_slice, timeout_ms)
        handles = [None] * world
        dist.all_gather_object(handles, self.xr.export(), group=group)
        for p in range(world):
            if p != rank:
                self.xr.attach(p, handles[p])
        dist.barrier(group=group)

    def batch(self, op, key, val=None, out=None, stream=None):
        """Collective.  op uint8[n], key 32-bit[n], val 32-bit[n] (this rank's slice);
        returns uint8[n] results in the slice's order."""
        return self.xr.batch(self.local, op, key, val, out=out, stream=stream)

    def export(self):
        return export_global(self.local, self.key_lo)


class LoopbackShards:
    """`world` shards driven by ONE process on the current device, exchanging through the
    same windows and kernels as PeerShardedGFSL (attach_local instead of IPC); each shard
    runs on its own stream and every phase is enqueued for all shards before the next
    (split-phase barriers), so the device barriers between the shards are real and never
    wait on a launch that is not yet enqueued.  Used to
    test the exchange on one GPU; ``batch`` takes a GLOBAL batch and splits it into
    `world` contiguous slices, like `world` ranks would hold it."""

    def __init__(self, key_range: int, world: int, max_slice: int, capacity: int = 0,
                 timeout_ms: int = 20000, **gfsl_kw):
        self.key_range, self.world = int(key_range), int(world)
        self.bounds = [shard_bounds(self.key_range, world, r) for r in range(world)]
        self.local = []
        for lo, hi, _ in self.bounds:
            width = max(1, hi - lo)
            self.local.append(G.GFSL(width, capacity=capacity or width, **gfsl_kw))
        self.xr = [G.XRoute(r, world, self.key_range, max_slice, timeout_ms) for r in range(world)]
        for r in range(world):
            for p in range(world):
                if p != r:
                    self.xr[r].attach_local(p, self.xr[p])
        self.streams = [torch.cuda.Stream() for _ in range(world)]

    def slices(self, n: int):
        q, rem = divmod(n, self.world)
        out, a = [], 0
        for r in range(self.world):
            b = a + q + (1 if r < rem else 0)
            out.append((a, b))
            a = b
        return out

    def batch(self, op, key, val=None):
        n = op.numel()
        if val is None:
            val = torch.zeros_like(key)
        cur = torch.cuda.current_stream()
        sl = self.slices(n)
        out = torch.empty(n, dtype=torch.uint8, device=op.device)
        for s in self.streams:
            s.wait_stream(cur)
        for r, (a, b) in enumerate(sl):
            self.xr[r].send(op[a:b], key[a:b], val[a:b], stream=self.streams[r])
        for r in range(self.world):
            self.xr[r].push(stream=self.streams[r])
        recv, errs = [], []
        for r, (a, b) in enumerate(sl):
            recv.append(self.xr[r].recv(stream=self.streams[r]))
            st = self.xr[r].local(self.local[r], n_hint=max(1, b - a), stream=self.streams[r])
            if st != G.GFSL_OK:
                errs.append((st, r))
            self.xr[r].done(stream=self.streams[r])
        for r, (a, b) in enumerate(sl):
            self.xr[r].finish(out[a:b], stream=self.streams[r])
        for s in self.streams:
            cur.wait_stream(s)
        self.recv_ptrs = [x[1] for x in recv]
        if errs:
            G._check(errs[0][0], f"gfsl_xr_local (shard {errs[0][1]})")
        return out

    def last_recv(self):
        """The received op count of every shard in the last batch (synchronises; tests)."""
        torch.cuda.synchronize()
        return [G.read_device_u32(nd) for nd in self.recv_ptrs]

    def export(self, r: int):
        lo = self.bounds[r][0]
        return export_global(self.local[r], lo)

