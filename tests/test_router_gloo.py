"""The N>1 exchange logic of the router (ShardedGFSL) on CPU: world_size 2 with gloo.

The CUDA steps (route plan/pack/unpack kernels and the local GFSL) are replaced by
plain CPU stand-ins (numpy stable partition, Oracle-A per shard); the exchange itself --
count all-to-all, payload all-to-all, result all-to-all, un-permutation -- is the
production code.  The global results and final set must equal one oracle's.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle.oracle_a import OracleMap
from paper_conf_ppopp_moscovicicp17_b200.router import ShardedGFSL, shard_bounds
from paper_conf_ppopp_moscovicicp17_b200.workload import SEED_BASE, Workload


class CpuKernels:
    """Stand-ins with the kernels' contract: the pack rebases a valid op's key to its
    destination's local key space (gfsl_route_pack), the local map is keyed locally."""

    def __init__(self, width):
        self.oracle = OracleMap(width)
        self.local = None

    def plan(self, op, key, key_range, world):
        opn, keyn = op.numpy(), key.numpy().view(np.uint32).astype(np.int64)
        span = -(-key_range // world)
        dest = np.where((opn <= 2) & (keyn < key_range), np.minimum(keyn // span, world - 1), 0)
        perm = np.argsort(dest, kind="stable").astype(np.int32)
        counts = np.bincount(dest, minlength=world).astype(np.int64)
        return torch.from_numpy(counts), torch.from_numpy(perm)

    def pack(self, perm, op, key, val, key_range, world):
        p = perm.long()
        span = -(-key_range // world)
        o = op[p].numpy()
        k = key[p].numpy().view(np.uint32).astype(np.int64)
        valid = (o <= 2) & (k < key_range)
        local = np.where(valid, k - np.minimum(k // span, world - 1) * span, k).astype(np.uint32)
        return op[p].contiguous(), torch.from_numpy(local.view(np.int32)), val[p].contiguous()

    def local_batch(self, op, key, val):
        r = self.oracle.batch(op.numpy(), key.numpy().view(np.uint32), val.numpy().view(np.uint32))
        return torch.from_numpy(r)

    def unpack(self, perm, res_routed, n):
        out = torch.empty(n, dtype=torch.uint8)
        out[perm.long()] = res_routed
        return out


def _worker(rank, world, port, R, B, nb, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        lo, hi, _ = shard_bounds(R, world, rank)
        sg = ShardedGFSL(R, rank, world, kernels=CpuKernels(hi - lo))
        w = Workload(R, B * world, mix=(20, 20, 60), seed=SEED_BASE + 5)
        out = []
        for b in range(nb):
            op, key, val, _ = w.make_batch(b)
            if b == 1:  # a few invalid ops
                op[3] = 7
                key[5] = R + 3
            sl = slice(rank * B, (rank + 1) * B)
            r = sg.batch(op[sl].contiguous(), key[sl].to(torch.int32).contiguous(),
                         val[sl].to(torch.int32).contiguous())
            out.append(r.numpy())
        ks, vs = sg.k.oracle.export()
        assert ks.size == 0 or ks.max() < hi - lo          # local key space
        ks = (ks.astype(np.int64) + lo).astype(np.uint32)
        q.put((rank, out, ks, vs))
    finally:
        dist.destroy_process_group()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("world", [2])
def test_router_matches_single_oracle(world):
    R, B, nb = 5_000, 700, 5
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, R, B, nb, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = {}
    for _ in range(world):
        rank, out, ks, vs = q.get(timeout=120)
        got[rank] = (out, ks, vs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    # the same global batches through one oracle
    o = OracleMap(R)
    w = Workload(R, B * world, mix=(20, 20, 60), seed=SEED_BASE + 5)
    for b in range(nb):
        op, key, val, _ = w.make_batch(b)
        if b == 1:
            op[3] = 7
            key[5] = R + 3
        exp = o.batch(op.numpy(), key.numpy().astype(np.uint32), val.numpy().astype(np.uint32))
        res = np.concatenate([got[r][0][b] for r in range(world)])
        assert np.array_equal(res, exp), b
    ks = np.concatenate([got[r][1] for r in range(world)])
    vs = np.concatenate([got[r][2] for r in range(world)])
    ok, ov = o.export()
    assert np.array_equal(ks, ok) and np.array_equal(vs, ov)


def test_shard_bounds_cover_range():
    for R in [1, 7, 1000, 10**9]:
        for G in [1, 2, 3, 8]:
            spans = [shard_bounds(R, G, g)[:2] for g in range(G)]
            assert spans[0][0] == 0 and spans[-1][1] == R
            for (a, b), (c, d) in zip(spans, spans[1:]):
                assert b == c and a <= b
