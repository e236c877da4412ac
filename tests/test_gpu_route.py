"""GPU tests of the multi-GPU route kernels (B5) and of range sharding on one GPU.

* gfsl_route_plan / _pack / _unpack vs a numpy stable partition (bit-exact perm/counts);
* a loopback of G shards on one GPU (G local GFSLs; the all-to-all is the identity of a
  single process) vs one oracle: the sharded results and final set are the global ones.
"""
import numpy as np
import pytest
import torch

from oracle.oracle_a import OracleMap
from paper_conf_ppopp_moscovicicp17_b200 import gfsl as G
from paper_conf_ppopp_moscovicicp17_b200.router import shard_bounds
from paper_conf_ppopp_moscovicicp17_b200.workload import SEED_BASE, Workload

pytestmark = pytest.mark.gpu


def ref_plan(op, key, R, world):
    key = key.astype(np.int64)
    span = -(-R // world)
    dest = np.where((op <= 2) & (key < R), np.minimum(key // span, world - 1), 0)
    return np.bincount(dest, minlength=world), np.argsort(dest, kind="stable")


@pytest.mark.parametrize("world", [1, 2, 3, 8, 64])
@pytest.mark.parametrize("n", [0, 1, 1023, 1024, 1025, 100_000])
def test_route_plan_pack_unpack(world, n):
    rng = np.random.default_rng(n + world)
    R = 1_000_003
    op = rng.integers(0, 4, n).astype(np.uint8)
    key = rng.integers(0, R + 100, n).astype(np.uint32)
    val = rng.integers(0, 2**32, n, dtype=np.uint64).astype(np.uint32)
    dev = torch.device("cuda")
    op_d = torch.from_numpy(op).to(dev)
    key_d = torch.from_numpy(key.view(np.int32)).to(dev)
    val_d = torch.from_numpy(val.view(np.int32)).to(dev)
    counts, perm = G.route_plan(op_d, key_d, R, world)
    ec, ep = ref_plan(op, key, R, world)
    assert counts.cpu().numpy().tolist() == ec.tolist()
    assert np.array_equal(perm.cpu().numpy(), ep.astype(np.int32))
    so, sk, sv = G.route_pack(perm, op_d, key_d, val_d, R, world)
    assert np.array_equal(so.cpu().numpy(), op[ep])
    # valid ops' keys in their destination's local key space; invalid ones unchanged
    span = -(-R // world)
    k64, o8 = key.astype(np.int64), op
    valid = (o8 <= 2) & (k64 < R)
    local = np.where(valid, k64 - np.minimum(k64 // span, world - 1) * span, k64).astype(np.uint32)
    assert np.array_equal(sk.cpu().numpy().view(np.uint32), local[ep])
    assert np.array_equal(sv.cpu().numpy().view(np.uint32), val[ep])
    rr = torch.arange(n, device=dev).to(torch.uint8)
    out = torch.empty(n, dtype=torch.uint8, device=dev)
    G.route_unpack(perm, rr, out)
    exp = np.empty(n, np.uint8)
    exp[ep] = np.arange(n).astype(np.uint8)
    assert np.array_equal(out.cpu().numpy(), exp)


@pytest.mark.parametrize("world", [2, 4])
def test_loopback_shards_match_global_oracle(world):
    R, B = 200_000, 40_000
    dev = torch.device("cuda")
    shards = [G.GFSL(shard_bounds(R, world, g)[1] - shard_bounds(R, world, g)[0])
              for g in range(world)]
    o = OracleMap(R)
    w = Workload(R, B, mix=(20, 20, 60), seed=SEED_BASE + 9)
    for b in range(6):
        op, key, val, _ = w.make_batch(b)
        op_d = op.to(dev)
        key_d = key.to(torch.int32).to(dev)
        val_d = val.to(torch.int32).to(dev)
        counts, perm = G.route_plan(op_d, key_d, R, world)
        so, sk, sv = G.route_pack(perm, op_d, key_d, val_d, R, world)
        parts, s = [], 0
        for g, c in enumerate(counts.tolist()):
            parts.append(shards[g].batch(so[s:s + c], sk[s:s + c], sv[s:s + c]) if c else
                         torch.empty(0, dtype=torch.uint8, device=dev))
            s += c
        res = torch.empty(B, dtype=torch.uint8, device=dev)
        G.route_unpack(perm, torch.cat(parts), res)
        exp = o.batch(op.numpy(), key.numpy().astype(np.uint32), val.numpy().astype(np.uint32))
        assert np.array_equal(res.cpu().numpy(), exp)
    ks = np.concatenate([sh.validate()[1].astype(np.int64) + shard_bounds(R, world, g)[0]
                         for g, sh in enumerate(shards)]).astype(np.uint32)
    vs = np.concatenate([sh.validate()[2] for sh in shards])
    ok, ov = o.export()
    assert np.array_equal(ks, ok) and np.array_equal(vs, ov)
