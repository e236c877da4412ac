"""GPU tests of the fused peer-memory exchange (gfsl_xr_*).

* LoopbackShards: G shards in one process, each on its own stream, exchanging through
  the production windows, push/pull kernels and device barriers: results element by
  element and the union of the shards' final sets equal one Oracle-A over the global
  batches (ragged slices, empty slices, invalid ops, every op on one shard).
* Two processes on the one GPU, each mapping the other's window through CUDA IPC
  (PeerShardedGFSL, the one-rank-per-GPU production class): same checks.
* A peer that never arrives: the barrier times out, the call returns GFSL_ETIMEOUT and
  the handle stays failed (no hang).
"""
import os
import socket

import numpy as np
import pytest
import torch

from oracle.oracle_a import OracleMap
from paper_conf_ppopp_moscovicicp17_b200 import gfsl as G
from paper_conf_ppopp_moscovicicp17_b200.router import LoopbackShards
from paper_conf_ppopp_moscovicicp17_b200.workload import SEED_BASE, Workload

pytestmark = pytest.mark.gpu


def _to_dev(op, key, val, dev):
    return (op.to(dev), key.to(torch.int32).to(dev), val.to(torch.int32).to(dev))


def _check_final(ls, o):
    ex = [ls.export(r) for r in range(ls.world)]
    ks = np.concatenate([x[1] for x in ex])
    vs = np.concatenate([x[2] for x in ex])
    ok, ov = o.export()
    assert np.array_equal(ks, ok) and np.array_equal(vs, ov)


@pytest.mark.parametrize("world", [2, 3, 4, 8])
def test_loopback_exchange_matches_global_oracle(world):
    R, B = 300_007, 50_001  # ragged shards and slices
    dev = torch.device("cuda")
    ls = LoopbackShards(R, world, max_slice=-(-B // world))
    o = OracleMap(R)
    w = Workload(R, B, mix=(20, 20, 60), seed=SEED_BASE + 31 + world)
    for b in range(6):
        op, key, val, _ = w.make_batch(b)
        res = ls.batch(*_to_dev(op, key, val, dev))
        exp = o.batch(op.numpy(), key.numpy().astype(np.uint32), val.numpy().astype(np.uint32))
        assert np.array_equal(res.cpu().numpy(), exp), f"batch {b}"
        assert sum(ls.last_recv()) == B
    _check_final(ls, o)


def test_loopback_edge_batches():
    R, world = 100_000, 4
    dev = torch.device("cuda")
    ls = LoopbackShards(R, world, max_slice=20_000)
    o = OracleMap(R)
    rng = np.random.default_rng(5)

    def run(op, key, val):
        res = ls.batch(torch.from_numpy(op).to(dev), torch.from_numpy(key.view(np.int32)).to(dev),
                       torch.from_numpy(val.view(np.int32)).to(dev))
        exp = o.batch(op, key, val)
        assert np.array_equal(res.cpu().numpy(), exp)

    # prefill: distinct keys
    k = rng.permutation(R)[:40_000].astype(np.uint32)
    run(np.ones(k.size, np.uint8), k, rng.integers(0, 2**32, k.size, dtype=np.uint64).astype(np.uint32))
    # empty batch and batches smaller than the world (empty slices)
    for n in (0, 1, 3):
        kk = rng.permutation(R)[:n].astype(np.uint32)
        run(rng.integers(0, 3, n).astype(np.uint8), kk, np.zeros(n, np.uint32))
    # every op on the last shard; invalid keys and op codes go to shard 0 and stay invalid
    n = 20_000
    kk = (R - 1 - rng.permutation(R // 4)[:n]).astype(np.uint32)
    op = rng.integers(0, 3, n).astype(np.uint8)
    op[::97] = 7
    kk[::89] = R + 5
    run(op, kk, rng.integers(0, 2**32, n, dtype=np.uint64).astype(np.uint32))
    _check_final(ls, o)


def test_timeout_when_a_peer_never_arrives():
    """Rank 1 never sends: rank 0's count barrier expires, its received count is 0, its
    results are INVALID, no call blocks, and the handle reports GFSL_ETIMEOUT from then on."""
    dev = torch.device("cuda")
    a = G.XRoute(0, 2, 1000, 16, timeout_ms=200)
    b = G.XRoute(1, 2, 1000, 16, timeout_ms=200)
    a.attach_local(1, b)
    local = G.GFSL(500)
    op = torch.zeros(4, dtype=torch.uint8, device=dev)
    key = torch.arange(4, dtype=torch.int32, device=dev)
    out = torch.zeros(4, dtype=torch.uint8, device=dev)
    a.send(op, key)  # rank 1 never sends
    a.push()
    cap, nd, o, k, v, r = a.recv()
    assert cap == 32
    local.batch_dn(o, k, v, r, cap, nd, n_hint=4)
    a.done()
    try:
        a.finish(out)
    except G.GFSLError as e:   # may already see the error word
        assert e.status == G.GFSL_ETIMEOUT
    torch.cuda.synchronize()
    assert G.read_device_u32(nd) == 0
    assert out.cpu().tolist() == [0xFF] * 4
    assert a.status() == G.GFSL_ETIMEOUT
    with pytest.raises(G.GFSLError) as e:
        a.send(op, key)
    assert e.value.status == G.GFSL_ETIMEOUT
    local.close()
    b.close()
    a.close()


def test_local_failure_still_completes_the_exchange():
    """A shard whose local batch fails (a sticky GFSL_EPOOL here) answers its received ops
    INVALID and still takes part in every barrier (gfsl_xr_local): the other shard's ops
    are answered and nobody times out."""
    R, world = 40_000, 2
    dev = torch.device("cuda")
    ls = LoopbackShards(R, world, max_slice=20_000, timeout_ms=10_000)
    ls.local[1].close()
    ls.local[1] = G.GFSL(R // 2, capacity=10)          # a tiny pool: exhausted at once
    keys = torch.randperm(R, generator=torch.Generator().manual_seed(3))[:30_000].to(torch.int32)
    op = torch.ones(keys.numel(), dtype=torch.uint8)
    ls.batch(op.to(dev), keys.to(dev), keys.to(dev))   # shard 1 raises GFSL_EPOOL on device
    torch.cuda.synchronize()
    out = None
    with pytest.raises(G.GFSLError) as e:
        out = ls.batch(op.to(dev), keys.to(dev), keys.to(dev))  # shard 1 fails on the host
    assert e.value.status == G.GFSL_EPOOL
    torch.cuda.synchronize()
    # the exchange completed: the same call again gives shard 0's answers (present now ->
    # Insert false) and INVALID for shard 1's, with no timeout on either window
    with pytest.raises(G.GFSLError):
        ls.batch(op.to(dev), keys.to(dev), keys.to(dev))
    for x in ls.xr:
        assert x.status() == G.GFSL_OK
    k = keys.numpy().astype(np.int64)
    sl = ls.slices(k.size)
    res = []
    # re-run with results kept: drive the phases by hand to read the output
    outs = torch.empty(k.size, dtype=torch.uint8, device=dev)
    op_d, key_d = op.to(dev), keys.to(dev)
    torch.cuda.synchronize()
    for r, (a, b) in enumerate(sl):
        ls.xr[r].send(op_d[a:b], key_d[a:b], key_d[a:b], stream=ls.streams[r])
    for r in range(world):
        ls.xr[r].push(stream=ls.streams[r])
    for r, (a, b) in enumerate(sl):
        ls.xr[r].recv(stream=ls.streams[r])
        res.append(ls.xr[r].local(ls.local[r], n_hint=b - a, stream=ls.streams[r]))
        ls.xr[r].done(stream=ls.streams[r])
    for r, (a, b) in enumerate(sl):
        ls.xr[r].finish(outs[a:b], stream=ls.streams[r])
    torch.cuda.synchronize()
    assert res == [G.GFSL_OK, G.GFSL_EPOOL]
    o = outs.cpu().numpy()
    assert (o[k < R // 2] == 0).all() and (o[k >= R // 2] == 0xFF).all()


def _ipc_worker(rank, world, port, R, B, nb, outdir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch.distributed as dist
    from paper_conf_ppopp_moscovicicp17_b200.router import PeerShardedGFSL
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    dev = torch.device("cuda", 0)
    q, rem = divmod(B, world)
    sl = [(r * q + min(r, rem), (r + 1) * q + min(r + 1, rem)) for r in range(world)]
    g = PeerShardedGFSL(R, rank, world, max_slice=q + 1, timeout_ms=30000)
    w = Workload(R, B, mix=(20, 20, 60), seed=SEED_BASE + 77)
    outs = []
    for b in range(nb):
        op, key, val, _ = w.make_batch(b)
        a, e = sl[rank]
        res = g.batch(*_to_dev(op[a:e].contiguous(), key[a:e].contiguous(), val[a:e].contiguous(), dev))
        outs.append(res.cpu().numpy())
    _, ks, vs = g.export()
    np.savez(os.path.join(outdir, f"r{rank}.npz"), res=np.concatenate(outs), ks=ks, vs=vs)
    dist.barrier()
    dist.destroy_process_group()


def test_two_processes_ipc_windows(tmp_path):
    import torch.multiprocessing as mp
    R, B, nb, world = 100_000, 20_001, 4, 2
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    mp.spawn(_ipc_worker, args=(world, port, R, B, nb, str(tmp_path)), nprocs=world, join=True)
    o = OracleMap(R)
    w = Workload(R, B, mix=(20, 20, 60), seed=SEED_BASE + 77)
    q, rem = divmod(B, world)
    sl = [(r * q + min(r, rem), (r + 1) * q + min(r + 1, rem)) for r in range(world)]
    got = [np.load(tmp_path / f"r{r}.npz") for r in range(world)]
    off = [0] * world
    for b in range(nb):
        op, key, val, _ = w.make_batch(b)
        exp = o.batch(op.numpy(), key.numpy().astype(np.uint32), val.numpy().astype(np.uint32))
        for r, (a, e) in enumerate(sl):
            assert np.array_equal(got[r]["res"][off[r]:off[r] + e - a], exp[a:e]), f"batch {b} rank {r}"
            off[r] += e - a
    ok, ov = o.export()
    assert np.array_equal(np.concatenate([x["ks"] for x in got]), ok)
    assert np.array_equal(np.concatenate([x["vs"] for x in got]), ov)
