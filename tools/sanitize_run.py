"""Small end-to-end run for compute-sanitizer: concurrent and serial batches with splits,
merges, zombies, upkeep and rebuilds, checked against the oracle."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from oracle.oracle_a import OracleMap
from paper_conf_ppopp_moscovicicp17_b200.gfsl import GFSL
from paper_conf_ppopp_moscovicicp17_b200.workload import SEED_BASE, Workload

dev = torch.device("cuda")
for N, serial in [(16, False), (32, False), (16, True)]:
    R = 3000
    g = GFSL(R, chunk_entries=N, serial_updates=serial, rebuild_every=1)
    o = OracleMap(R)
    w = Workload(R, 800, mix=(40, 40, 20), seed=SEED_BASE + N)
    for b in range(10):
        op, key, val, _ = w.make_batch(b)
        r = g.batch(op.to(dev), key.to(torch.int32).to(dev), val.to(torch.int32).to(dev)).cpu().numpy()
        e = o.batch(op.numpy(), key.numpy().astype(np.uint32), val.numpy().astype(np.uint32))
        assert np.array_equal(r, e)
    rep, ks, vs = g.validate()
    assert rep.violations == 0 and np.array_equal(ks, o.export()[0])
    print("ok", N, serial, g.stats())

# combining mode (R26) with duplicate keys, and the async host entry point
R = 2000
g = GFSL(R, combine=True, rebuild_every=1)
o = OracleMap(R)
rng = np.random.default_rng(5)
outs = []
for b in range(6):
    op = rng.integers(0, 3, 1500).astype(np.uint8)
    key = rng.integers(0, R, 1500).astype(np.uint32)
    val = rng.integers(0, 2**32, 1500, dtype=np.uint64).astype(np.uint32)
    h = (torch.from_numpy(op).pin_memory(), torch.from_numpy(key.view(np.int32)).pin_memory(),
         torch.from_numpy(val.view(np.int32)).pin_memory())
    outs.append((g.batch_host_async(*h), o.batch(op, key, val, combine=True), h))
torch.cuda.synchronize()
assert all(np.array_equal(r.numpy(), e) for r, e, _ in outs)
rep, ks, vs = g.validate()
assert rep.violations == 0 and np.array_equal(ks, o.export()[0]) and np.array_equal(vs, o.export()[1])
print("ok combine+async", g.stats())

# round 2: the paths added this round -- derived paths (R41) in lazy batches with rebuilds,
# the chunk-grouped update path (R40, opt-in), the small-batch kernel, the forced coarse
# directory (8-key min-key window), eight mutations per warp (a batch of >= 64K ops)
os.environ["GFSL_SMALL_BATCH"] = "16384"
os.environ["GFSL_DIR_CAP"] = "1024"
for N, group in [(16, 0), (32, 0), (16, 1)]:
    R = 150_000
    g = GFSL(R, chunk_entries=N, rebuild_every=2, group=group)
    o = OracleMap(R)
    rng = np.random.default_rng(11 + N + group)
    k0 = rng.permutation(R)[: R // 2].astype(np.uint32)
    g.batch(torch.from_numpy(np.ones(k0.size, np.uint8)).to(dev), torch.from_numpy(k0.view(np.int32)).to(dev),
            torch.from_numpy(k0.view(np.int32)).to(dev))
    o.batch(np.ones(k0.size, np.uint8), k0, k0)
    for b, n in enumerate([3000, 20000, 70000, 5000]):
        key = rng.choice(R, n, replace=False).astype(np.uint32)
        op = rng.choice([0, 1, 2], n, p=[0.2, 0.4, 0.4]).astype(np.uint8)
        val = rng.integers(0, 2**32, n, dtype=np.uint64).astype(np.uint32)
        r = g.batch(torch.from_numpy(op).to(dev), torch.from_numpy(key.view(np.int32)).to(dev),
                    torch.from_numpy(val.view(np.int32)).to(dev)).cpu().numpy()
        assert np.array_equal(r, o.batch(op, key, val)), (N, group, b)
    assert g.check().violations == 0
    print("ok round-2 paths", N, group, g.stats())
