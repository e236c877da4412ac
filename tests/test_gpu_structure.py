"""GPU structure parity (T2 of SURVEY §4): the CUDA path in serial mode (one team applies
a batch's updates in op order) builds exactly Oracle-B's pool -- every DATA / NEXT entry,
the lock states (not the lock versions, which count lock sessions), the head array,
the level counters and the bump counters -- after every batch.  And the paper's worked
examples run on the GPU from the fixture pools give Oracle-B's (pinned) results.
"""
import numpy as np
import pytest
import torch

from oracle.oracle_b import GFSLModel
from paper_conf_ppopp_moscovicicp17_b200.gfsl import GFSL, REBUILD_NEVER
from paper_conf_ppopp_moscovicicp17_b200.workload import SEED_BASE, Workload
from tests import gfsl_fixtures as fx

pytestmark = pytest.mark.gpu


def model_like(g: GFSL, key_range, rebuild_every=0):
    meta, _ = g.dump()
    return GFSLModel(meta["chunk_entries"], key_range, meta["cap_bottom"], meta["cap_upper"],
                     rebuild_every=rebuild_every, p_chunk_q32=g.cfg.p_chunk_q32)


def assert_same_structure(g: GFSL, m: GFSLModel, where=""):
    meta, ent = g.dump()
    N = m.N
    ref = np.array(m.pool, dtype=np.uint64)
    assert ent.shape == ref.shape
    a, b = ent.copy(), ref.copy()
    a[:, N - 1] &= np.uint64(0xFFFFFFFF)   # lock state only; versions count lock sessions
    b[:, N - 1] &= np.uint64(0xFFFFFFFF)
    bad = np.argwhere(a != b)
    assert bad.size == 0, f"{where}: {len(bad)} entries differ, first (chunk, entry) {bad[:5].tolist()}: gpu={[hex(int(a[tuple(x)])) for x in bad[:3]]} oracle={[hex(int(b[tuple(x)])) for x in bad[:3]]}"
    assert meta["head"][:N] == m.head[:N], where
    assert meta["counters"][:N] == m.counter[:N], where
    assert [meta["used_bottom"], meta["used_upper"]] == m.bump, where


def dev(op, key, val):
    d = torch.device("cuda")
    return (torch.as_tensor(np.asarray(op, np.uint8)).to(d),
            torch.as_tensor(np.asarray(key, np.uint32).view(np.int32)).to(d),
            None if val is None else torch.as_tensor(np.asarray(val, np.uint32).view(np.int32)).to(d))


@pytest.mark.parametrize("N,R,B,nb,mix", [
    (6, 300, 120, 25, (35, 35, 30)),
    (12, 600, 200, 20, (35, 35, 30)),
    (16, 2000, 400, 12, (30, 30, 40)),
    (32, 3000, 700, 12, (30, 30, 40)),
    (32, 400, 200, 30, (50, 50, 0)),
    (16, 300, 150, 30, (45, 55, 0)),
])
def test_serial_mode_is_byte_identical_to_oracle_b(N, R, B, nb, mix):
    g = GFSL(R, chunk_entries=N, serial_updates=True, rebuild_every=REBUILD_NEVER)
    m = model_like(g, R)
    assert_same_structure(g, m, "init")
    w = Workload(R, B, mix=mix, seed=SEED_BASE + 17 * N)
    for b in range(nb):
        op, key, val, _ = w.make_batch(b)
        opn, kn, vn = op.numpy(), key.numpy().astype(np.uint32), val.numpy().astype(np.uint32)
        r_gpu = g.batch(*dev(opn, kn, vn)).cpu().numpy()
        r_ora = np.array(m.batch(opn.tolist(), kn.tolist(), vn.tolist()), np.uint8)
        assert np.array_equal(r_gpu, r_ora), f"batch {b}"
        assert_same_structure(g, m, f"after batch {b}")
    st = g.stats()
    assert st["splits"] > 0
    if mix[2] == 0:
        assert st["merges"] > 0


@pytest.mark.parametrize("N,p", [(6, 0.5), (16, 0.25), (32, 0.5)])
def test_serial_p_chunk_byte_identical_to_oracle_b(N, p):
    """p_chunk < 1 (isKeyRaised; R28): same pool as Oracle-B."""
    R = 400 if N == 6 else 3000
    g = GFSL(R, chunk_entries=N, serial_updates=True, rebuild_every=REBUILD_NEVER, p_chunk=p)
    m = model_like(g, R)
    assert m.p_chunk_q32 == int(p * 2**32)
    w = Workload(R, 300, mix=(40, 30, 30), seed=SEED_BASE + 29 * N)
    for b in range(16):
        op, key, val, _ = w.make_batch(b)
        opn, kn, vn = op.numpy(), key.numpy().astype(np.uint32), val.numpy().astype(np.uint32)
        r_gpu = g.batch(*dev(opn, kn, vn)).cpu().numpy()
        r_ora = np.array(m.batch(opn.tolist(), kn.tolist(), vn.tolist()), np.uint8)
        assert np.array_equal(r_gpu, r_ora), f"batch {b}"
        assert_same_structure(g, m, f"after batch {b}")


@pytest.mark.parametrize("N", [16, 32])
def test_serial_fill_then_drain_byte_identical(N):
    """Grow to a multi-level structure, then delete most keys: merges, splitRemove,
    zombies, level counters going back down."""
    R = 6000
    g = GFSL(R, chunk_entries=N, serial_updates=True, rebuild_every=REBUILD_NEVER)
    m = model_like(g, R)
    rng = np.random.default_rng(N)
    perm = rng.permutation(R).astype(np.uint32)
    for s in range(0, R, 1500):
        k = perm[s:s + 1500]
        r_gpu = g.batch(*dev(np.ones(k.size, np.uint8), k, k)).cpu().numpy()
        assert np.array_equal(r_gpu, np.array(m.batch([1] * k.size, k.tolist(), k.tolist()), np.uint8))
        assert_same_structure(g, m, f"fill {s}")
    perm2 = rng.permutation(R).astype(np.uint32)[: R - 50]
    for s in range(0, perm2.size, 997):
        k = perm2[s:s + 997]
        r_gpu = g.batch(*dev(np.full(k.size, 2, np.uint8), k, None)).cpu().numpy()
        assert np.array_equal(r_gpu, np.array(m.batch([2] * k.size, k.tolist()), np.uint8))
        assert_same_structure(g, m, f"drain {s}")
    assert g.stats()["merges"] > 0


@pytest.mark.parametrize("N,every", [(16, 1), (32, 2), (6, 1), (12, 3), (16, 5)])
def test_serial_with_rebuild_byte_identical(N, every):
    """R24 on the GPU (rebuild kernels) equals Oracle-B's rebuild, entry for entry, at a
    fixed period (the library's default wear schedule, R29, is a GPU-side policy that
    Oracle-B does not model; the concurrent parity tests run under it)."""
    R = 3000 if N >= 16 else 500
    g = GFSL(R, chunk_entries=N, serial_updates=True, rebuild_every=every)
    m = model_like(g, R, rebuild_every=every)
    w = Workload(R, R // 4, mix=(30, 30, 40), seed=SEED_BASE + 5 * N)
    for b in range(14):
        if b == 7:  # an explicit gfsl_rebuild between batches
            g.rebuild()
            m.rebuild_now()
        op, key, val, _ = w.make_batch(b)
        opn, kn, vn = op.numpy(), key.numpy().astype(np.uint32), val.numpy().astype(np.uint32)
        r_gpu = g.batch(*dev(opn, kn, vn)).cpu().numpy()
        r_ora = np.array(m.batch(opn.tolist(), kn.tolist(), vn.tolist()), np.uint8)
        assert np.array_equal(r_gpu, r_ora), f"batch {b}"
        assert_same_structure(g, m, f"after batch {b}")
    rep, _, _ = g.validate()
    assert rep.violations == 0


def run_fixture_on_gpu(spec, N, ops, keys, vals=None):
    """Loads the fixture into a GPU handle with the same pool geometry as Oracle-B,
    runs one serial batch on both, and checks they end identical."""
    g = GFSL(100, capacity=64, chunk_entries=N, serial_updates=True, rebuild_every=REBUILD_NEVER)
    meta0, _ = g.dump()
    m, names = fx.build(spec, N, key_range=100, cap_bottom=meta0["cap_bottom"],
                        cap_upper=meta0["cap_upper"])
    meta, ent = fx.image(m)
    g.load(meta, ent.reshape(-1, N))
    assert_same_structure(g, m, "loaded fixture")
    r_gpu = g.batch(*dev(ops, keys, vals)).cpu().numpy().tolist()
    r_ora = m.batch(list(ops), list(keys), None if vals is None else list(vals))
    assert r_gpu == r_ora
    assert_same_structure(g, m, "after the worked example")
    rep, _, _ = g.validate()
    assert rep.violations == 0
    return r_gpu, m, names, g


def test_gpu_fig41_contains():
    r, *_ = run_fixture_on_gpu(fx.FC, 6, [0, 0, 0], [17, 52, 70])
    assert r == [1, 0, 0]


def test_gpu_fig42_insert_15():
    r, m, n, g = run_fixture_on_gpu(fx.FI, 6, [1], [15], [777])
    assert r == [1]
    assert [k for k in m.keys(n["E"]) if k != 0xFFFFFFFF] == [11, 16, 18, 22]


def test_gpu_fig44_split_22():
    r, m, n, g = run_fixture_on_gpu(fx.FS, 6, [1], [22], [5])
    assert r == [1] and m.counter[0] == 2


def test_gpu_fig45_delete_13_merge():
    r, m, n, g = run_fixture_on_gpu(fx.FD, 12, [2], [13])
    assert r == [1] and m.zombie(n["E"])
    r2 = g.batch(*dev([0, 0, 0], [17, 13, 26], None)).cpu().numpy().tolist()
    assert r2 == [1, 0, 1]


def test_gpu_fig46_delete_no_merge():
    r, m, n, g = run_fixture_on_gpu(fx.FDN, 12, [2, 2], [13, 22])
    assert r == [1, 1]
