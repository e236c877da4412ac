"""Per-op latency of the update kernel with ONE team (serial mode): n inserts / deletes of
keys in distinct chunks, time / n.  python tools/op_latency.py [R] [n]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from bench import prefill_gpu
from paper_conf_ppopp_moscovicicp17_b200.gfsl import GFSL
from paper_conf_ppopp_moscovicicp17_b200.workload import SEED_BASE, prefill_keys

R = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
n = int(sys.argv[2]) if len(sys.argv) > 2 else 200
dev = torch.device("cuda")
rng = np.random.default_rng(0)
for serial in (True,):
    g = GFSL(R, capacity=R, profile_phases=True, serial_updates=serial)
    prefill_gpu(g, R, R // 2, dev)
    perm = prefill_keys(SEED_BASE, R, R).numpy()
    present, absent = perm[:R // 2], perm[R // 2:]
    for name, op, keys in [("delete", 2, rng.choice(present, n, replace=False)),
                           ("insert", 1, rng.choice(absent, n, replace=False)),
                           ("contains-only", 0, rng.choice(present, n, replace=False))]:
        g.phase_times()
        k = torch.as_tensor(keys.astype(np.int64)).to(torch.int32).to(dev)
        g.batch(torch.full((n,), op, dtype=torch.uint8, device=dev), k, k)
        ph, _ = g.phase_times()
        st = g.stats()
        print(f"{name:14s} n={n} update={ph['update']*1e3:8.1f} us -> {ph['update']*1e3/n:6.2f} us/op  splits={st['splits']} merges={st['merges']}")
