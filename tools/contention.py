"""Update-kernel latency vs contention: deletes of keys from distinct chunks (one per
chunk, no lock contention) vs the same number of random present keys; inserts likewise.
python tools/contention.py [R] [n]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from bench import prefill_gpu
from paper_conf_ppopp_moscovicicp17_b200.gfsl import GFSL
from paper_conf_ppopp_moscovicicp17_b200.workload import SEED_BASE, prefill_keys

R = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
n = int(sys.argv[2]) if len(sys.argv) > 2 else 25_000
dev = torch.device("cuda")


def fresh():
    g = GFSL(R, capacity=R, profile_phases=True)
    prefill_gpu(g, R, R // 2, dev)
    return g


def run(g, op, keys, name):
    g.phase_times()
    k = torch.as_tensor(np.asarray(keys, np.int64)).to(torch.int32).to(dev)
    g.batch(torch.full((k.numel(),), op, dtype=torch.uint8, device=dev), k, k)
    ph, _ = g.phase_times()
    print(f"{name:28s} n={k.numel():7d} search={ph['contains']*1e3:7.1f} us update={ph['update']*1e3:7.1f} us")


g = fresh()
meta, ent = g.dump()
N = meta["chunk_entries"]
lo = (ent & 0xFFFFFFFF).astype(np.int64)
# level-0 chain
c, chain = meta["head"][0], []
while c != 0xFFFFFFFF:
    chain.append(c)
    c = int(ent[c, N - 2] >> np.uint64(32))
# one key per chunk (the 2nd key: never the chunk minimum, so never at level 1)
one = [int(lo[c, 1]) - 1 for c in chain[1:] if lo[c, 1] not in (0, 0xFFFFFFFF) and lo[c, 2] != 0xFFFFFFFF]
one = one[::max(1, len(one) // n)][:n]
run(g, 2, one, "delete distinct chunks")
g = fresh()
present = prefill_keys(SEED_BASE, R, R // 2).numpy()
run(g, 2, present[:len(one)], "delete random")
g = fresh()
# inserts: one absent key per chunk (just above its 2nd key, if absent)
absent_all = set(prefill_keys(SEED_BASE, R, R).numpy()[R // 2:].tolist())
ins = []
for c in chain[1:]:
    k2 = int(lo[c, 1]) - 1
    if k2 + 1 in absent_all:
        ins.append(k2 + 1)
ins = ins[:len(one)]
run(g, 1, ins, "insert distinct chunks")
g = fresh()
run(g, 1, list(absent_all)[:len(ins)], "insert random")
