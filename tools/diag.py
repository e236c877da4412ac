"""Structure diagnostics on the GPU: per-level sizes, fill, down-pointer staleness and
chunk reads per Contains, fresh and after churn.  python tools/diag.py [R] [N]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_moscovicicp17_b200.gfsl import GFSL  # noqa: E402
from paper_conf_ppopp_moscovicicp17_b200.workload import (  # noqa: E402
    SEED_BASE, Workload, prefill_keys, prefill_values)


def analyse(g: GFSL, tag: str):
    meta, ent = g.dump()
    N = meta["chunk_entries"]
    lo = (ent & 0xFFFFFFFF).astype(np.uint64)
    hi = (ent >> np.uint64(32)).astype(np.uint64)
    rep, _, _ = g.validate(export=False, raise_on_violation=False)
    print(f"== {tag}: keys={rep.keys} height={rep.height} viol=0x{rep.violations:x} "
          f"underfull={rep.underfull} pool_used={rep.pool_used}")
    holder = {}
    levels = []
    for l in range(N):
        c = meta["head"][l]
        chain = []
        while c != 0xFFFFFFFF and len(chain) < 10_000_000:
            chain.append(c)
            c = int(hi[c, N - 2])
        nz = [c for c in chain if lo[c, N - 1] != 2]
        keys = [(int(lo[c, i]), int(hi[c, i]), c) for c in nz for i in range(N - 2)
                if lo[c, i] != 0xFFFFFFFF and lo[c, i] != 0]
        levels.append((chain, nz, keys))
        if l <= rep.height + 1:
            fill = np.mean([sum(1 for i in range(N - 2) if lo[c, i] != 0xFFFFFFFF) for c in nz]) if nz else 0
            print(f"  L{l}: chunks={len(nz)} zombies={len(chain) - len(nz)} keys={len(keys)} "
                  f"fill={fill:.2f} counter={meta['counters'][l]}")
    # staleness: for each key at level l+1, lateral hops from its pointer to its chunk at l
    for l in range(min(rep.height, N - 1)):
        pos = {c: i for i, c in enumerate(levels[l][0])}
        where = {k: c for k, _, c in levels[l][2]}
        hops = []
        for k, ptr, _ in levels[l + 1][2]:
            if k in where and ptr in pos:
                hops.append(pos[where[k]] - pos[ptr])
        if hops:
            h = np.array(hops)
            print(f"  ptr L{l + 1}->L{l}: mean hops={h.mean():.3f} max={h.max()} "
                  f"frac>0={np.mean(h > 0):.3f}")


def reads_per_contains(g: GFSL, R, dev):
    g.configure(count_reads=1)
    s0 = g.stats()
    k = torch.randint(0, R, (200_000,), device=dev, dtype=torch.int32)
    g.batch(torch.zeros(k.numel(), dtype=torch.uint8, device=dev), k)
    torch.cuda.synchronize()
    s1 = g.stats()
    g.configure(count_reads=0)
    ops = s1["contains_ops"] - s0["contains_ops"]
    print(f"  reads/contains={(s1['contains_reads'] - s0['contains_reads']) / ops:.3f} "
          f"L0 reads={(s1['contains_reads_l0'] - s0['contains_reads_l0']) / ops:.3f}")


def main():
    R = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
    N = int(sys.argv[2]) if len(sys.argv) > 2 else 32
    dev = torch.device("cuda")
    for serial in (False,):
        g = GFSL(R, chunk_entries=N, serial_updates=serial)
        k = prefill_keys(SEED_BASE, R, R // 2, device=dev)
        v = prefill_values(SEED_BASE, k)
        g.batch(torch.ones(k.numel(), dtype=torch.uint8, device=dev), k.to(torch.int32), v.to(torch.int32))
        torch.cuda.synchronize()
        analyse(g, f"fresh prefill R={R} N={N} serial={serial}")
        reads_per_contains(g, R, dev)
        w = Workload(R, R // 16 * 10, mix=(10, 10, 80), seed=SEED_BASE + 1)
        for b in range(16):
            op, key, val, _ = w.make_batch(b, device=dev)
            g.batch(op, key.to(torch.int32), val.to(torch.int32))
            if b in (3, 15):
                torch.cuda.synchronize()
                analyse(g, f"after {b + 1} batches of 10/10/80")
                reads_per_contains(g, R, dev)
        print(g.stats())


if __name__ == "__main__":
    main()
