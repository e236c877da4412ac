"""Update-phase breakdown on a C2-like structure: insert-only / delete-only batches of a
given size, phase times and lock retries.  python tools/upd_breakdown.py [R] [B]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from bench import prefill_gpu
from paper_conf_ppopp_moscovicicp17_b200.gfsl import GFSL
from paper_conf_ppopp_moscovicicp17_b200.workload import SEED_BASE, prefill_keys

R = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
B = int(sys.argv[2]) if len(sys.argv) > 2 else 62_500
dev = torch.device("cuda")
g = GFSL(R, capacity=R, profile_phases=True)
prefill_gpu(g, R, R // 2, dev)
perm = prefill_keys(SEED_BASE, R, R, device=dev)
absent = perm[R // 2:]
present = perm[:R // 2]
g.phase_times()
for name, op, keys in [("insert-absent", 1, absent[:B]), ("delete-present", 2, present[:B]),
                       ("insert-present", 1, present[B:2 * B]), ("delete-absent", 2, absent[B:2 * B]),
                       ("insert-absent-2", 1, absent[B:2 * B])]:
    s0 = g.stats()
    g.batch(torch.full((keys.numel(),), op, dtype=torch.uint8, device=dev), keys.to(torch.int32),
            keys.to(torch.int32))
    ph, nb = g.phase_times()
    s1 = g.stats()
    print(f"{name:16s} n={keys.numel()} search={ph['contains']:.4f} update={ph['update']:.4f} ms "
          f"mut={s1['mutations'] - s0['mutations']} retries={s1['lock_retries'] - s0['lock_retries']} "
          f"splits={s1['splits'] - s0['splits']} merges={s1['merges'] - s0['merges']}")
