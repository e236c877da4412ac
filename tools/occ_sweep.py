"""Update-kernel time vs update blocks per SM (phase timing).  python tools/occ_sweep.py C3"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from bench import CONFIGS, make_inputs, prefill_gpu
from paper_conf_ppopp_moscovicicp17_b200 import gfsl as G
from paper_conf_ppopp_moscovicicp17_b200.workload import SEED_BASE, Workload

cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
R, pre, B, nb, mix, dist, N = CONFIGS[cfg]
dev = torch.device("cuda")
g = G.GFSL(R, capacity=R, chunk_entries=N, rebuild_every=-1 & 0xFFFFFFFF)
prefill_gpu(g, R, pre, dev)
w = Workload(R, B, mix=mix, dist=dist, seed=SEED_BASE + 1)
b = 0
for bps in (6, 5, 4, 3, 2, 1, 6):
    g.configure(update_blocks_per_sm=bps, profile_phases=1)
    g.phase_times()
    for _ in range(4):
        g.batch(*make_inputs(w, b, dev)[:3])
        b += 1
    torch.cuda.synchronize()
    ms, n = g.phase_times()
    st = g.stats()
    print(f"{cfg} update blocks/SM {bps}: update {ms['update'] / n * 1e3:7.1f} us/batch  search {ms['contains'] / n * 1e3:6.1f}")
