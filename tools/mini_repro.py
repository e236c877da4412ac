import sys, os
sys.path.insert(0, "/root/repo")
import numpy as np, torch
from paper_conf_ppopp_moscovicicp17_b200.gfsl import GFSL
from paper_conf_ppopp_moscovicicp17_b200.workload import SEED_BASE, prefill_keys, prefill_values
R = 20000
g = GFSL(R, chunk_entries=32, contains_team=8)
k = prefill_keys(SEED_BASE, R, 10000); v = prefill_values(SEED_BASE, k)
r = g.batch(torch.ones(10000, dtype=torch.uint8, device="cuda"), k.to(torch.int32).cuda(), v.to(torch.int32).cuda())
torch.cuda.synchronize(); print(r.sum())
