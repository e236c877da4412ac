"""Time the prefill of a config (inserts only) on the GPU."""
import sys, time, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from bench import prefill_gpu, CONFIGS
from paper_conf_ppopp_moscovicicp17_b200.gfsl import GFSL
cfg = sys.argv[1]
R, pre, B, nb, mix, dist, N = CONFIGS[cfg]
g = GFSL(R, capacity=R, chunk_entries=N)
t = time.time(); prefill_gpu(g, R, pre, torch.device("cuda")); torch.cuda.synchronize()
print(cfg, "prefill", pre, "keys in", round(time.time() - t, 2), "s")
rep, _, _ = g.validate(export=False)
print("keys", rep.keys, "height", rep.height, "viol", rep.violations, "chunks", rep.chunks[:rep.height+1])
