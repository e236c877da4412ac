"""Cost of one upper-level rebuild with the level-0 relocation (R24 + R38) at a config's
size: prefill (bulk), a few batches, then gfsl_rebuild timed with CUDA events (the rebuild
runs only when a batch mutated the structure since the last one).
python tools/rebuild_cost.py [C5]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_ppopp_moscovicicp17_b200.gfsl import GFSL  # noqa: E402
from paper_conf_ppopp_moscovicicp17_b200.workload import SEED_BASE, Workload  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
R, pre, B, nb, mix, dist, N = bench.CONFIGS[cfg]
dev = torch.device("cuda")
g = GFSL(R, capacity=R, chunk_entries=N)  # default wear policy: no rebuild within 6 batches
bench.prefill_gpu(g, R, pre, dev)
w = Workload(R, B, mix=mix, dist=dist, seed=SEED_BASE + 1)
out = []
for rep in range(3):
    for b in range(2):
        g.batch(*bench.make_batch(cfg, w, 2 * rep + b, dev)[:3])
    torch.cuda.synchronize()
    a, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    g.rebuild()
    e.record()
    torch.cuda.synchronize()
    out.append(a.elapsed_time(e))
d = g.check()
print(json.dumps({"config": cfg, "rebuild_ms": [round(x, 3) for x in out], "batch_ops": B,
                  "violations": d.violations, "keys": d.keys}))
