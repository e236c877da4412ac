"""Build a config's structure, run warm-up batches, then exactly one profiled batch
(cudaProfilerStart/Stop) -- for `ncu --profile-from-start off`.
python tools/prof_step.py C4-32 [--team 4] [--warmup 2]"""
import argparse, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from bench import CONFIGS, make_inputs, prefill_gpu
from paper_conf_ppopp_moscovicicp17_b200.gfsl import GFSL
from paper_conf_ppopp_moscovicicp17_b200.workload import SEED_BASE, Workload

ap = argparse.ArgumentParser()
ap.add_argument("config")
ap.add_argument("--team", type=int, default=0)
ap.add_argument("--warmup", type=int, default=2)
ap.add_argument("--prefill", default="bulk", choices=["bulk", "per-op"])
ap.add_argument("--chunk", type=int, default=0)
a = ap.parse_args()
R, pre, B, nb, mix, dist, N = CONFIGS[a.config]
N = a.chunk or N
dev = torch.device("cuda")
g = GFSL(R, capacity=R, chunk_entries=N, contains_team=a.team)
prefill_gpu(g, R, pre, dev, per_op=a.prefill == "per-op")
w = Workload(R, B, mix=mix, dist=dist, seed=SEED_BASE + 1)
batches = [make_inputs(w, b, dev) for b in range(a.warmup + 1)]
for b in range(a.warmup):
    g.batch(*batches[b][:3])
# as bench.py does before every timed step: flush L2 with a 256-MiB write
torch.empty(256 << 20, dtype=torch.uint8, device=dev).zero_()
torch.cuda.synchronize()
torch.cuda.profiler.start()
g.batch(*batches[a.warmup][:3])
torch.cuda.synchronize()
torch.cuda.profiler.stop()
print("profiled one batch of", B, "ops on", a.config)
