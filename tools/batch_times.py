"""Per-batch phase times and structure counters of a bench config, as bench.py runs it
(same prefill, same batches, L2 flushed before each batch), with profile_phases on.
python tools/batch_times.py CFG [--group on|off] [--bulk auto|off|always] [--steps K]"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_ppopp_moscovicicp17_b200.gfsl import GFSL  # noqa: E402
from paper_conf_ppopp_moscovicicp17_b200.workload import SEED_BASE, Workload  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("config")
ap.add_argument("--group", default="off", choices=["on", "off"])
ap.add_argument("--bulk", default="auto", choices=["auto", "off", "always"])
ap.add_argument("--steps", type=int, default=0)
ap.add_argument("--warmup", type=int, default=3)
a = ap.parse_args()
R, pre, B, nb, mix, dist, N = bench.CONFIGS[a.config]
perm = a.config in bench.PERM_CONFIGS
steps = a.steps or nb
W = 0 if perm else a.warmup
dev = torch.device("cuda")
w = Workload(R, B, mix=mix, dist="uniform" if dist == "perm" else dist, seed=SEED_BASE + 1, dedup=True)
inputs = []
for b in range(W + steps):
    op, key, val, _ = bench.make_batch(a.config, w, b, dev)
    inputs.append((op.contiguous(), key.contiguous(), val.contiguous()))
def run(show):
    g = GFSL(R, capacity=R, chunk_entries=N, profile_phases=True)
    if pre:
        bench.prefill_gpu(g, R, pre, dev)
    g.configure(bulk={"auto": 0, "off": 1, "always": 2}[a.bulk], group=1 if a.group == "on" else 0)
    for b in range(W):
        g.batch(*inputs[b])
    torch.cuda.synchronize()
    g.phase_times()
    flush = torch.empty(bench.L2_FLUSH_BYTES, dtype=torch.uint8, device=dev)
    keys = ["splits", "merges", "lock_retries", "mutations", "grouped", "kernel_launches"]
    prev = g.stats()
    if show: print(f"{a.config} group={a.group} bulk={a.bulk}: batch  intake search update upkeep+rebuild total event (ms) | " + " ".join(keys))
    tot = 0.0
    for j in range(steps):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        g.batch(*inputs[W + j])
        e1.record()
        torch.cuda.synchronize()
        ev_ms = e0.elapsed_time(e1)
        ms, _ = g.phase_times()
        st = g.stats()
        tot += ev_ms
        vals = [ms.get(k, 0.0) for k in ("intake", "contains", "update", "upkeep", "total")] + [ev_ms]
        if show: print(f"  {j:3d} " + " ".join(f"{v:8.4f}" for v in vals) + " | " +
              " ".join(str(st[k] - prev[k]) for k in keys))
        prev = st
    if show: print(f"  sum {tot:.4f} ms -> {B * steps / tot / 1e3:.1f} Mops/s")
    g.close()


run(False)  # a warm process (lazy module loading, allocator pools), as bench.py's run -1
run(True)
