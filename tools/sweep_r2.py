"""NEXT-4: the paper's workload sweep on one B200 -- Fig 5.3 (mixes [1,1,98],
[5,5,90], [10,10,80], [20,20,60], 10M ops, key ranges 10K-100M, half-full start) and Fig
5.4 (Contains-only 10M ops on a full structure; Insert-only R ops from empty; Delete-only R
ops from full), each point `--runs` independent runs with a 95% CI.
Batches hold at most R / (2 x mutating fraction) ops so that the <=1-mutation-per-key
contract stays cheap for the generator (R2).
    python tools/sweep_r2.py OUT.jsonl [--runs 3] [--ranges 10000,100000,...]"""
import argparse
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ap = argparse.ArgumentParser()
ap.add_argument("out")
ap.add_argument("--runs", type=int, default=3)
ap.add_argument("--ranges", default="10000,100000,1000000,10000000,100000000")
ap.add_argument("--chunk", type=int, default=16)
a = ap.parse_args()
points = []
for R in [int(x) for x in a.ranges.split(",")]:
    for mix in ((1, 1, 98), (5, 5, 90), (10, 10, 80), (20, 20, 60)):
        mut = (mix[0] + mix[1]) / 100.0
        B = int(min(10_000_000, max(1000, R / (2 * mut))))
        nb = max(1, 10_000_000 // B)
        points.append((f"mix{mix[0]}-{mix[1]}-{mix[2]}", f"{R}:{R // 2}:{B}:{nb}:{mix[0]},{mix[1]},{mix[2]}:uniform:{a.chunk}"))
    B = min(10_000_000, R)
    points.append(("contains", f"{R}:{R}:{min(10_000_000, 10_000_000)}:1:0,0,100:uniform:{a.chunk}"))
    Bi = max(1000, R // 8)
    points.append(("insert", f"{R}:0:{Bi}:{R // Bi}:100,0,0:perm:{a.chunk}"))
    points.append(("delete", f"{R}:{R}:{Bi}:{R // Bi}:0,100,0:perm:{a.chunk}"))
with open(a.out, "a") as f:
    for name, spec in points:
        cmd = [sys.executable, "bench.py", "--config", "custom", "--custom", spec, "--runs", str(a.runs),
               "--no-e2e", "--no-cpu-baseline", "--no-ubench", "--warmup", "3"]
        r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=1200)
        line = next((l for l in r.stdout.splitlines()[::-1] if l.startswith("{")), None)
        rec = {"point": name, "spec": spec, "rc": r.returncode}
        if line:
            d = json.loads(line)
            rec.update(value=d["value"], runs=d["runs"], ms_per_step=d["ms_per_step"],
                       phases=d["phase_ms_per_step"], reads=d["chunk_reads_per_contains"],
                       board=d["clocks"].get("uuid"))
        else:
            rec["err"] = r.stderr[-800:]
        f.write(json.dumps(rec) + "\n")
        f.flush()
        print(json.dumps(rec), flush=True)
