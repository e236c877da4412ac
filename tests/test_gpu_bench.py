"""bench.py end to end on the GPU: the 1-GPU JSON line carries the contract's keys, and
the N>1 path (router + NCCL-style all-to-all exchange, or the fused peer-window exchange) runs as 2 ranks sharing one GPU over gloo."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def run(cmd, timeout=600):
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=timeout)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    return json.loads(lines[-1])


def test_bench_single_gpu_line():
    d = run([sys.executable, "bench.py", "--config", "C1", "--steps", "4", "--runs", "3"])
    for k in ["metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step",
              "higher_is_better", "scaling", "dtype", "config", "roofline", "cpu_baseline",
              "clocks", "gpu_launches", "e2e", "runs"]:
        assert k in d, k
    assert d["value"] > 0 and d["roofline"]["peak"] > 0 and d["cpu_baseline"]["kind"] == "oracle"
    assert d["runs"]["n"] == 3 and d["runs"]["ci95_half_width"] is not None
    assert d["cpu_baseline"]["cores"] >= 1 and d["e2e"]["value"] > 0


def test_bench_single_op_config():
    """INS-1M (Fig 5.4b): R inserts into an empty structure, timed from the first."""
    d = run([sys.executable, "bench.py", "--config", "INS-1M", "--runs", "2", "--no-e2e",
             "--no-cpu-baseline", "--no-ubench"])
    assert d["value"] > 0 and d["mutations_per_step"] == 125_000


@pytest.mark.parametrize("exchange,port", [("nccl", 29533), ("peer", 29534)])
def test_bench_two_ranks_gloo(exchange, port):
    d = run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
             "--master-addr", "127.0.0.1", "--master-port", str(port), "bench.py", "--gpus", "2",
             "--config", "C2", "--steps", "3", "--runs", "2", "--dist-backend", "gloo", "--validate",
             "--no-ubench", "--exchange", exchange])
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["validate"]["violations"] == 0
    assert d["scaling"] == "strong" and d["config"]["key_range"] == 1_000_000
    assert d["structure"]["shard"] == [0, 500_000] and d["e2e"]["value"] > 0
