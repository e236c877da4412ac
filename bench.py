#!/usr/bin/env python3
"""GFSL batched Contains/Insert/Delete benchmark on B200 (BASELINE.json `metric`).

One JSON line on rank 0.  A "step" is one collective `gfsl_batch` over one global batch of
synthetic ops (search kernel -> update kernel -> upkeep; with N > 1 GPUs also the route
kernels and the peer-window exchange); `value` is Mops/s = all ops of the K timed steps /
the slowest rank's summed CUDA-event step time, averaged over `--runs` independent runs
(the paper's 10 runs with a 95% CI), each on a freshly prefilled structure with
the same seeds.  Inputs are resident in HBM before each timed step; L2 is flushed (a
256 MiB write) before every timed step.

    python bench.py [--config C5] [--gpus N --steps K --warmup W] [--runs 10] [--impl reference]

Default workload: C5 (BASELINE.json configs[4]): a 1B-key range, 500M keys
prefilled in random order, 125M-op global batches of [10,10,80] uniform ops.  N > 1 is
STRONG scaling: the key range stays 1B, shard g owns [g*ceil(R/N), (g+1)*ceil(R/N)) as a
GFSL over its local key space, each rank issues its 1/N slice of every global batch, and the
fused route kernels move ops and results through the peers' windows.
Other configs (C1 .. C4, NEXT-4 workloads): `--config`.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import sys
import threading
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from paper_conf_ppopp_moscovicicp17_b200.workload import (  # noqa: E402
    SEED_BASE, Workload, prefill_keys, prefill_values)

METRIC = "Mops/s (mixed insert/delete/contains)"
L2_BYTES = 126 << 20          # B200 L2 (B200_PROFILING.md)
L2_FLUSH_BYTES = 256 << 20

# name: (R, prefill, batch, n_batches, mix, dist, N)
# N = chunk entries.  The paper's runs use N = 32; on B200 N = 16 (128-B chunks,
# 2-lane teams) is faster on every config measured: a chunk read costs L1
# data-pipe wavefronts in proportion to its bytes, and since level 0 is entered directly
# from the directory (R37/R38) the smaller level 1 of N = 32 no longer pays off (C5 in one
# gpurun call: 7534 vs 6660 Mops/s).  The C4 pair compares the two; --chunk N overrides.
CONFIGS = {
    "C1": (10_000, 5_000, 6_250, 16, (10, 10, 80), "uniform", 16),
    "C2": (1_000_000, 500_000, 625_000, 16, (10, 10, 80), "uniform", 16),
    "C2-100": (1_000_000, 1_000_000, 10_000_000, 1, (0, 0, 100), "uniform", 16),
    "C2-2020": (1_000_000, 500_000, 312_500, 32, (20, 20, 60), "uniform", 16),
    "C2-5050": (1_000_000, 500_000, 125_000, 80, (50, 50, 0), "uniform", 16),
    "C3": (10_000_000, 5_000_000, 6_250_000, 16, (10, 10, 80), "uniform", 16),
    "C3-zipf": (10_000_000, 5_000_000, 6_250_000, 16, (10, 10, 80), "zipf", 16),
    "C4-32": (100_000_000, 100_000_000, 50_000_000, 10, (0, 0, 100), "uniform", 32),
    "C4-16": (100_000_000, 100_000_000, 50_000_000, 10, (0, 0, 100), "uniform", 16),
    "C5": (1_000_000_000, 500_000_000, 125_000_000, 8, (10, 10, 80), "uniform", 16),
    # one shard of C5 strong-scaled over G = 2 / 4 / 8 GPUs (R/G keys, its 1/G slice of
    # every global batch, uniform in the shard's local key space), on one GPU: the local
    # work of each rank of `--gpus G --config C5` without the exchange
    "C5-S2": (500_000_000, 250_000_000, 62_500_000, 8, (10, 10, 80), "uniform", 16),
    "C5-S4": (250_000_000, 125_000_000, 31_250_000, 8, (10, 10, 80), "uniform", 16),
    "C5-S8": (125_000_000, 62_500_000, 15_625_000, 8, (10, 10, 80), "uniform", 16),
    # NEXT-4: the paper's other workloads (Fig 5.3 mixes, Fig 5.4b/c single-op runs)
    "M1-1-98": (1_000_000, 500_000, 625_000, 16, (1, 1, 98), "uniform", 16),
    "M5-5-90": (1_000_000, 500_000, 625_000, 16, (5, 5, 90), "uniform", 16),
    "M20-20-60-10M": (10_000_000, 5_000_000, 625_000, 16, (20, 20, 60), "uniform", 16),
    # Fig 5.4b/c: R Inserts into an EMPTY structure / R Deletes from a FULL one,
    # as one timed run from the first op (warm-up batches would change the start state)
    "INS-1M": (1_000_000, 0, 125_000, 8, (100, 0, 0), "perm", 16),
    "DEL-1M": (1_000_000, 1_000_000, 125_000, 8, (0, 100, 0), "perm", 16),
    # NEXT-1: raw Zipf(0.99) -- mutating keys i.i.d. too (no redraws), so hot keys carry
    # long Insert/Delete chains; run in combining mode (R26), exact for any batch
    "C2-zipf-raw": (1_000_000, 500_000, 625_000, 16, (10, 10, 80), "zipf", 16),
    "C3-zipf-raw": (10_000_000, 5_000_000, 6_250_000, 16, (10, 10, 80), "zipf", 16),
}
COMBINE_CONFIGS = {"C2-zipf-raw", "C3-zipf-raw"}
# single-op configs: every key once, in permutation order, no warm-up batches
PERM_CONFIGS = {"INS-1M", "DEL-1M"}


def combine_mode(args) -> bool:
    return args.config in COMBINE_CONFIGS or getattr(args, "combine", False)


def load_traffic(cfg):
    """ncu DRAM bytes per launch of each kernel for this config (profiles/traffic_*.json)."""
    import glob
    for p in sorted(glob.glob(os.path.join(ROOT, "profiles", "traffic_r*.json")), reverse=True):
        try:
            with open(p) as f:
                t = json.load(f)["traffic_bytes_per_launch"].get(cfg)
            if t:
                return t, os.path.basename(p)
        except Exception:
            pass
    return {}, None


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md)"


def ci95(xs):
    """Mean and the half-width of its 95% confidence interval (Student t)."""
    n = len(xs)
    m = statistics.fmean(xs)
    if n < 2:
        return m, None
    t = {2: 12.706, 3: 4.303, 4: 3.182, 5: 2.776, 6: 2.571, 7: 2.447, 8: 2.365, 9: 2.306,
         10: 2.262, 11: 2.228, 12: 2.201, 16: 2.131, 21: 2.086, 31: 2.042}
    tv = t.get(n) or min((v for k, v in t.items() if k <= n), default=1.96)
    return m, tv * statistics.stdev(xs) / math.sqrt(n)


class ClockSampler:
    """NVML SM clock + throttle reasons, sampled in a thread during the timed region."""

    REASONS = {
        0x0000000000000008: "hw_slowdown", 0x0000000000000040: "hw_thermal_slowdown",
        0x0000000000000020: "sw_thermal_slowdown", 0x0000000000000004: "sw_power_cap",
        0x0000000000000080: "hw_power_brake_slowdown",
    }

    def __init__(self, dev_index: int):
        self.samples, self.reasons, self.ok = [], set(), False
        self.max_mhz = None
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.hdl = pynvml.nvmlDeviceGetHandleByIndex(dev_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.hdl, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception:
            self.ok = False
        self._stop = threading.Event()
        self.t = None

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.hdl, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.hdl)
                for bit, name in self.REASONS.items():
                    if r & bit:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.002)

    def start(self):
        if self.ok and self.t is None:
            self._stop.clear()
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()

    def pause(self):
        if self.ok and self.t is not None:
            self._stop.set()
            self.t.join()
            self.t = None

    def result(self):
        self.pause()
        out = {"sm_mhz": statistics.median(self.samples) if self.samples else None,
               "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
               "samples": len(self.samples)}
        if self.ok:  # which board this ran on (box-to-box variance of HBM random access)
            nv = self.nv
            for k, f in (("mem_mhz", lambda: nv.nvmlDeviceGetClockInfo(self.hdl, nv.NVML_CLOCK_MEM)),
                         ("mem_max_mhz", lambda: nv.nvmlDeviceGetMaxClockInfo(self.hdl, nv.NVML_CLOCK_MEM)),
                         ("ecc", lambda: nv.nvmlDeviceGetEccMode(self.hdl)[0]),
                         ("uuid", lambda: nv.nvmlDeviceGetUUID(self.hdl)),
                         ("vbios", lambda: nv.nvmlDeviceGetVbiosVersion(self.hdl))):
                try:
                    v = f()
                    out[k] = v.decode() if isinstance(v, bytes) else v
                except Exception:
                    pass
        return out


def dist_setup(backend="nccl"):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if backend == "gloo":  # test path: several ranks may share one GPU
        local = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    if world > 1:
        import torch.distributed as dist
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    return world, rank, local


def barrier(world):
    if world > 1:
        import torch.distributed as dist
        dist.barrier()


def max_over_ranks(x: float, world: int) -> float:
    if world == 1:
        return x
    import torch.distributed as dist
    dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor([x], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def slices(n: int, world: int):
    q, rem = divmod(n, world)
    out, a = [], 0
    for r in range(world):
        b = a + q + (1 if r < rem else 0)
        out.append((a, b))
        a = b
    return out


# --------------------------------------------------------------------------------------
# inputs (seeded, synthetic)

def make_batch(cfg_name, w: Workload, b: int, dev):
    """Global batch b of the config: (op u8, key i32, val i32) on `dev`."""
    R, pre, B, nb, mix, dist, N = CONFIGS[cfg_name]
    if dist == "perm":  # Fig 5.4b/c: every key of [0, R) once, in random order
        key = prefill_keys(SEED_BASE + 2, R, B, start=b * B, device=dev)
        op = torch.full((B,), 1 if mix[0] else 2, dtype=torch.uint8, device=dev)
        val = prefill_values(SEED_BASE + 2, key)
        return op, key.to(torch.int32), val.to(torch.int32), 0
    op, key, val, redraws = w.make_batch(b, device=dev)
    return op.contiguous(), key.to(torch.int32).contiguous(), val.to(torch.int32).contiguous(), redraws


def make_inputs(w: Workload, b: int, dev):  # (tools/ compatibility)
    op, key, val, redraws = w.make_batch(b, device=dev)
    return op.contiguous(), key.to(torch.int32).contiguous(), val.to(torch.int32).contiguous(), redraws


def prefill_gpu(g, R, count, dev, key_lo=0, key_hi=None, seed=SEED_BASE, per_op=False):
    """Random-order inserts of the first `count` elements of the keyed permutation of
    [0, R).  Default: ONE insert batch, which the library applies through its bulk path
    (R34: sorted and merged into level 0, upper levels rebuilt).  per_op=True:
    the paper's per-op Insert path, in insert-only batches that grow with the structure (a
    batch never exceeds ~1/4 of the keys present, so concurrent inserts spread over many
    chunks), then a rebuild.  With [key_lo, key_hi) (a shard), only the keys in the shard
    are inserted, in the same order, rebased to the shard's local key space (as the route
    kernels rebase them)."""
    key_hi = R if key_hi is None else key_hi
    parts = []
    for s in range(0, count, 1 << 25):
        k = prefill_keys(seed, R, min(1 << 25, count - s), start=s, device=dev)
        if key_lo or key_hi != R:
            k = k[(k >= key_lo) & (k < key_hi)]
        parts.append(k)
    k = torch.cat(parts) if parts else torch.empty(0, dtype=torch.int64, device=dev)
    del parts
    v = prefill_values(seed, k).to(torch.int32)
    k = (k - key_lo).to(torch.int32)
    cap = (1 << 29) - 1  # GFSL_MAX_BATCH
    ones = torch.ones(min(k.numel(), cap), dtype=torch.uint8, device=dev)
    have = 0
    while have < k.numel():
        c = min(k.numel() - have, max(4096, have // 4), 1 << 26) if per_op else min(k.numel() - have, cap)
        g.batch(ones[:c], k[have:have + c], v[have:have + c])
        have += c
    del k, v, ones
    if per_op:
        g.rebuild()  # bulk-load compaction of the upper levels (gfsl_rebuild, R29)
    torch.cuda.synchronize()


# --------------------------------------------------------------------------------------
# reference arm / cpu baseline: the oracle as it stands, on this host's cores

def oracle_sample(cfg_name, steps, warmup, budget_s=20.0, threads=1, combine=False):
    """Times Oracle-A (the sequential Pugh skiplist, S1 batches) on a bounded sample of the
    config on `threads` host threads, range-sharded as SURVEY 8(d)(ii): thread t owns a
    contiguous key range with its own skiplist, and each batch is pre-bucketed by key (the
    bucketing time is reported separately).  The oracle calls release the GIL (ctypes), so
    the shards run in parallel.  Sample: the config itself when small; else key-range
    shards of 2M keys each (one per thread) at the config's prefill density and mix."""
    from concurrent.futures import ThreadPoolExecutor
    from oracle.oracle_a import OracleMap
    R, pre, B, nb, mix, dist, N = CONFIGS[cfg_name]
    T = max(1, int(threads))
    if R > 4_000_000:
        Rs = 2_000_000 * T
        pre_s = int(round(pre * Rs / R))
        note = f"key range [0,{Rs}) ({T} shards of 2M keys) of R={R} at the same fill, same mix"
    else:
        Rs, pre_s, note = R, pre, f"the config itself (R={R})"
    Bs = min(B, 250_000 * T) if R > 4_000_000 else min(B, 1_000_000)
    bounds = [(t * Rs // T, (t + 1) * Rs // T) for t in range(T)]
    maps = [OracleMap(Rs) for _ in range(T)]
    pool = ThreadPoolExecutor(T)
    if pre_s:
        k = prefill_keys(SEED_BASE, Rs, pre_s).numpy()
        v = prefill_values(SEED_BASE, torch.from_numpy(k)).numpy().astype(np.uint32)
        k = k.astype(np.uint32)
        parts = [(k >= lo) & (k < hi) for lo, hi in bounds]
        list(pool.map(lambda t: maps[t].batch(np.ones(int(parts[t].sum()), np.uint8), k[parts[t]], v[parts[t]]),
                      range(T)))
    w = Workload(Rs, Bs, mix=mix, dist="uniform" if dist == "perm" else dist, seed=SEED_BASE + 1,
                 dedup=not combine)
    batches = []
    for b in range(warmup + steps):
        op, key, val, _ = w.make_batch(b)
        batches.append((op.numpy(), key.numpy().astype(np.uint32), val.numpy().astype(np.uint32)))

    def bucket(batch):
        op, key, val = batch
        shard = np.minimum((key.astype(np.int64) * T) // Rs, T - 1)
        order = np.argsort(shard, kind="stable")
        cuts = np.searchsorted(shard[order], np.arange(T + 1))
        return [(op[order[cuts[t]:cuts[t + 1]]], key[order[cuts[t]:cuts[t + 1]]],
                 val[order[cuts[t]:cuts[t + 1]]]) for t in range(T)], order

    def run(parts):
        return list(pool.map(lambda t: maps[t].batch(*parts[t], combine=combine), range(T)))

    for b in range(warmup):
        run(bucket(batches[b])[0])
    t_total = t_bucket = 0.0
    n_total = done = 0
    for b in range(warmup, warmup + steps):
        t0 = time.perf_counter()
        parts, _ = bucket(batches[b])
        t1 = time.perf_counter()
        run(parts)
        t2 = time.perf_counter()
        t_bucket += t1 - t0
        t_total += t2 - t1
        n_total += Bs
        done += 1
        if t_total + t_bucket > budget_s:
            break
    pool.shutdown()
    for m in maps:
        m.close()
    mops = n_total / t_total / 1e6
    return {"mops": mops, "mops_incl_bucketing": n_total / (t_total + t_bucket) / 1e6,
            "seconds": t_total, "bucket_seconds": t_bucket, "batches": done, "batch_ops": Bs,
            "threads": T, "note": note}


def cpu_info():
    model = None
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except Exception:
        pass
    return {"nproc": os.cpu_count(), "model": model}


def cpu_baseline_obj(cfg, steps, combine, budget_each=12.0):
    T = os.cpu_count() or 1
    mt = oracle_sample(cfg, min(steps, 16), 1, budget_s=budget_each, threads=T, combine=combine)
    st = oracle_sample(cfg, min(steps, 16), 1, budget_s=budget_each / 2, threads=1, combine=combine)
    return {"value": round(mt["mops"], 4), "unit": "Mops/s", "cores": mt["threads"], "kind": "oracle",
            "sample": (f"{mt['batches']} batches of {mt['batch_ops']} ops ({mt['seconds']:.1f} s) on "
                       f"{mt['threads']} threads, range-sharded Oracle-A (sequential Pugh skiplist, S1 "
                       f"batches) per thread; {mt['note']}; bucketing by key range excluded "
                       f"({mt['bucket_seconds']:.2f} s; incl. it {mt['mops_incl_bucketing']:.2f} Mops/s)"),
            "single_thread": {"value": round(st["mops"], 4), "cores": 1,
                              "sample": f"{st['batches']} batches of {st['batch_ops']} ops; {st['note']}"},
            "cpu": cpu_info()}


def run_reference(args, world, rank):
    if rank != 0:
        return
    cfg = args.config
    T = os.cpu_count() or 1
    r = oracle_sample(cfg, args.steps, args.warmup, budget_s=60.0, threads=T, combine=combine_mode(args))
    line = {
        "impl": "reference", "metric": METRIC, "value": round(r["mops"], 4), "unit": "Mops/s",
        "n_gpus": args.gpus, "steps": r["batches"], "warmup": args.warmup,
        "ms_per_step": round(1000 * r["seconds"] / max(r["batches"], 1), 3), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": cfg, "batch_ops_sampled": r["batch_ops"]},
        "cpu_baseline": {"value": round(r["mops"], 4), "unit": "Mops/s", "cores": r["threads"],
                         "kind": "oracle",
                         "sample": (f"{r['batches']} batches of {r['batch_ops']} ops on {r['threads']} "
                                    f"threads, range-sharded Oracle-A (sequential Pugh skiplist, S1 "
                                    f"batches); {r['note']}"),
                         "cpu": cpu_info()},
        "e2e": {"value": round(r["mops"], 4), "unit": "Mops/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# --------------------------------------------------------------------------------------
# GPU arm

class Setup:
    """The run's handle factory: one GFSL (N = 1) or this rank's shard of a range-sharded
    GFSL with the fused peer-window exchange (default) or the NCCL all-to-all router."""

    def __init__(self, args, world, rank, dev):
        self.args, self.world, self.rank, self.dev = args, world, rank, dev
        R, pre, B, nb, mix, dist, N = CONFIGS[args.config]
        self.N = args.chunk or N
        self.R, self.pre, self.B = R, pre, B
        from paper_conf_ppopp_moscovicicp17_b200.router import shard_bounds
        self.lo, self.hi, _ = shard_bounds(R, world, rank) if world > 1 else (0, R, R)
        self.sl = slices(B, world)[rank]
        self.max_slice = max(b - a for a, b in slices(B, world))

    def create(self):
        a, kw = self.args, dict(chunk_entries=self.N, contains_team=self.args.team,
                                 contains_blocks_per_sm=self.args.contains_blocks,
                                 update_blocks_per_sm=self.args.update_blocks)
        if self.world > 1 and a.exchange == "peer":
            from paper_conf_ppopp_moscovicicp17_b200.router import PeerShardedGFSL
            g = PeerShardedGFSL(self.R, self.rank, self.world, max_slice=self.max_slice, **kw)
            local = g.local
        elif self.world > 1:
            from paper_conf_ppopp_moscovicicp17_b200.router import ShardedGFSL
            g = ShardedGFSL(self.R, self.rank, self.world, **kw)
            local = g.local
        else:
            from paper_conf_ppopp_moscovicicp17_b200.gfsl import GFSL
            g = GFSL(self.R, capacity=self.R, **kw)
            local = g
        if self.pre:
            prefill_gpu(local, self.R, self.pre, self.dev, key_lo=self.lo, key_hi=self.hi,
                        per_op=self.args.prefill == "per-op")
        local.configure(bulk={"auto": 0, "off": 1, "always": 2}[a.bulk],
                        group=1 if a.group == "on" else 0,
                        combine=1 if combine_mode(a) else 0,
                        p_chunk_q32=max(1, int(a.p_chunk * 2**32)) if a.p_chunk < 1.0 else 0,
                        l2_window=a.l2_window, no_pdl=1 if a.no_pdl else 0,
                        rebuild_every=0xFFFFFFFF if a.rebuild_every < 0 else a.rebuild_every)
        barrier(self.world)
        return g, local

    @staticmethod
    def close(g):
        if hasattr(g, "xr"):
            g.xr.close()
        (g.local if hasattr(g, "local") else g).close()
        torch.cuda.synchronize()


def run_gpu(args, world, rank, local_rank):
    dev = torch.device("cuda", local_rank)
    S = Setup(args, world, rank, dev)
    R, pre, B, nb, mix, dist, N0 = CONFIGS[args.config]
    N = S.N
    perm_cfg = args.config in PERM_CONFIGS
    steps = args.steps if args.steps else nb
    W = 0 if perm_cfg else args.warmup
    hbm_peak, peak_kind = load_peaks()
    PROF = 0 if perm_cfg else 3  # extra batches after the timed region, for the per-kernel breakdown
    a, b_ = S.sl

    # the global batches (same seeds on every rank); this rank keeps its slice
    w = Workload(R, B, mix=mix, dist="uniform" if dist == "perm" else dist, seed=SEED_BASE + 1,
                 dedup=not combine_mode(args))
    inputs, redraws = [], 0
    for b in range(W + steps + PROF):
        op, key, val, rd = make_batch(args.config, w, b, dev)
        inputs.append((op[a:b_].contiguous(), key[a:b_].contiguous(), val[a:b_].contiguous()))
        redraws += rd
        del op, key, val
    n_local = b_ - a
    flush = torch.empty(L2_FLUSH_BYTES, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream()
    clocks = ClockSampler(local_rank)

    runs_mops, runs_ms, launches, lib_launches, wall_total = [], [], 0, 0, 0.0
    extras = {}
    # single-op configs start from a fixed state, so their warm-up is one whole untimed run
    # of the sequence on a throwaway handle (run -1)
    for run in range(-1 if perm_cfg else 0, args.runs):
        g, local_g = S.create()
        for b in range(W):
            g.batch(*inputs[b])
        torch.cuda.synchronize()
        st0 = local_g.stats()
        starts = [torch.cuda.Event(enable_timing=True) for _ in range(steps)]
        ends = [torch.cuda.Event(enable_timing=True) for _ in range(steps)]
        barrier(world)
        torch.cuda.synchronize()
        clocks.start()
        wall0 = time.perf_counter()
        for j in range(steps):
            flush.zero_()  # L2 flush between timed steps (outside the step's events)
            starts[j].record(stream)
            g.batch(*inputs[W + j])
            ends[j].record(stream)
        torch.cuda.synchronize()
        barrier(world)
        clocks.pause()
        if run < 0:
            S.close(g)
            continue
        wall_total += time.perf_counter() - wall0
        local_ms = sum(s.elapsed_time(e) for s, e in zip(starts, ends))
        total_ms = max_over_ranks(local_ms, world)
        runs_ms.append(total_ms)
        runs_mops.append(B * steps / (total_ms / 1e3) / 1e6)
        st_t = local_g.stats()
        if run == 0:
            extras = run_extras(args, S, g, local_g, inputs, W, steps, PROF, st0, st_t, flush, dev)
            # our kernels launched inside the timed region (counted by libgfsl at enqueue),
            # plus the route/exchange kernels: peer exchange 3 plan + counts + wait + push +
            # arrive + wait + arrive + wait + pull per step; NCCL router 3 plan + pack + unpack
            route_k = (11 if args.exchange == "peer" else 5) if world > 1 else 0
            launches = int(st_t["kernel_launches"] - st0["kernel_launches"]) + route_k * steps
            lib_launches = int(st_t["library_launches"] - st0["library_launches"])
        S.close(g)

    mean_mops, half = ci95(runs_mops)
    mean_ms = statistics.fmean(runs_ms)
    clk = clocks.result()

    e2e = None
    if not args.no_e2e:
        e2e = run_e2e(args, S, inputs, W, steps, world, dev)

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline_obj(args.config, steps, combine_mode(args))

    if rank == 0:
        ex = extras
        line = {
            "metric": METRIC, "value": round(mean_mops, 3), "unit": "Mops/s", "n_gpus": world,
            "steps": steps, "warmup": W if not perm_cfg else "one untimed run of the whole sequence",
            "ms_per_step": round(mean_ms / steps, 4),
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": "u32", "data": "synthetic",
            "runs": {"n": len(runs_mops), "mean": round(mean_mops, 3),
                     "ci95_half_width": None if half is None else round(half, 3),
                     "values": [round(x, 2) for x in runs_mops],
                     "how": "each run: a fresh handle, the same seeded prefill, W warm-up and K timed steps "
                            "(the paper's 10 runs with a 95% CI, P:1009)"},
            "config": {"workload": args.config, "key_range": R,
                       "rebuild_every": "never" if args.rebuild_every < 0 else (args.rebuild_every or "default: ops since the last rebuild >= 5 x min(capacity, ops up to it) (R29)"),
                       "prefill": pre, "batch_ops": B, "mix_ins_del_con": list(mix), "keys": dist,
                       "semantics": "combining (R26): mutations in input order, any batch" if combine_mode(args)
                       else "S1 snapshot, <=1 mutation per key (R1/R2)",
                       "chunk_entries": N, "p_chunk": args.p_chunk, "contains_team": ex.get("contains_team"),
                       "prefill_path": ("one batch through the bulk path (R34)" if args.prefill == "bulk"
                                        else "per-op Inserts in growing batches + rebuild"),
                       "bulk_timed": args.bulk,
                       "grouped_updates": args.group,
                       "l2": "flushed (256 MiB write) between timed steps",
                       "parallelism": f"range-shard x{world} (strong: global R and batch fixed)" if world > 1 else "1 GPU",
                       "exchange": (("peer windows (CUDA IPC, fused route kernels, device-side counts)"
                                     if args.exchange == "peer" else "NCCL all-to-all") if world > 1 else None)},
            "roofline": ex.get("roofline"),
            "roofline_kernels": ex.get("roofline_kernels"),
            "search_gathers": ex.get("gather"),
            "random_access_roofline": ex.get("rand"),
            "structure": ex.get("structure"),
            "mutations_per_step": ex.get("n_mut"),
            "phase_ms_per_step": ex.get("phases"),
            "chunk_reads_per_contains": ex.get("reads"),
            "chunk_reads_l0_per_contains": ex.get("reads_l0"),
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": launches,
            "library_launches": lib_launches,  # CUB radix-sort kernels (combining mode only)
            "clocks": clk,
            "wall_s_timed_region": round(wall_total, 4),
            "generator_redraws": int(redraws),
            "validate": ex.get("validate"),
        }
        print(json.dumps(line), flush=True)


def run_extras(args, S, g, local_g, inputs, W, steps, PROF, st0, st_t, flush, dev):
    """Run 0's measurements after its timed region: per-kernel phase times (CUDA events
    between the kernels of PROF extra batches), chunk reads per Contains (counting build,
    untimed Contains-only replay), the structure's level sizes, the roofline objects, and
    the validator when asked."""
    world, rank = S.world, S.rank
    N = S.N
    Cb = N * 8
    hbm_peak, peak_kind = load_peaks()
    n_mut = (st_t["mutations"] - st0["mutations"]) / max(steps, 1)
    phases, nbat = {"intake": 0, "contains": 0, "update": 0, "upkeep": 0}, 0
    if PROF:
        local_g.configure(profile_phases=1)
        local_g.phase_times()
        for j in range(PROF):
            flush.zero_()
            g.batch(*inputs[W + steps + j])
        torch.cuda.synchronize()
        phases, nbat = local_g.phase_times()
        local_g.configure(profile_phases=0)
    # chunk reads per Contains: a Contains-only replay of the last batch's keys of this shard
    local_g.configure(count_reads=1)
    c0 = local_g.stats()
    key_last = inputs[-1][1].to(torch.int64)
    if world > 1:  # the keys of this rank's slice that fall in its own shard, rebased
        key_last = key_last[(key_last >= S.lo) & (key_last < S.hi)] - S.lo
    key_last = key_last.to(torch.int32).contiguous()
    if key_last.numel():
        local_g.batch(torch.zeros(key_last.numel(), dtype=torch.uint8, device=dev), key_last)
    torch.cuda.synchronize()
    c1 = local_g.stats()
    local_g.configure(count_reads=0)
    cops = max(1, c1["contains_ops"] - c0["contains_ops"])
    reads = (c1["contains_reads"] - c0["contains_reads"]) / cops
    reads_l0 = (c1["contains_reads_l0"] - c0["contains_reads_l0"]) / cops
    meta = local_g.meta()
    l0_bytes = max(0, meta["counters"][0]) * Cb
    l1_bytes = max(0, meta["counters"][1]) * Cb
    # ops the search kernel of this rank handles per launch (uniform routing: ~B/world)
    n_search = S.B / world
    nb = max(nbat, 1)
    c_ms, u_ms = phases["contains"] / nb, phases["update"] / nb
    i_ms, k_ms = phases["intake"] / nb, phases["upkeep"] / nb

    # Which level of the hierarchy bounds the search kernel: HBM once level 0
    # no longer fits the L2; then the compulsory bytes are the level-0 gathers plus the
    # level-1 gathers that miss (level 1 resident for the fraction L2 / its size).
    resident = l0_bytes <= L2_BYTES
    miss1 = 0.0 if l1_bytes <= L2_BYTES else 1.0 - L2_BYTES / l1_bytes
    upper = max(0.0, reads - reads_l0)
    rand = None
    if not args.no_ubench and rank == 0:
        from paper_conf_ppopp_moscovicicp17_b200.gfsl import ubench
        # the gathers span the config's level-0 footprint (a power of two >= it, 512 MiB ..
        # 16 GiB): TLB reach and DRAM locality depend on it, and a ceiling measured over 16
        # GiB was exceeded by C4-16's chunk gathers over 1.3 GB (round 2)
        ub_bytes = 512 << 20
        while ub_bytes < l0_bytes and ub_bytes < (16 << 30):
            ub_bytes <<= 1
        r_hbm, t_hbm = ubench(Cb, ub_bytes)
        r_l2, t_l2 = ubench(Cb, 32 << 20)
        rand = {"block_bytes": Cb, "R_rand_hbm_GBps": round(r_hbm, 1), "R_rand_l2_GBps": round(r_l2, 1),
                "chase_latency_hbm_ns": round(t_hbm, 1), "chase_latency_l2_ns": round(t_l2, 1),
                "buffer_MiB": ub_bytes >> 20,
                "how": "gfsl_ubench: random aligned chunk-size gathers over a buffer the size of the config's "
                       "level 0 (rounded up to a power of two; 32 MiB for L2), the search kernel's team "
                       "shape, 4/8/16 gathers in flight per team (best kept)"}
    # R37/R38: a traversal entered at level 0 reads no upper level; its index lookup is one
    # 32-B sector of the sorted min keys (4 B per level-0 chunk), compulsory from DRAM for
    # the part of that array the L2 cannot hold beside the 16-MiB directory
    idx_bytes = 4.0 * max(0, meta["counters"][0])
    idx_miss = 0.0 if idx_bytes <= 0 else max(0.0, 1.0 - (L2_BYTES - (18 << 20)) / idx_bytes)
    l0_entry = upper < 0.05
    if resident:
        bound, peak, pk = "l2", (rand["R_rand_l2_GBps"] if rand else None), "measured R_rand_l2 (gfsl_ubench)"
        s_bytes = n_search * reads * Cb
        bytes_note = "every chunk gather (all levels) x C_b: the structure is L2-resident"
    elif l0_entry:
        bound, peak, pk = "hbm", hbm_peak, peak_kind
        s_bytes = n_search * (reads_l0 * Cb + idx_miss * 32)
        bytes_note = ("level-0 gathers x C_b + one 32-B sector of the sorted min keys x its L2 miss "
                      f"fraction {idx_miss:.3f} per op (level 0 entered from the directory, R37/R38; "
                      "SURVEY 8(d)'s level-0 bytes plus the index that replaced level 1)")
    else:
        bound, peak, pk = "hbm", hbm_peak, peak_kind
        s_bytes = n_search * (reads_l0 + upper * miss1) * Cb
        bytes_note = ("(level-0 gathers + upper-level gathers x the level-1 miss fraction "
                      f"{miss1:.3f} = 1 - L2/level-1 bytes) x C_b per op (SURVEY 8(d))")
    u_bytes = n_mut * (Cb + 8 * (N // 2 + 2))
    traffic, tsrc = load_traffic(args.config) if world == 1 else ({}, None)

    def roof(bytes_per_launch, ms, kernel, note):
        if ms <= 0 or bytes_per_launch <= 0 or not peak:
            return None
        ach = bytes_per_launch / (ms / 1e3) / 1e9
        r = {"bound": bound, "achieved": round(ach, 1), "peak": peak, "unit": "GB/s",
             "frac": round(ach / peak, 4), "traffic": None, "peak_kind": pk, "kernel": kernel,
             "algorithmic_bytes_per_launch": int(bytes_per_launch), "algorithmic_bytes": note,
             "launch_ms": round(ms, 4)}
        t = traffic.get(kernel)
        if t is not None:
            r["traffic"] = int(t)
            r["traffic_source"] = f"profiles/{tsrc} (ncu dram__bytes_read.sum + dram__bytes_write.sum, one launch)"
            r["traffic_GBps"] = round(t / (ms / 1e3) / 1e9, 1)
        if rand and bound == "hbm":
            r["frac_of_random_access_peak"] = round(ach / rand["R_rand_hbm_GBps"], 4)
            if kernel == "search":
                # what R_rand bounds: fully random C_b-byte gathers, i.e. the level-0 chunk
                # reads of uniform keys; the index reads (sorted min keys, directory) are
                # 32-B sectors with locality (row-buffer hits), so the kernel's whole DRAM
                # traffic (ncu) can exceed R_rand while its chunk gathers stay below it
                g_rate = n_search * reads_l0 / (ms / 1e3)
                r_rate = rand["R_rand_hbm_GBps"] * 1e9 / Cb
                r["random_gathers"] = {
                    "level0_gathers_per_s": round(g_rate / 1e9, 3), "ceiling_gathers_per_s": round(r_rate / 1e9, 3),
                    "unit": "G gathers/s", "frac": round(g_rate / r_rate, 4),
                    "note": "level-0 chunk gathers of the search kernel vs gfsl_ubench's random C_b-byte gather rate"}
        return r

    roof_c = roof(s_bytes, c_ms, "search", bytes_note)
    roof_u = roof(u_bytes, u_ms, "update", "per mutation: the chunk read under the lock + the entries "
                                           "written, C_b + 8 (N/2 + 2) B")
    roofline = roof_c if c_ms >= u_ms else roof_u
    gather = {"chunk_gathers_per_op": round(reads, 3),
              "gather_GBps": round(n_search * reads * Cb / (c_ms / 1e3) / 1e9, 1) if c_ms > 0 else None,
              "note": "all chunk gathers of the search kernel incl. cache-resident upper levels"}
    rep = None
    if args.validate:
        rep_obj, _, _ = local_g.validate(export=False)
        rep = {"keys": rep_obj.keys, "height": rep_obj.height, "violations": rep_obj.violations}
    return {
        "roofline": roofline, "roofline_kernels": {"search": roof_c, "update": roof_u},
        "gather": gather, "rand": rand, "n_mut": round(n_mut, 1), "reads": round(reads, 3),
        "reads_l0": round(reads_l0, 3), "validate": rep,
        "phases": {"intake": round(i_ms, 4), "search": round(c_ms, 4), "update": round(u_ms, 4),
                   "upkeep_rebuild": round(k_ms, 4)},
        "structure": {"level0_chunks": meta["counters"][0], "level1_chunks": meta["counters"][1],
                      "level0_MB": round(l0_bytes / 2**20, 1), "level1_MB": round(l1_bytes / 2**20, 1),
                      "height": max([l for l in range(1, 32) if meta["counters"][l] > 0], default=0),
                      "l2_MB": L2_BYTES >> 20, "shard": [S.lo, S.hi] if world > 1 else None},
        "contains_team": local_g.cfg.contains_team or (4 if N == 32 else 2),
    }


def run_e2e(args, S, inputs, W, steps, world, dev):
    """End to end through the public API with HOST buffers: every step copies its ops in
    from pinned host memory and its results back, inside the timed region.  N = 1:
    gfsl_batch_host_async (copy-in of step j+1 overlaps step j's kernels), K steps back to
    back on a caller stream, wall clock to the last result in host memory.  N > 1: per
    step the rank's slice is copied in, the collective batch runs, the results are copied
    out (one stream); wall clock, max over ranks."""
    host = [tuple(x.cpu().pin_memory() for x in inp) for inp in inputs]
    # a workload without Inserts reads no value: its caller passes none (values = NULL)
    no_ins = CONFIGS[args.config][4][0] == 0 if args.config in CONFIGS else False
    if no_ins:
        host = [(o, k, None) for o, k, _ in host]
    n_local = host[0][0].numel()
    outs = [torch.empty(n_local, dtype=torch.uint8).pin_memory() for _ in range(steps)]
    reps = 3 if S.R <= 10_000_000 else 1
    t_pipes, zc = [], False
    for _rep in range(reps):
        g, local_g = S.create()
        if world == 1:
            out_w = torch.empty(n_local, dtype=torch.uint8).pin_memory()
            for b in range(W):
                g.batch_host(*host[b], out=out_w)
            side = torch.cuda.Stream()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            with torch.cuda.stream(side):
                for j in range(steps):
                    g.batch_host_async(*host[W + j], out=outs[j])
            torch.cuda.synchronize()
            t_pipes.append(time.perf_counter() - t0)
            zc = local_g.stats().get("zero_copy_batches", 0) > 0
        else:
            bufs = [torch.empty_like(x, device=dev) for x in inputs[0]]
            for b in range(W):
                for d_, h_ in zip(bufs, host[b]):
                    if h_ is not None:
                        d_.copy_(h_, non_blocking=True)
                g.batch(*bufs)
            torch.cuda.synchronize()
            barrier(world)
            t0 = time.perf_counter()
            for j in range(steps):
                for d_, h_ in zip(bufs, host[W + j]):
                    if h_ is not None:
                        d_.copy_(h_, non_blocking=True)
                r = g.batch(*bufs)
                outs[j].copy_(r, non_blocking=True)
            torch.cuda.synchronize()
            t_pipes.append(max_over_ranks(time.perf_counter() - t0, world))
        S.close(g)
    t_pipe = sorted(t_pipes)[len(t_pipes) // 2]
    B = S.B
    # H2D per step: op (1 B) + key (4 B) copied, and the values: copied (4 B per op), or --
    # when the library reads them zero-copy from the pinned buffer -- 4 B per Insert
    n_ins = sum(int((host[W + j][0] == 1).sum()) for j in range(steps)) / max(steps, 1)
    h2d = B * 5 + (0 if no_ins else (int(round(4 * n_ins * world)) if zc else B * 4))
    return {"value": round(B * steps / t_pipe / 1e6, 3), "unit": "Mops/s",
            "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": B,
            "values": ("none (no Inserts in the workload: values = NULL)" if no_ins else
                       "Insert values read zero-copy from the pinned host buffer by the search kernel"
                       if zc else "copied"),
            "how": ("gfsl_batch_host_async on a caller stream, K steps back to back from pinned host "
                    "buffers, wall clock from the first call to the last result in host memory"
                    if world == 1 else
                    "per rank and step: H2D of its slice from pinned memory, the collective batch, "
                    "D2H of its results; wall clock over K steps, max over ranks")
                   + f"; L2 not flushed; median of {reps} run(s)",
            "runs_mops": [round(B * steps / t / 1e6, 1) for t in t_pipes]}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=0, help="timed steps (0 = the config's batch count)")
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--runs", type=int, default=10, help="independent runs (fresh prefill each; P:1009)")
    ap.add_argument("--impl", default="gfsl", choices=["gfsl", "reference"])
    ap.add_argument("--config", default="C5", choices=sorted(CONFIGS) + ["custom"])
    ap.add_argument("--custom", default=None,
                    help="R:prefill:batch:batches:i,d,c:dist:N for --config custom (sweeps, "
                         "tools/sweep_r2.py); dist uniform | zipf | perm")
    ap.add_argument("--team", type=int, default=0)
    ap.add_argument("--chunk", type=int, default=0)
    ap.add_argument("--contains-blocks", type=int, default=0,
                    help="cap on Contains-kernel blocks per SM (0 = occupancy default; sweeps)")
    ap.add_argument("--update-blocks", type=int, default=0,
                    help="cap on update-kernel blocks per SM (0 = occupancy default; sweeps)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--validate", action="store_true")
    ap.add_argument("--no-ubench", action="store_true", help="skip the B6 roofline microbenchmark")
    ap.add_argument("--no-pdl", action="store_true", help="no programmatic dependent launch (ablation)")
    ap.add_argument("--p-chunk", type=float, default=1.0,
                    help="isKeyRaised probability (P:1068-1072, R28) for the timed batches; 1 = the default")
    ap.add_argument("--combine", action="store_true",
                    help="combining mode (R26) for any config (always on for *-raw configs)")
    ap.add_argument("--rebuild-every", type=int, default=0,
                    help="rebuild the upper levels after every k-th batch (R24); "
                         "0 = library default (R29 wear rule), -1 = never (the paper's dynamics only)")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="gloo: exercise the multi-rank path with ranks sharing a GPU (no timing value)")
    ap.add_argument("--exchange", default="peer", choices=["peer", "nccl"],
                    help="N>1 exchange: peer = fused route kernels over CUDA-IPC windows "
                         "(NEXT-3); nccl = torch.distributed all-to-all (baseline)")
    ap.add_argument("--prefill", default="bulk", choices=["bulk", "per-op"],
                    help="prefill through the bulk path (one batch, R34; default) or the paper's "
                         "per-op Insert path in growing batches")
    ap.add_argument("--bulk", default="auto", choices=["auto", "off", "always"],
                    help="the library's bulk path for the timed batches (R34; auto = the library "
                         "default rule); off = the paper's per-op Insert / Delete only")
    ap.add_argument("--group", default="off", choices=["on", "off"],
                    help="chunk-grouped mutations (R40, opt-in): the ops of a batch that target "
                         "one bottom chunk are applied in one lock session; off (default) = one per op")
    ap.add_argument("--l2-window", type=int, default=0,
                    help="L2 access-policy window for the search kernel: 1 = the upper-level pool, "
                         "2 = the level-1 directory (ablations)")
    args = ap.parse_args()
    if args.config == "custom":
        R, pre, B, nb, mix, dist, N = args.custom.split(":")
        CONFIGS["custom"] = (int(R), int(pre), int(B), int(nb), tuple(int(x) for x in mix.split(",")),
                             dist, int(N))
        if dist == "perm":
            PERM_CONFIGS.add("custom")
    if args.warmup < 3:
        args.warmup = 3
    if args.p_chunk <= 0:
        ap.error("--p-chunk must be > 0 (p_chunk_q32 = 0 means p_chunk = 1)")
    args.runs = max(1, args.runs)
    if args.impl == "reference":
        world = int(os.environ.get("WORLD_SIZE", "1"))
        rank = int(os.environ.get("RANK", "0"))
        if args.steps == 0:
            args.steps = CONFIGS[args.config][3]
        run_reference(args, world, rank)
        return
    world, rank, local = dist_setup(args.dist_backend)
    run_gpu(args, world, rank, local)
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
