#!/usr/bin/env python3
"""GFSL batched Contains/Insert/Delete benchmark on B200 (BASELINE.json `metric`).

One JSON line on rank 0.  A "step" is one `gfsl_batch` (classify -> Contains kernel ->
update kernel) over one batch of synthetic ops; `value` is Mops/s over the K timed
steps (all ops of all ranks / the slowest rank's summed step time).  Inputs are
resident in HBM before each timed step; L2 is flushed (a 256 MiB write) between steps.

    python bench.py [--config C2] [--gpus N --steps K --warmup W] [--impl reference]

Configs: C1, C2 (default: R=1M, 10/10/80, the paper's
Table 5.1 workload), C2-100, C2-2020, C2-5050, C3, C3-zipf, C4-32, C4-16, C5.
N>1: weak scaling, each rank owns a key-range shard of the same size as the 1-GPU
config, every rank draws ops over the whole key space and the batch is routed to the
owners with NCCL all-to-all.
"""
from __future__ import annotations

import argparse
import json
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

# name: (R, prefill, batch, n_batches, mix, dist, N)
# N = chunk entries.  The paper's runs use N = 32; on B200 a chunk read costs L1
# data-pipe wavefronts in proportion to its bytes, and N = 16 (128-B chunks, 2-lane teams)
# is faster on every config measured, so it is the default here; the
# C4 pair compares the two, and --chunk 32 runs any config at the paper's size.
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
    # NEXT-4: the paper's other workloads (Fig 5.3 mixes, Fig 5.4b/c single-op runs)
    "M1-1-98": (1_000_000, 500_000, 625_000, 16, (1, 1, 98), "uniform", 16),
    "M5-5-90": (1_000_000, 500_000, 625_000, 16, (5, 5, 90), "uniform", 16),
    "M20-20-60-10M": (10_000_000, 5_000_000, 625_000, 16, (20, 20, 60), "uniform", 16),
    "INS-1M": (1_000_000, 0, 125_000, 8, (100, 0, 0), "uniform", 16),     # R inserts, empty start
    "DEL-1M": (1_000_000, 1_000_000, 125_000, 8, (0, 100, 0), "uniform", 16),  # R deletes, full start
    # NEXT-1: raw Zipf(0.99) -- mutating keys i.i.d. too (no redraws), so hot keys carry
    # long Insert/Delete chains; run in combining mode (R26), exact for any batch
    "C2-zipf-raw": (1_000_000, 500_000, 625_000, 16, (10, 10, 80), "zipf", 16),
    "C3-zipf-raw": (10_000_000, 5_000_000, 6_250_000, 16, (10, 10, 80), "zipf", 16),
}
COMBINE_CONFIGS = {"C2-zipf-raw", "C3-zipf-raw"}


def combine_mode(args) -> bool:
    return args.config in COMBINE_CONFIGS or getattr(args, "combine", False)
L2_FLUSH_BYTES = 256 << 20


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
        return float(d["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


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
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()

    def stop(self):
        if self.ok:
            self._stop.set()
            self.t.join()
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
                "samples": len(self.samples)}


def dist_setup(backend="nccl"):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if backend == "gloo":  # test path: several ranks may share one GPU
        local = local % max(1, torch.cuda.device_count())
    if world > 1:
        import torch.distributed as dist
        torch.cuda.set_device(local)
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    else:
        torch.cuda.set_device(local)
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


# --------------------------------------------------------------------------------------
# reference arm / cpu baseline: the oracle as it stands, on this host's cores

def oracle_sample(cfg_name, steps, warmup, budget_s=20.0, per_step_ops=1_000_000, combine=False):
    """Times Oracle-A on a bounded sample of the config's own batches (1 host thread)."""
    from oracle.oracle_a import OracleMap
    R, pre, B, nb, mix, dist, N = CONFIGS[cfg_name]
    if pre > 4_000_000:
        # bounded sample of a big config: one key-range shard of 2M keys with the same
        # prefill density and the ops that fall into it (DESIGN.md §CPU baseline)
        shard = 2_000_000
        Rs = shard
        pre_s = int(round(pre * shard / R))
        note = f"key-range shard [0,{shard}) of R={R} at the same fill, same mix"
    else:
        Rs, pre_s, note = R, pre, f"the config itself (R={R})"
    o = OracleMap(Rs)
    k = prefill_keys(SEED_BASE, Rs, pre_s)
    o.batch(np.ones(pre_s, np.uint8), k.numpy().astype(np.uint32),
            prefill_values(SEED_BASE, k).numpy().astype(np.uint32))
    Bs = min(B, per_step_ops)
    w = Workload(Rs, Bs, mix=mix, dist=dist, seed=SEED_BASE + 1, dedup=not combine)
    batches = []
    for b in range(warmup + steps):
        op, key, val, _ = w.make_batch(b)
        batches.append((op.numpy(), key.numpy().astype(np.uint32), val.numpy().astype(np.uint32)))
    for b in range(warmup):
        o.batch(*batches[b], combine=combine)
    t_total, n_total, done = 0.0, 0, 0
    for b in range(warmup, warmup + steps):
        t0 = time.perf_counter()
        o.batch(*batches[b], combine=combine)
        t_total += time.perf_counter() - t0
        n_total += Bs
        done += 1
        if t_total > budget_s:
            break
    o.close()
    mops = n_total / t_total / 1e6
    return mops, t_total, done, Bs, note


def run_reference(args, world, rank):
    cfg = args.config
    if rank != 0:
        return
    mops, t, done, Bs, note = oracle_sample(cfg, args.steps, args.warmup, budget_s=60.0,
                                            combine=combine_mode(args))
    line = {
        "impl": "reference", "metric": METRIC, "value": round(mops, 4), "unit": "Mops/s",
        "n_gpus": args.gpus, "steps": done, "warmup": args.warmup,
        "ms_per_step": round(1000 * t / max(done, 1), 3), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": cfg, "batch_ops_sampled": Bs},
        "cpu_baseline": {"value": round(mops, 4), "unit": "Mops/s", "cores": 1,
                         "kind": "oracle",
                         "sample": f"{done} batches of {Bs} ops; {note}; Oracle-A (sequential Pugh skiplist, S1 batches)"},
        "e2e": {"value": round(mops, 4), "unit": "Mops/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# --------------------------------------------------------------------------------------
# GPU arm

def make_inputs(w: Workload, b: int, dev):
    op, key, val, redraws = w.make_batch(b, device=dev)
    return op.contiguous(), key.to(torch.int32).contiguous(), val.to(torch.int32).contiguous(), redraws


def prefill_gpu(g, R, count, dev, chunk=1 << 24, key_lo=0, seed=SEED_BASE):
    """Random-order inserts in insert-only batches that grow with the structure
    (a batch never exceeds ~1/4 of the keys already present, so concurrent inserts spread
    over many chunks instead of queueing on the few chunks of a small structure)."""
    s = 0
    while s < count:
        c = min(chunk, count - s, max(4096, s // 4))
        k = prefill_keys(seed, R, c, start=s, device=dev) + key_lo
        v = prefill_values(seed, k)
        g.batch(torch.ones(c, dtype=torch.uint8, device=dev), k.to(torch.int32),
                v.to(torch.int32))
        s += c
    g.rebuild()  # bulk-load compaction (gfsl_rebuild, R29), as a user would after a load
    torch.cuda.synchronize()


def run_gpu(args, world, rank, local):
    from paper_conf_ppopp_moscovicicp17_b200.gfsl import GFSL
    dev = torch.device("cuda", local)
    R1, pre1, B1, nb, mix, dist, N = CONFIGS[args.config]
    if args.chunk:
        N = args.chunk
    steps = args.steps if args.steps else nb
    W = args.warmup
    hbm_peak, peak_kind = load_peaks()

    # weak scaling: each rank owns a shard of R1 keys and issues B1 ops per step
    R = R1 * world
    if world > 1 and args.exchange == "peer":
        # fused exchange (NEXT-3): route kernels store/load straight through peer windows
        from paper_conf_ppopp_moscovicicp17_b200.router import PeerShardedGFSL
        g = PeerShardedGFSL(R, rank, world, max_slice=B1, capacity=R1, chunk_entries=N,
                            contains_team=args.team)
        lo = g.key_lo
        prefill_gpu(g.local, R1, pre1, dev, key_lo=lo, seed=SEED_BASE + 1000 * rank)
    elif world > 1:
        from paper_conf_ppopp_moscovicicp17_b200.router import ShardedGFSL
        g = ShardedGFSL(R, rank, world, capacity=R1, chunk_entries=N,
                        contains_team=args.team)
        lo = g.key_lo
        prefill_gpu(g.local, R1, pre1, dev, key_lo=lo, seed=SEED_BASE + 1000 * rank)
    else:
        g = GFSL(R, capacity=R, chunk_entries=N, contains_team=args.team,
                 contains_blocks_per_sm=args.contains_blocks, update_blocks_per_sm=args.update_blocks)
        prefill_gpu(g, R, pre1, dev)
    def apply_options(h):
        """The run's library options (identical for the timed and the e2e handles)."""
        h.configure(combine=1 if combine_mode(args) else 0,
                    p_chunk_q32=int(args.p_chunk * 2**32) if args.p_chunk < 1.0 else 0,
                    l2_window=1 if args.l2_window else 0, no_pdl=1 if args.no_pdl else 0,
                    rebuild_every=0xFFFFFFFF if args.rebuild_every < 0 else args.rebuild_every)

    apply_options(g.local if world > 1 else g)
    PROF = 3  # extra batches after the timed region, for the per-kernel breakdown
    w = Workload(R, B1, mix=mix, dist=dist, seed=SEED_BASE + 1 + 7919 * rank,
                 dedup=not combine_mode(args))
    inputs = [make_inputs(w, b, dev) for b in range(W + steps + PROF)]
    redraws = sum(x[3] for x in inputs)
    flush = torch.empty(L2_FLUSH_BYTES, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream()

    for b in range(W):
        g.batch(*inputs[b][:3])
    torch.cuda.synchronize()
    barrier(world)
    local_g = g.local if world > 1 else g
    st0 = local_g.stats()
    mut0 = st0["mutations"]

    starts = [torch.cuda.Event(enable_timing=True) for _ in range(steps)]
    ends = [torch.cuda.Event(enable_timing=True) for _ in range(steps)]
    clocks = ClockSampler(local)
    barrier(world)
    torch.cuda.synchronize()
    clocks.start()
    wall0 = time.perf_counter()
    for j in range(steps):
        flush.zero_()  # L2 flush between timed steps (outside the step's events)
        starts[j].record(stream)
        g.batch(*inputs[W + j][:3])
        ends[j].record(stream)
    torch.cuda.synchronize()
    wall = time.perf_counter() - wall0
    barrier(world)
    clk = clocks.stop()
    step_ms = [s.elapsed_time(e) for s, e in zip(starts, ends)]
    local_ms = sum(step_ms)
    total_ms = max_over_ranks(local_ms, world)
    ops_total = B1 * steps * world
    mops = ops_total / (total_ms / 1e3) / 1e6
    st_t = local_g.stats()
    n_mut = (st_t["mutations"] - mut0) / max(steps, 1)
    # our kernels launched inside the timed region (counted by libgfsl at enqueue), plus the
    # route kernels of the multi-GPU path: NCCL exchange 3 plan + pack + unpack per step;
    # peer exchange 3 plan + counts + push + 2 barriers + pull per step
    route_k = (8 if args.exchange == "peer" else 5) if world > 1 else 0
    launches = int(st_t["kernel_launches"] - st0["kernel_launches"]) + route_k * steps
    lib_launches = int(st_t["library_launches"] - st0["library_launches"])
    # per-kernel breakdown: CUDA events between the kernels of PROF extra batches (events
    # between kernels would defeat the programmatic dependent launch of the timed steps)
    local_g.configure(profile_phases=1)
    local_g.phase_times()
    for j in range(PROF):
        flush.zero_()
        g.batch(*inputs[W + steps + j][:3])
    torch.cuda.synchronize()
    phases, nbat = local_g.phase_times()
    local_g.configure(profile_phases=0)

    # algorithmic bytes: chunk reads per Contains op, counted on a Contains-only replay
    # of the last timed batch's keys (untimed, non-mutating)
    Cb = N * 8
    local_g.configure(count_reads=1)
    st0 = local_g.stats()
    key_last = inputs[W + steps + PROF - 1][1]
    if world > 1:
        key_last = key_last[(key_last >= g.key_lo) & (key_last < g.key_hi)].contiguous()
    local_g.batch(torch.zeros(key_last.numel(), dtype=torch.uint8, device=dev), key_last)
    torch.cuda.synchronize()
    st1 = local_g.stats()
    local_g.configure(count_reads=0)
    cops = max(1, st1["contains_ops"] - st0["contains_ops"])
    reads_per_op = (st1["contains_reads"] - st0["contains_reads"]) / cops
    reads_l0_per_op = (st1["contains_reads_l0"] - st0["contains_reads_l0"]) / cops

    n_search = B1  # the search kernel traverses every valid op of the batch
    c_ms = phases["contains"] / max(nbat, 1)
    u_ms = phases["update"] / max(nbat, 1)
    i_ms = phases["intake"] / max(nbat, 1)
    k_ms = phases["upkeep"] / max(nbat, 1)

    def roof(bytes_per_launch, ms, kernel):
        if ms <= 0 or bytes_per_launch <= 0:
            return None
        ach = bytes_per_launch / (ms / 1e3) / 1e9
        return {"bound": "hbm", "achieved": round(ach, 1), "peak": hbm_peak, "unit": "GB/s",
                "frac": round(ach / hbm_peak, 4), "traffic": None, "peak_kind": peak_kind,
                "kernel": kernel, "algorithmic_bytes_per_launch": int(bytes_per_launch)}
    # search kernel: SURVEY 8(d) -- the compulsory DRAM bytes of a traversal are its
    # bottom-level chunk gathers (upper levels are cache-resident): L0 reads x C_b
    s_bytes = n_search * reads_l0_per_op * Cb
    # update kernel: per mutation one chunk read under the lock + the entries written
    u_bytes = n_mut * (Cb + 8 * (N // 2 + 2))
    roof_c = roof(s_bytes, c_ms, "search")
    roof_u = roof(u_bytes, u_ms, "update")
    traffic, tsrc = load_traffic(args.config) if world == 1 else ({}, None)
    for r, kname in ((roof_c, "search"), (roof_u, "update")):
        if r is not None and traffic.get(kname) is not None:
            r["traffic"] = int(traffic[kname])
            r["traffic_source"] = f"profiles/{tsrc} (ncu, one launch of this config)"
    roofline = roof_c if c_ms >= u_ms else roof_u
    # B6: achievable random-access throughput for this chunk size, measured
    # now on this GPU -- the denominator of the north star's ">= 40%" target
    rand = None
    if not args.no_ubench and rank == 0:
        from paper_conf_ppopp_moscovicicp17_b200.gfsl import ubench
        r_hbm, t_hbm = ubench(Cb, 16 << 30)
        r_l2, t_l2 = ubench(Cb, 32 << 20)
        rand = {"block_bytes": Cb, "R_rand_hbm_GBps": round(r_hbm, 1), "R_rand_l2_GBps": round(r_l2, 1),
                "chase_latency_hbm_ns": round(t_hbm, 1), "chase_latency_l2_ns": round(t_l2, 1)}
        for r in (roof_c, roof_u):
            if r is not None:
                r["frac_of_random_access_peak"] = round(r["achieved"] / r_hbm, 4)
                if r.get("traffic"):
                    ms_k = c_ms if r["kernel"] == "search" else u_ms
                    r["dram_GBps_measured_traffic"] = round(r["traffic"] / (ms_k / 1e3) / 1e9, 1)
                    r["frac_traffic_of_random_access_peak"] = round(r["dram_GBps_measured_traffic"] / r_hbm, 4)
    gather = {"chunk_gathers_per_op": round(reads_per_op, 3),
              "gather_GBps": round(n_search * reads_per_op * Cb / (c_ms / 1e3) / 1e9, 1) if c_ms > 0 else None,
              "note": "all chunk gathers of the search kernel incl. L1/L2-resident upper levels"}

    rep = None
    if args.validate:
        rep_obj, _, _ = local_g.validate(export=False)
        rep = {"keys": rep_obj.keys, "height": rep_obj.height, "violations": rep_obj.violations}
    contains_team = local_g.cfg.contains_team or (4 if N == 32 else 2)

    # end to end through the C ABI with host buffers (fresh handle, same sequence)
    e2e = None
    if not args.no_e2e and world == 1:
        g.close()  # the timed handle is done: free its pool for the e2e handles
        g2 = GFSL(R, capacity=R, chunk_entries=N, contains_team=args.team,
                 contains_blocks_per_sm=args.contains_blocks, update_blocks_per_sm=args.update_blocks)
        prefill_gpu(g2, R, pre1, dev)
        apply_options(g2)
        host = [(x[0].cpu().pin_memory(), x[1].cpu().pin_memory(), x[2].cpu().pin_memory())
                for x in inputs]
        out = torch.empty(B1, dtype=torch.uint8).pin_memory()
        outs = [torch.empty(B1, dtype=torch.uint8).pin_memory() for _ in range(steps)]
        for b in range(W):
            g2.batch_host(*host[b], out=out)
        # (a) synchronous calls, one per step, L2 flushed before each (outside the timer)
        t_sync = 0.0
        for j in range(steps):
            flush.zero_()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            g2.batch_host(*host[W + j], out=out)
            t_sync += time.perf_counter() - t0
        last_sync = out.clone()
        g2.close()  # one extra handle at a time (a 1B-key pool is ~72 GB)
        # (b) the headline: the K steps back to back through gfsl_batch_host_async, as a
        # user streams batches (copy-in of step j+1 overlaps the kernels of step j), from
        # the first call until every step's results are in host memory; wall clock
        # the wall clock of ~K short steps is noisy: small configs run the whole sequence
        # 3 times, each on a freshly prefilled handle, and report the median
        reps = 3 if R <= 10_000_000 else 1
        t_pipes = []
        for _rep in range(reps):
            g3 = GFSL(R, capacity=R, chunk_entries=N, contains_team=args.team,
                      contains_blocks_per_sm=args.contains_blocks, update_blocks_per_sm=args.update_blocks)
            prefill_gpu(g3, R, pre1, dev)
            apply_options(g3)
            out_w = torch.empty(B1, dtype=torch.uint8).pin_memory()
            for b in range(W):
                g3.batch_host(*host[b], out=out_w)
            # issued on a stream of the caller's own (as a serving loop would), not on the
            # legacy default stream: measured 142 vs 246 us/step at C2 (tools/e2e_probe.py)
            side = torch.cuda.Stream()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            with torch.cuda.stream(side):
                for j in range(steps):
                    g3.batch_host_async(*host[W + j], out=outs[j])
            torch.cuda.synchronize()
            t_pipes.append(time.perf_counter() - t0)
            # both handles ran the same sequence: their answers must agree
            assert torch.equal(last_sync, outs[-1]), "e2e paths disagree"
            g3.close()
        t_pipe = sorted(t_pipes)[len(t_pipes) // 2]
        e2e = {"value": round(B1 * steps / t_pipe / 1e6, 3), "unit": "Mops/s",
               "h2d_bytes_per_step": B1 * 9, "d2h_bytes_per_step": B1,
               "how": "gfsl_batch_host_async on a caller stream, K steps back to back from pinned host buffers, wall "
                      "clock from the first call to the last result in host memory; L2 not "
                      "flushed between these steps; median of %d runs of the sequence" % reps,
               "runs_mops": [round(B1 * steps / t / 1e6, 1) for t in t_pipes],
               "sync_per_step": {"value": round(B1 * steps / t_sync / 1e6, 3), "unit": "Mops/s",
                                 "how": "gfsl_batch_host (synchronous) per step, L2 flushed before "
                                        "each step, summed wall time of the calls"}}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cm, ct, cdone, cBs, note = oracle_sample(args.config, min(steps, 16), 1, budget_s=15.0,
                                                combine=combine_mode(args))
        cpu = {"value": round(cm, 4), "unit": "Mops/s", "cores": 1, "kind": "oracle",
               "sample": f"{cdone} batches of {cBs} ops ({ct:.1f} s); {note}"}

    if rank == 0:
        line = {
            "metric": METRIC, "value": round(mops, 3), "unit": "Mops/s", "n_gpus": world,
            "steps": steps, "warmup": W, "ms_per_step": round(total_ms / steps, 4),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": "u32", "data": "synthetic",
            "config": {"workload": args.config, "key_range": R,
                       "rebuild_every": "never" if args.rebuild_every < 0 else (args.rebuild_every or "default: ops since the last rebuild >= 5 x min(capacity, ops up to it) (R29)"), "prefill": pre1 * world,
                       "batch_ops": B1 * world, "mix_ins_del_con": list(mix), "keys": dist,
                       "semantics": "combining (R26): mutations in input order, any batch" if combine_mode(args)
                       else "S1 snapshot, <=1 mutation per key (R1/R2)",
                       "chunk_entries": N, "p_chunk": args.p_chunk, "contains_team": contains_team,
                       "l2": "flushed (256 MiB write) between timed steps",
                       "parallelism": f"range-shard x{world}" if world > 1 else "1 GPU",
                       "exchange": (("peer windows (CUDA IPC, fused route kernels)" if args.exchange == "peer"
                                     else "NCCL all-to-all") if world > 1 else None)},
            "roofline": roofline,
            "roofline_kernels": {"search": roof_c, "update": roof_u},
            "search_gathers": gather,
            "random_access_roofline": rand,
            "mutations_per_step": round(n_mut, 1),
            "phase_ms_per_step": {"intake": round(i_ms, 4), "search": round(c_ms, 4),
                                  "update": round(u_ms, 4), "upkeep_rebuild": round(k_ms, 4)},
            "chunk_reads_per_contains": round(reads_per_op, 3),
            "chunk_reads_l0_per_contains": round(reads_l0_per_op, 3),
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": launches,
            "library_launches": lib_launches,  # CUB radix-sort kernels (combining mode only)
            "clocks": clk,
            "wall_s_timed_region": round(wall, 4),
            "generator_redraws": int(redraws),
            "validate": rep,
        }
        print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=0, help="timed steps (0 = the config's batch count)")
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="gfsl", choices=["gfsl", "reference"])
    ap.add_argument("--config", default="C2", choices=sorted(CONFIGS))
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
                         "0 = library default (4), -1 = never (the paper's dynamics only)")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="gloo: exercise the multi-rank path with ranks sharing a GPU (no timing value)")
    ap.add_argument("--exchange", default="peer", choices=["peer", "nccl"],
                    help="N>1 exchange: peer = fused route kernels over CUDA-IPC windows "
                         "(NEXT-3); nccl = torch.distributed all-to-all (baseline)")
    ap.add_argument("--l2-window", action="store_true",
                    help="pin the upper-level pool in L2 (access-policy window; ablation)")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
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
