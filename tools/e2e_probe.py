"""Where does the e2e (host-buffer) step time go?  C2 by default.
python tools/e2e_probe.py [CFG]
Prints: device-resident back-to-back wall time per step (no L2 flush), the async
host-buffer pipeline's wall time per step, the CPU time per enqueue call, and the time of
the step's copies alone (H2D of op/key/val, D2H of results)."""
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
from paper_conf_ppopp_moscovicicp17_b200.gfsl import GFSL  # noqa: E402
from paper_conf_ppopp_moscovicicp17_b200.workload import Workload  # noqa: E402


def main():
    cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
    R, pre, B, nb, mix, dist, N = bench.CONFIGS[cfg]
    dev = torch.device("cuda", 0)
    steps, W = nb, 3
    w = Workload(R, B, mix=mix, dist=dist, seed=bench.SEED_BASE + 1, dedup=True)
    inputs = [bench.make_inputs(w, b, dev) for b in range(W + steps)]
    host = [(x[0].cpu().pin_memory(), x[1].cpu().pin_memory(), x[2].cpu().pin_memory()) for x in inputs]
    outs = [torch.empty(B, dtype=torch.uint8).pin_memory() for _ in range(W + steps)]

    def fresh():
        g = GFSL(R, capacity=R, chunk_entries=N)
        bench.prefill_gpu(g, R, pre, dev)
        return g

    g = fresh()
    for b in range(W):
        g.batch(*inputs[b][:3])
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for j in range(steps):
        g.batch(*inputs[W + j][:3])
    torch.cuda.synchronize()
    dev_us = (time.perf_counter() - t0) / steps * 1e6
    g.close()

    g = fresh()
    for b in range(W):
        g.batch_host(*host[b], out=outs[b])
    torch.cuda.synchronize()
    cpu = []
    t0 = time.perf_counter()
    for j in range(steps):
        a = time.perf_counter()
        g.batch_host_async(*host[W + j], out=outs[W + j])
        cpu.append(time.perf_counter() - a)
    torch.cuda.synchronize()
    pipe_us = (time.perf_counter() - t0) / steps * 1e6
    g.close()

    # the library's async pipeline again, issued on a side (non-legacy) stream
    g = fresh()
    side = torch.cuda.Stream()
    for b in range(W):
        g.batch_host(*host[b], out=outs[b])
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    with torch.cuda.stream(side):
        for j in range(steps):
            g.batch_host_async(*host[W + j], out=outs[W + j])
    torch.cuda.synchronize()
    print(f"{cfg}: async host pipeline on a side stream {(time.perf_counter() - t0) / steps * 1e6:.1f} us/step")
    g.close()

    # the same pipeline emulated with torch copies on a side stream + the device entry
    # point, with an event timeline (start/end of each H2D and each batch, in us)
    g = fresh()
    cs = torch.cuda.Stream()
    s = torch.cuda.current_stream()
    slots = [[torch.empty_like(x, device=dev) for x in host[0]] for _ in range(2)]
    res = [torch.empty(B, dtype=torch.uint8, device=dev) for _ in range(2)]
    used = [torch.cuda.Event() for _ in range(2)]
    for e in used:
        e.record(s)
    ev = []
    torch.cuda.synchronize()
    base = torch.cuda.Event(enable_timing=True)
    base.record(s)
    t0 = time.perf_counter()
    for j in range(steps):
        b = j & 1
        e = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        cs.wait_event(used[b])
        with torch.cuda.stream(cs):
            e[0].record(cs)
            for x, y in zip(slots[b], host[W + j]):
                x.copy_(y, non_blocking=True)
            e[1].record(cs)
        s.wait_event(e[1])
        e[2].record(s)
        g.batch(slots[b][0], slots[b][1], slots[b][2], out=res[b])
        e[3].record(s)
        used[b].record(s)
        outs[W + j].copy_(res[b], non_blocking=True)
        ev.append(e)
    torch.cuda.synchronize()
    emu_us = (time.perf_counter() - t0) / steps * 1e6
    print(f"{cfg}: emulated pipeline {emu_us:.1f} us/step")
    for j, e in enumerate(ev[:6]):
        print("  step", j, " ".join(f"{base.elapsed_time(x) * 1e3:8.1f}" for x in e))
    g.close()

    d = [torch.empty_like(x, device=dev) for x in host[0]]
    r = torch.empty(B, dtype=torch.uint8, device=dev)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for j in range(steps):
        for x, y in zip(d, host[W + j]):
            x.copy_(y, non_blocking=True)
    torch.cuda.synchronize()
    h2d_us = (time.perf_counter() - t0) / steps * 1e6
    t0 = time.perf_counter()
    for j in range(steps):
        outs[j].copy_(r, non_blocking=True)
    torch.cuda.synchronize()
    d2h_us = (time.perf_counter() - t0) / steps * 1e6
    print(f"{cfg}: device back-to-back {dev_us:.1f} us/step; async host pipeline {pipe_us:.1f} us/step; "
          f"enqueue CPU mean {sum(cpu) / len(cpu) * 1e6:.1f} us max {max(cpu) * 1e6:.1f}; "
          f"H2D alone {h2d_us:.1f} us ({B * 9 / h2d_us / 1e3:.1f} GB/s); D2H alone {d2h_us:.1f} us")


if __name__ == "__main__":
    main()
