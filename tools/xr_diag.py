"""Diagnostic of the loopback exchange: host time of each call, flags and error words."""
import ctypes
import time

import numpy as np
import torch

from paper_conf_ppopp_moscovicicp17_b200 import gfsl as G

dev = torch.device("cuda")
torch.cuda.init()
W = 2
xs = [G.XRoute(r, W, 1000, 64, timeout_ms=3000) for r in range(W)]
for r in range(W):
    for p in range(W):
        if p != r:
            xs[r].attach_local(p, xs[p])
streams = [torch.cuda.Stream() for _ in range(W)]
print("stream flags/ptrs", [s.cuda_stream for s in streams], flush=True)
side = torch.cuda.Stream()


def window(x):
    b, n = ctypes.c_void_p(), ctypes.c_uint64()
    x.lib.gfsl_xr_window(x.h, ctypes.byref(b), ctypes.byref(n))
    return b.value


def dump(tag):
    out = []
    for x in xs:
        buf = torch.empty(2048, dtype=torch.uint8, pin_memory=True)
        G.load_library()
        cudart = ctypes.CDLL("libcudart.so")
        out.append(buf)
    print(tag, flush=True)


op = torch.zeros(10, dtype=torch.uint8, device=dev)
key = torch.arange(10, dtype=torch.int32, device=dev)
torch.cuda.synchronize()
for r in range(W):
    t = time.perf_counter()
    xs[r].send(op, key, None, stream=streams[r])
    print(f"send {r}: {1e3*(time.perf_counter()-t):.2f} ms", flush=True)
for r in range(W):
    t = time.perf_counter()
    try:
        print("recv", r, xs[r].recv(), flush=True)
    except Exception as e:
        print("recv", r, "failed", e, flush=True)
    print(f"recv {r}: {1e3*(time.perf_counter()-t):.2f} ms", flush=True)
