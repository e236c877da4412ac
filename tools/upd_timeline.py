"""Per-warp timeline of the update kernel (update_multi / update_dual) (needs a library built with
-DGFSL_DEBUG_TIMING in place of libgfsl.so).  python tools/upd_timeline.py [config]"""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from bench import CONFIGS, make_inputs, prefill_gpu
from paper_conf_ppopp_moscovicicp17_b200 import gfsl as G
from paper_conf_ppopp_moscovicicp17_b200.workload import SEED_BASE, Workload

cfg = sys.argv[1] if len(sys.argv) > 1 else "C2"
R, pre, B, nb, mix, dist, N = CONFIGS[cfg]
dev = torch.device("cuda")
g = G.GFSL(R, capacity=R, chunk_entries=N)
prefill_gpu(g, R, pre, dev)
w = Workload(R, B, mix=mix, dist=dist, seed=SEED_BASE + 1)
lib = G.load_library()
n = 148 * 64 * 48 + 64
buf = (ctypes.c_ulonglong * n)()
buf0 = (ctypes.c_ulonglong * n)()
for b in range(4):
    if b == 3:
        torch.empty(256 << 20, dtype=torch.uint8, device=dev).zero_()  # bench.py's L2 flush
        torch.cuda.synchronize()
        lib.gfsl_debug_times(ctypes.c_void_p(g.h), buf0, ctypes.c_uint64(n))
    g.batch(*make_inputs(w, b, dev)[:3])
torch.cuda.synchronize()
lib.gfsl_debug_times(ctypes.c_void_p(g.h), buf, ctypes.c_uint64(n))

a = np.frombuffer(buf, dtype=np.uint64)[:148 * 64 * 48].reshape(-1, 48).astype(np.float64)
a = a[a[:, 0] > 0]
cnt = np.zeros(100, np.int64)
cnt[40:72] = a[:, 16:48].sum(0).astype(np.int64)
t0 = a[:, 0].min()
st, en, it = (a[:, 0] - t0) / 1e3, (a[:, 1] - t0) / 1e3, a[:, 2]
oc = a[:, 3:7].sum(0)
ser = a[:, 7]
print(f"{cfg}: warps={len(a)} iterations={it.sum():.0f} kernel span={en.max():.1f} us")
print("outcomes done/defer/cont/full:", oc.astype(int).tolist())
print("start pct 0/50/90/100:", np.percentile(st, [0, 50, 90, 100]).round(1))
fo = a[:, 8]
if (fo > 0).any():
    print("first-op pct 0/50/90/100:", np.percentile((fo[fo > 0] - t0) / 1e3, [0, 50, 90, 100]).round(1),
          f"(warps with an op: {(fo > 0).sum()})")
    busy = en[fo > 0]
    print("end of warps with ops pct 50/90/99/100:", np.percentile(busy, [50, 90, 99, 100]).round(1))
print("end   pct 0/50/90/99/100:", np.percentile(en, [0, 50, 90, 99, 100]).round(1))
print("iterations/warp pct 0/50/100:", np.percentile(it, [0, 50, 100]))
dur = (en - st) * 1e3 * 1.965
print(f"serial-section share {ser.sum() / dur.sum():.2f}; cycles per iteration excl. serial {(dur.sum() - ser.sum()) / it.sum():.0f};"
      f" serial cycles per cont/full op {ser.sum() / max(oc[2] + oc[3], 1):.0f}")
for name, i in (("insert_locked: split_insert(0)", 40), ("  .. split_chunk(0)", 46), ("  .. update_down_ptrs(0)", 48),
                ("  raise_levels", 42), ("  unlocks", 44), ("delete_upper: exact checks", 50), ("  upper levels", 52),
                ("  bottom remove", 54), ("full ops", 58), ("cont delete", 60), ("cont insert", 62)):
    c = cnt[i + 1]
    print(f"  {name:34s} n={c:7d}  cycles/call {cnt[i] / max(c, 1):8.0f}")
print("  merges:", cnt[56])

ph = cnt[[64, 69, 65, 66, 67, 68]].astype(np.float64)
nit = max(it.sum(), 1)
print("per-iteration phase cycles (lane 0 of each warp): staging wait %.0f, take/stage records %.0f, CAS %.0f, read %.0f, decide+write %.0f, fence+release %.0f" % tuple(ph / nit))
print("  of which: take a staged record %.0f, queue-item wait %.0f, stage_pair %.0f" % (cnt[70] / nit, (int(cnt[71]) & 0xFFFFFFFF) / nit, (int(cnt[71]) >> 32) / nit))
