"""Thin Python binding of libgfsl (include/gfsl.h) -- argument marshalling only.

Every step of a batch runs in the sm_100a kernels of ``csrc/``; this module passes
device pointers, sizes and the current CUDA stream through the C ABI.  There is no CPU
fallback: if ``libgfsl.so`` is missing or no CUDA device is present, constructing a
``GFSL`` raises.

Tensors: op types ``uint8``; keys/values 32-bit (``int32`` or ``uint32`` tensors, read as
uint32 bit patterns); results ``uint8`` (0 false, 1 true, 0xFF invalid).
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# GFSL_LIB: an alternative build of the same library (tools/ experiments only)
LIB_PATH = os.environ.get("GFSL_LIB") or os.path.join(_HERE, "libgfsl.so")

GFSL_OK, GFSL_EINVAL, GFSL_ENOMEM, GFSL_EPOOL, GFSL_ECUDA, GFSL_ECORRUPT, GFSL_ETIMEOUT = range(7)
CONTAINS, INSERT, DELETE = 0, 1, 2
RES_FALSE, RES_TRUE, RES_INVALID = 0, 1, 0xFF
REBUILD_DEFAULT, REBUILD_NEVER = 0, 0xFFFFFFFF  # rebuild_every: library default period / never
CHECK_SNAPSHOT, CHECK_CROSS = 1, 2
BULK_AUTO, BULK_OFF, BULK_ALWAYS = 0, 1, 2
GROUP_OFF, GROUP_ON = 0, 1
STATUS_NAMES = ["OK", "EINVAL", "ENOMEM", "EPOOL", "ECUDA", "ECORRUPT", "ETIMEOUT"]
XR_HANDLE_BYTES = 64


class gfsl_config(ctypes.Structure):
    _fields_ = [("chunk_entries", ctypes.c_uint32), ("contains_team", ctypes.c_uint32),
                ("contains_blocks_per_sm", ctypes.c_uint32),
                ("update_blocks_per_sm", ctypes.c_uint32),
                ("serial_updates", ctypes.c_uint32), ("count_reads", ctypes.c_uint32),
                ("profile_phases", ctypes.c_uint32), ("l2_window", ctypes.c_uint32),
                ("no_pdl", ctypes.c_uint32),
                ("rebuild_every", ctypes.c_uint32), ("combine", ctypes.c_uint32),
                ("p_chunk_q32", ctypes.c_uint32), ("bulk", ctypes.c_uint32),
                ("group", ctypes.c_uint32)]


class gfsl_report(ctypes.Structure):
    _fields_ = [("keys", ctypes.c_uint64), ("height", ctypes.c_uint32),
                ("chunk_entries", ctypes.c_uint32), ("chunks", ctypes.c_uint64 * 32),
                ("zombies", ctypes.c_uint64 * 32), ("level_keys", ctypes.c_uint64 * 32),
                ("counters", ctypes.c_int64 * 32), ("pool_used", ctypes.c_uint64 * 2),
                ("pool_cap", ctypes.c_uint64 * 2), ("violations", ctypes.c_uint32),
                ("first_violation", ctypes.c_uint32), ("restarts", ctypes.c_uint64),
                ("underfull", ctypes.c_uint64), ("reserved", ctypes.c_uint64 * 3)]


class gfsl_stats(ctypes.Structure):
    _fields_ = [("batches", ctypes.c_uint64), ("ops", ctypes.c_uint64),
                ("restarts", ctypes.c_uint64), ("splits", ctypes.c_uint64),
                ("merges", ctypes.c_uint64), ("zombie_unlinks", ctypes.c_uint64),
                ("lock_retries", ctypes.c_uint64), ("contains_reads", ctypes.c_uint64),
                ("contains_reads_l0", ctypes.c_uint64), ("contains_ops", ctypes.c_uint64),
                ("mutations", ctypes.c_uint64), ("kernel_launches", ctypes.c_uint64),
                ("library_launches", ctypes.c_uint64), ("grouped", ctypes.c_uint64),
                ("zero_copy_batches", ctypes.c_uint64)]


class gfsl_meta(ctypes.Structure):
    _fields_ = [("head", ctypes.c_uint32 * 32), ("counters", ctypes.c_int32 * 32),
                ("used_bottom", ctypes.c_uint32), ("used_upper", ctypes.c_uint32),
                ("cap_bottom", ctypes.c_uint32), ("cap_upper", ctypes.c_uint32),
                ("chunk_entries", ctypes.c_uint32), ("reserved", ctypes.c_uint32 * 3)]


# Every symbol include/gfsl.h declares (checked by tests/test_abi.py).
EXPORTS = [
    "gfsl_create", "gfsl_create_ex", "gfsl_destroy", "gfsl_batch", "gfsl_batch_dn", "gfsl_batch_host",
    "gfsl_batch_host_async",
    "gfsl_validate", "gfsl_check", "gfsl_export", "gfsl_last_error", "gfsl_get_stats", "gfsl_dump", "gfsl_load",
    "gfsl_route_plan", "gfsl_route_pack", "gfsl_route_unpack", "gfsl_phase_times",
    "gfsl_configure", "gfsl_ubench", "gfsl_rebuild",
    "gfsl_xr_create", "gfsl_xr_destroy", "gfsl_xr_export", "gfsl_xr_attach",
    "gfsl_xr_attach_local", "gfsl_xr_send", "gfsl_xr_push", "gfsl_xr_recv", "gfsl_xr_local",
    "gfsl_xr_done",
    "gfsl_xr_finish", "gfsl_xr_batch",
    "gfsl_xr_status", "gfsl_xr_window",
]

_lib = None


def load_library(path: str = LIB_PATH):
    """Load libgfsl.so and declare the C signatures.  Raises if it is missing."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise RuntimeError(
            f"{path} is missing: build it with `python -m paper_conf_ppopp_moscovicicp17_b200.build`"
            " (there is no CPU fallback)")
    lib = ctypes.CDLL(path)
    if os.environ.get("GFSL_LIB"):
        # an experimental build of another revision (tools/ A/B runs): declare only the
        # entry points it has
        class _Tolerant:
            def __init__(self, l):
                object.__setattr__(self, "_l", l)

            def __getattr__(self, name):
                try:
                    return getattr(self._l, name)
                except AttributeError:
                    return type("Missing", (), {})()

        real = lib
        lib = _Tolerant(real)
    vp, u64, u32, i32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int
    lib.gfsl_create.restype = vp
    lib.gfsl_create.argtypes = [u64, u64]
    lib.gfsl_create_ex.restype = vp
    lib.gfsl_create_ex.argtypes = [u64, u64, ctypes.POINTER(gfsl_config)]
    lib.gfsl_destroy.restype = None
    lib.gfsl_destroy.argtypes = [vp]
    lib.gfsl_batch.restype = i32
    lib.gfsl_batch.argtypes = [vp, vp, vp, vp, vp, u64, vp]
    lib.gfsl_batch_dn.restype = i32
    lib.gfsl_batch_dn.argtypes = [vp, vp, vp, vp, vp, u64, vp, u64, vp]
    lib.gfsl_batch_host.restype = i32
    lib.gfsl_batch_host.argtypes = [vp, vp, vp, vp, vp, u64, vp]
    lib.gfsl_batch_host_async.restype = i32
    lib.gfsl_batch_host_async.argtypes = [vp, vp, vp, vp, vp, u64, vp]
    lib.gfsl_validate.restype = i32
    lib.gfsl_validate.argtypes = [vp, ctypes.POINTER(gfsl_report), vp, vp, u64,
                                  ctypes.POINTER(u64)]
    lib.gfsl_check.restype = i32
    lib.gfsl_check.argtypes = [vp, ctypes.POINTER(gfsl_report), u32]
    lib.gfsl_export.restype = i32
    lib.gfsl_export.argtypes = [vp, vp, vp, u64, ctypes.POINTER(u64)]
    lib.gfsl_last_error.restype = ctypes.c_char_p
    lib.gfsl_last_error.argtypes = []
    lib.gfsl_get_stats.restype = i32
    lib.gfsl_get_stats.argtypes = [vp, ctypes.POINTER(gfsl_stats)]
    lib.gfsl_dump.restype = i32
    lib.gfsl_dump.argtypes = [vp, ctypes.POINTER(gfsl_meta), vp, u64]
    lib.gfsl_load.restype = i32
    lib.gfsl_load.argtypes = [vp, ctypes.POINTER(gfsl_meta), vp, u64]
    lib.gfsl_ubench.restype = i32
    lib.gfsl_ubench.argtypes = [u32, u64, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_double)]
    lib.gfsl_rebuild.restype = i32
    lib.gfsl_rebuild.argtypes = [vp, vp]
    lib.gfsl_configure.restype = i32
    lib.gfsl_configure.argtypes = [vp, ctypes.POINTER(gfsl_config)]
    lib.gfsl_phase_times.restype = i32
    lib.gfsl_phase_times.argtypes = [vp, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(u64)]
    lib.gfsl_route_plan.restype = i32
    lib.gfsl_route_plan.argtypes = [vp, vp, u64, u64, u32, vp, vp, vp]
    lib.gfsl_route_pack.restype = i32
    lib.gfsl_route_pack.argtypes = [vp, vp, vp, vp, u64, u64, u32, vp, vp, vp, vp]
    lib.gfsl_route_unpack.restype = i32
    lib.gfsl_route_unpack.argtypes = [vp, vp, u64, vp, vp]
    lib.gfsl_xr_create.restype = vp
    lib.gfsl_xr_create.argtypes = [u32, u32, u64, u64, u64]
    lib.gfsl_xr_destroy.restype = None
    lib.gfsl_xr_destroy.argtypes = [vp]
    lib.gfsl_xr_export.restype = i32
    lib.gfsl_xr_export.argtypes = [vp, vp]
    lib.gfsl_xr_attach.restype = i32
    lib.gfsl_xr_attach.argtypes = [vp, u32, vp]
    lib.gfsl_xr_attach_local.restype = i32
    lib.gfsl_xr_attach_local.argtypes = [vp, u32, vp]
    lib.gfsl_xr_send.restype = i32
    lib.gfsl_xr_send.argtypes = [vp, vp, vp, vp, u64, vp]
    lib.gfsl_xr_push.restype = i32
    lib.gfsl_xr_push.argtypes = [vp, vp]
    lib.gfsl_xr_recv.restype = i32
    lib.gfsl_xr_recv.argtypes = [vp, ctypes.POINTER(vp), ctypes.POINTER(vp), ctypes.POINTER(vp),
                                 ctypes.POINTER(vp), ctypes.POINTER(u64), ctypes.POINTER(vp), vp]
    lib.gfsl_xr_local.restype = i32
    lib.gfsl_xr_local.argtypes = [vp, vp, u64, vp]
    lib.gfsl_xr_done.restype = i32
    lib.gfsl_xr_done.argtypes = [vp, vp]
    lib.gfsl_xr_finish.restype = i32
    lib.gfsl_xr_finish.argtypes = [vp, vp, vp]
    lib.gfsl_xr_batch.restype = i32
    lib.gfsl_xr_batch.argtypes = [vp, vp, vp, vp, vp, vp, u64, vp]
    lib.gfsl_xr_status.restype = i32
    lib.gfsl_xr_status.argtypes = [vp]
    lib.gfsl_xr_window.restype = i32
    lib.gfsl_xr_window.argtypes = [vp, ctypes.POINTER(vp), ctypes.POINTER(u64)]
    _lib = lib._l if hasattr(lib, "_l") else lib
    return _lib


class GFSLError(RuntimeError):
    def __init__(self, status: int, what: str):
        self.status = status
        name = STATUS_NAMES[status] if 0 <= status < len(STATUS_NAMES) else str(status)
        super().__init__(f"{what}: GFSL_{name}: {load_library().gfsl_last_error().decode()}")


def _check(status: int, what: str):
    if status != GFSL_OK:
        raise GFSLError(status, what)


def _ptr(t) -> int | None:
    return None if t is None else t.data_ptr()


def _stream(stream) -> int | None:
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return stream.cuda_stream


@dataclass
class Report:
    keys: int
    height: int
    chunks: list
    zombies: list
    level_keys: list
    counters: list
    pool_used: tuple
    pool_cap: tuple
    violations: int
    first_violation: int
    restarts: int
    underfull: int


class GFSL:
    """One GFSL map on the current CUDA device (C handle ``gfsl_t``)."""

    def __init__(self, key_range: int, capacity: int = 0, chunk_entries: int = 16,
                 contains_team: int = 0, serial_updates: bool = False,
                 contains_blocks_per_sm: int = 0, update_blocks_per_sm: int = 0,
                 count_reads: bool = False, profile_phases: bool = False,
                 rebuild_every: int = 0, combine: bool = False, p_chunk: float = 1.0,
                 bulk: int = 0, group: int = 0):
        import torch
        if not torch.cuda.is_available():
            raise RuntimeError("GFSL needs a CUDA device (there is no CPU fallback)")
        self.lib = load_library()
        cfg = gfsl_config(chunk_entries, contains_team, contains_blocks_per_sm,
                          update_blocks_per_sm, 1 if serial_updates else 0,
                          1 if count_reads else 0, 1 if profile_phases else 0, 0, 0,
                          rebuild_every, 1 if combine else 0,
                          0 if p_chunk >= 1.0 else max(1, int(p_chunk * 2**32)), bulk, group)
        if p_chunk <= 0:
            raise ValueError("p_chunk must be > 0 (p_chunk_q32 = 0 means p_chunk = 1)")
        self.key_range = int(key_range)
        self.chunk_entries = int(chunk_entries)
        self.cfg = cfg
        self.h = self.lib.gfsl_create_ex(self.key_range, int(capacity), ctypes.byref(cfg))
        if not self.h:
            raise RuntimeError("gfsl_create failed: " + self.lib.gfsl_last_error().decode())

    def close(self):
        if getattr(self, "h", None):
            self.lib.gfsl_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # ---- batches -------------------------------------------------------------------
    def batch(self, op, key, val=None, out=None, stream=None):
        """Asynchronous batch on device tensors; returns the uint8 result tensor."""
        import torch
        n = op.numel()
        assert op.dtype == torch.uint8 and op.is_cuda and op.is_contiguous()
        assert key.numel() == n and key.element_size() == 4 and key.is_cuda and key.is_contiguous()
        if val is not None:
            assert val.numel() == n and val.element_size() == 4 and val.is_cuda and val.is_contiguous()
        if out is None:
            out = torch.empty(n, dtype=torch.uint8, device=op.device)
        _check(self.lib.gfsl_batch(self.h, _ptr(op), _ptr(key), _ptr(val), _ptr(out), n,
                                   _stream(stream)), "gfsl_batch")
        return out

    def rebuild(self, stream=None):
        """Rebuild the upper levels now (gfsl_rebuild; R24/R29), e.g. after a bulk load."""
        _check(self.lib.gfsl_rebuild(self.h, _stream(stream)), "gfsl_rebuild")

    def batch_ptr(self, op_ptr: int, key_ptr: int, val_ptr: int | None, res_ptr: int, n: int,
                  stream=None):
        """Asynchronous batch on raw device pointers (e.g. an exchange window's arrays)."""
        _check(self.lib.gfsl_batch(self.h, op_ptr, key_ptr, val_ptr, res_ptr, n, _stream(stream)),
               "gfsl_batch")

    def batch_dn(self, op_ptr: int, key_ptr: int, val_ptr: int | None, res_ptr: int, n_max: int,
                 n_dev_ptr: int, n_hint: int = 0, stream=None):
        """Asynchronous batch whose op count lives in device memory (gfsl_batch_dn)."""
        _check(self.lib.gfsl_batch_dn(self.h, op_ptr, key_ptr, val_ptr, res_ptr, n_max, n_dev_ptr,
                                      n_hint, _stream(stream)), "gfsl_batch_dn")

    def batch_host(self, op, key, val=None, out=None, stream=None):
        """Synchronous batch on HOST tensors (the end-to-end entry point)."""
        import torch
        n = op.numel()
        assert not op.is_cuda and op.dtype == torch.uint8 and op.is_contiguous()
        assert not key.is_cuda and key.element_size() == 4 and key.is_contiguous()
        if out is None:
            out = torch.empty(n, dtype=torch.uint8, pin_memory=op.is_pinned())
        _check(self.lib.gfsl_batch_host(self.h, _ptr(op), _ptr(key), _ptr(val), _ptr(out), n,
                                        _stream(stream)), "gfsl_batch_host")
        return out

    def batch_host_async(self, op, key, val=None, out=None, stream=None):
        """Asynchronous batch on (pinned) HOST tensors: `out` holds the results once
        `stream` (default: the current one) has completed this batch."""
        import torch
        n = op.numel()
        assert not op.is_cuda and op.dtype == torch.uint8 and op.is_contiguous()
        assert not key.is_cuda and key.element_size() == 4 and key.is_contiguous()
        if out is None:
            out = torch.empty(n, dtype=torch.uint8, pin_memory=op.is_pinned())
        _check(self.lib.gfsl_batch_host_async(self.h, _ptr(op), _ptr(key), _ptr(val), _ptr(out),
                                              n, _stream(stream)), "gfsl_batch_host_async")
        return out

    # ---- inspection ----------------------------------------------------------------
    def validate(self, export: bool = True, raise_on_violation: bool = True):
        rep = gfsl_report()
        cnt = ctypes.c_uint64()
        st = self.lib.gfsl_validate(self.h, ctypes.byref(rep), None, None, 0, ctypes.byref(cnt))
        if st not in (GFSL_OK, GFSL_ECORRUPT):
            _check(st, "gfsl_validate")
        keys = vals = None
        if export and st == GFSL_OK:
            n = cnt.value
            keys = np.empty(n, dtype=np.uint32)
            vals = np.empty(n, dtype=np.uint32)
            st = self.lib.gfsl_validate(self.h, None, keys.ctypes.data, vals.ctypes.data, n, None)
        report = Report(rep.keys, rep.height, list(rep.chunks), list(rep.zombies),
                        list(rep.level_keys), list(rep.counters), tuple(rep.pool_used),
                        tuple(rep.pool_cap), rep.violations, rep.first_violation, rep.restarts,
                        rep.underfull)
        if st == GFSL_ECORRUPT and raise_on_violation:
            raise GFSLError(st, f"gfsl_validate (violations=0x{rep.violations:x})")
        return report, keys, vals

    def check(self, snapshot: bool = False, cross: bool = False, raise_on_violation: bool = True):
        """Device-side structural check (gfsl_check, B4): a Report; chunks[1] / zombies[1]
        count all upper levels together; .stale = level-1 stale separators (R33);
        .cross_checked = whether V6 / V11 were checked against the last snapshot."""
        rep = gfsl_report()
        flags = (CHECK_SNAPSHOT if snapshot else 0) | (CHECK_CROSS if cross else 0)
        st = self.lib.gfsl_check(self.h, ctypes.byref(rep), flags)
        if st not in (GFSL_OK, GFSL_ECORRUPT):
            _check(st, "gfsl_check")
        report = Report(rep.keys, rep.height, list(rep.chunks), list(rep.zombies),
                        list(rep.level_keys), list(rep.counters), tuple(rep.pool_used),
                        tuple(rep.pool_cap), rep.violations, rep.first_violation, rep.restarts,
                        rep.underfull)
        report.stale = rep.reserved[0]
        report.cross_checked = bool(rep.reserved[1])
        if st == GFSL_ECORRUPT and raise_on_violation:
            raise GFSLError(st, f"gfsl_check (violations=0x{rep.violations:x})")
        return report

    def export(self):
        """(keys, values): the live pairs in key order as int32 DEVICE tensors holding
        uint32 bit patterns (gfsl_export; sorted on the device)."""
        import torch
        cnt = ctypes.c_uint64()
        _check(self.lib.gfsl_export(self.h, None, None, 0, ctypes.byref(cnt)), "gfsl_export")
        n = cnt.value
        dev = torch.device("cuda", torch.cuda.current_device())
        keys = torch.empty(n, dtype=torch.int32, device=dev)
        vals = torch.empty(n, dtype=torch.int32, device=dev)
        _check(self.lib.gfsl_export(self.h, _ptr(keys), _ptr(vals), n, ctypes.byref(cnt)), "gfsl_export")
        return keys, vals

    def stats(self) -> dict:
        s = gfsl_stats()
        _check(self.lib.gfsl_get_stats(self.h, ctypes.byref(s)), "gfsl_get_stats")
        return {f: getattr(s, f) for f, _ in gfsl_stats._fields_ if f != "reserved"}

    def configure(self, **kw):
        """Change run-time options (contains_team, serial_updates, count_reads, ...)."""
        for k, v in kw.items():
            setattr(self.cfg, k, int(v))
        _check(self.lib.gfsl_configure(self.h, ctypes.byref(self.cfg)), "gfsl_configure")

    def phase_times(self):
        """(ms dict of intake/contains/update/total since the last call, batches)."""
        ms = (ctypes.c_double * 5)()
        nb = ctypes.c_uint64()
        _check(self.lib.gfsl_phase_times(self.h, ms, ctypes.byref(nb)), "gfsl_phase_times")
        return dict(intake=ms[0], contains=ms[1], update=ms[2], upkeep=ms[3], total=ms[4]), nb.value

    def meta(self):
        """Head array, level counters and pool use (gfsl_dump without the pool; synchronises)."""
        m = gfsl_meta()
        _check(self.lib.gfsl_dump(self.h, ctypes.byref(m), None, 0), "gfsl_dump")
        return dict(head=list(m.head), counters=list(m.counters), used_bottom=m.used_bottom,
                    used_upper=m.used_upper, cap_bottom=m.cap_bottom, cap_upper=m.cap_upper,
                    chunk_entries=m.chunk_entries)

    def dump(self):
        """(meta dict, entries uint64 array of shape [chunks, N]) -- test-only."""
        m = gfsl_meta()
        _check(self.lib.gfsl_dump(self.h, ctypes.byref(m), None, 0), "gfsl_dump")
        total = (m.cap_bottom + m.cap_upper) * m.chunk_entries
        ent = np.empty(total, dtype=np.uint64)
        _check(self.lib.gfsl_dump(self.h, ctypes.byref(m), ent.ctypes.data, total), "gfsl_dump")
        meta = dict(head=list(m.head), counters=list(m.counters), used_bottom=m.used_bottom,
                    used_upper=m.used_upper, cap_bottom=m.cap_bottom, cap_upper=m.cap_upper,
                    chunk_entries=m.chunk_entries)
        return meta, ent.reshape(-1, m.chunk_entries)

    def load(self, meta: dict, entries: np.ndarray):
        m = gfsl_meta()
        for i, v in enumerate(meta["head"]):
            m.head[i] = v
        for i, v in enumerate(meta["counters"]):
            m.counters[i] = v
        m.used_bottom, m.used_upper = meta["used_bottom"], meta["used_upper"]
        m.cap_bottom, m.cap_upper = meta["cap_bottom"], meta["cap_upper"]
        m.chunk_entries = meta["chunk_entries"]
        ent = np.ascontiguousarray(entries, dtype=np.uint64).reshape(-1)
        _check(self.lib.gfsl_load(self.h, ctypes.byref(m), ent.ctypes.data, ent.size), "gfsl_load")


def read_device_u32(dev_ptr: int) -> int:
    """One uint32 from device memory, synchronously (tests / diagnostics only)."""
    global _cudart
    if _cudart is None:
        import torch  # noqa: F401  (loads the CUDA runtime into the process)
        _cudart = ctypes.CDLL("libcudart.so.12")
        _cudart.cudaMemcpy.restype = ctypes.c_int
        _cudart.cudaMemcpy.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int]
    buf = ctypes.c_uint32()
    st = _cudart.cudaMemcpy(ctypes.addressof(buf), dev_ptr, 4, 2)  # cudaMemcpyDeviceToHost
    if st != 0:
        raise RuntimeError(f"cudaMemcpy failed ({st})")
    return buf.value


_cudart = None


# ---- multi-GPU routing primitives (B5) ------------------------------------------------
def route_plan(op, key, key_range: int, world: int, stream=None):
    """Returns (counts int64[world] on device, perm int32[n] on device)."""
    import torch
    lib = load_library()
    n = op.numel()
    counts = torch.empty(world, dtype=torch.int64, device=op.device)
    perm = torch.empty(n, dtype=torch.int32, device=op.device)
    _check(lib.gfsl_route_plan(_ptr(op), _ptr(key), n, key_range, world, _ptr(counts),
                               _ptr(perm), _stream(stream)), "gfsl_route_plan")
    return counts, perm


def route_pack(perm, op, key, val, key_range: int, world: int, stream=None):
    """Ops in routed order; keys rebased to their destination shard's local key space."""
    import torch
    lib = load_library()
    n = op.numel()
    so = torch.empty_like(op)
    sk = torch.empty_like(key)
    sv = torch.empty(n, dtype=key.dtype, device=op.device)
    _check(lib.gfsl_route_pack(_ptr(perm), _ptr(op), _ptr(key), _ptr(val), n, key_range, world,
                               _ptr(so), _ptr(sk), _ptr(sv), _stream(stream)), "gfsl_route_pack")
    return so, sk, sv


def route_unpack(perm, recv_res, out, stream=None):
    lib = load_library()
    _check(lib.gfsl_route_unpack(_ptr(perm), _ptr(recv_res), recv_res.numel(), _ptr(out),
                                 _stream(stream)), "gfsl_route_unpack")
    return out


def ubench(block_bytes: int = 256, buffer_bytes: int = 16 << 30):
    """B6 roofline denominators: (R_rand GB/s, dependent-gather latency ns)."""
    lib = load_library()
    g, c = ctypes.c_double(), ctypes.c_double()
    _check(lib.gfsl_ubench(block_bytes, buffer_bytes, ctypes.byref(g), ctypes.byref(c)), "gfsl_ubench")
    return g.value, c.value


# ---- fused exchange over peer memory (gfsl_xr_*) ----------------
class XRoute:
    """One rank's exchange window (C handle ``gfsl_xr_t``) on the current CUDA device."""

    def __init__(self, rank: int, world: int, key_range: int, max_slice: int,
                 timeout_ms: int = 0):
        self.lib = load_library()
        self.rank, self.world, self.max_slice = int(rank), int(world), int(max_slice)
        self.h = self.lib.gfsl_xr_create(self.rank, self.world, int(key_range),
                                         self.max_slice, int(timeout_ms))
        if not self.h:
            raise RuntimeError("gfsl_xr_create failed: " + self.lib.gfsl_last_error().decode())

    def close(self):
        if getattr(self, "h", None):
            self.lib.gfsl_xr_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def export(self) -> bytes:
        buf = (ctypes.c_char * XR_HANDLE_BYTES)()
        _check(self.lib.gfsl_xr_export(self.h, buf), "gfsl_xr_export")
        return bytes(buf)

    def attach(self, peer: int, handle: bytes):
        buf = (ctypes.c_char * XR_HANDLE_BYTES).from_buffer_copy(handle)
        _check(self.lib.gfsl_xr_attach(self.h, peer, buf), "gfsl_xr_attach")

    def attach_local(self, peer: int, other: "XRoute"):
        _check(self.lib.gfsl_xr_attach_local(self.h, peer, other.h), "gfsl_xr_attach_local")

    def send(self, op, key, val=None, stream=None):
        _check(self.lib.gfsl_xr_send(self.h, _ptr(op), _ptr(key), _ptr(val), op.numel(),
                                     _stream(stream)), "gfsl_xr_send")

    def push(self, stream=None):
        _check(self.lib.gfsl_xr_push(self.h, _stream(stream)), "gfsl_xr_push")

    def recv(self, stream=None):
        """(n_cap, n_dev_ptr, op_ptr, key_ptr, val_ptr, res_ptr): the window's receive
        arrays, their capacity and the device word holding the received count."""
        o, k, v, r, nd = (ctypes.c_void_p() for _ in range(5))
        m = ctypes.c_uint64()
        _check(self.lib.gfsl_xr_recv(self.h, ctypes.byref(o), ctypes.byref(k), ctypes.byref(v),
                                     ctypes.byref(r), ctypes.byref(m), ctypes.byref(nd),
                                     _stream(stream)), "gfsl_xr_recv")
        return m.value, nd.value, o.value, k.value, v.value, r.value

    def local(self, local: "GFSL", n_hint: int = 0, stream=None) -> int:
        """The local shard's batch on the window (gfsl_xr_local); returns the status
        (GFSL_OK, or the local error after the received ops were answered INVALID)."""
        return self.lib.gfsl_xr_local(self.h, local.h, n_hint, _stream(stream))

    def done(self, stream=None):
        _check(self.lib.gfsl_xr_done(self.h, _stream(stream)), "gfsl_xr_done")

    def finish(self, out, stream=None):
        _check(self.lib.gfsl_xr_finish(self.h, _ptr(out), _stream(stream)), "gfsl_xr_finish")
        return out

    def batch(self, local: "GFSL", op, key, val=None, out=None, stream=None):
        import torch
        if out is None:
            out = torch.empty(op.numel(), dtype=torch.uint8, device=op.device)
        _check(self.lib.gfsl_xr_batch(self.h, local.h, _ptr(op), _ptr(key), _ptr(val), _ptr(out),
                                      op.numel(), _stream(stream)), "gfsl_xr_batch")
        return out

    def status(self) -> int:
        return self.lib.gfsl_xr_status(self.h)
