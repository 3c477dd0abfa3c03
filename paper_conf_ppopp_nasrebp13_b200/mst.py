"""Thin ctypes binding of libmst.so (include/mst.h) — argument marshalling only.

Every step of the method runs in the library's CUDA kernels; this module only converts
torch tensors / numpy arrays to pointers and statuses to exceptions. torch is used for
device memory and streams. There is no CPU fallback: if the library cannot be loaded or
no CUDA device is present, calls raise.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from . import _build

MST_OK, MST_EINVAL, MST_ENOMEM, MST_ECUDA, MST_ENCCL, MST_EINTERNAL, MST_ENOTSUP = range(7)
STATUS_NAMES = {0: "MST_OK", 1: "MST_EINVAL", 2: "MST_ENOMEM", 3: "MST_ECUDA", 4: "MST_ENCCL",
                5: "MST_EINTERNAL", 6: "MST_ENOTSUP"}
MAX_ROUNDS = 64
K_INIT, K_MIN0, K_HOOK, K_JUMP, K_FILTER, K_OUTPUT, K_COMM, K_DENSE, K_LIGHT, K_COMPOSE, \
    K_SMALL, K_DEDUP, K_COUNT = range(13)
KERNEL_NAMES = ["init", "min0", "hook", "jump", "filter", "output", "comm", "dense", "light",
                "compose", "small", "dedup"]
# launch sub-kinds per kind (include/mst.h MST_SUB_*)
SUB_NAMES = {K_MIN0: ["min_all", "extract", "min_light", "singletons"],
             K_FILTER: ["sparse", "light", "switch", "transition", "member"],
             K_DENSE: ["dense_round", "dense_best", "tail"],
             K_COMPOSE: ["compose", "sample"]}

# every symbol include/mst.h declares
DEBUG_EXPORTS = ["mst_debug_filter_pass", "mst_shard_ranges",
                 "mst_create_dist_hostx"]  # include/mst_debug.h
EXPORTS = ["mst_create", "mst_create_host", "mst_run", "mst_run_host", "mst_solve_host",
           "mst_destroy", "mst_last_error", "mst_get_stats", "mst_set_profiling",
           "mst_get_unique_id", "mst_create_dist", "mst_create_sim", "mst_version",
           "mst_set_option", "mst_get_launch_times"]
MST_OPT_DENSE, MST_OPT_KEEP_EDGES, MST_OPT_DEVICE_TAIL, MST_OPT_COMPACT_TAU = 1, 2, 3, 4
MST_OPT_LIGHT_FIRST = 5
MST_OPT_UNION_FIND = 6
MST_OPT_SMALL = 7
MST_OPT_DEDUP = 8


class mst_stats(ctypes.Structure):
    _fields_ = [
        ("n", ctypes.c_int64), ("m", ctypes.c_int64), ("arcs0", ctypes.c_int64),
        ("rounds", ctypes.c_int32), ("nranks", ctypes.c_int32), ("rank", ctypes.c_int32),
        ("local_arcs0", ctypes.c_int64),
        ("n_r", ctypes.c_int64 * MAX_ROUNDS), ("a_r", ctypes.c_int64 * MAX_ROUNDS),
        ("num_edges", ctypes.c_int64), ("total_weight", ctypes.c_uint64),
        ("build_ms", ctypes.c_double), ("profiling", ctypes.c_int32),
        ("kernel_ms", ctypes.c_double * K_COUNT), ("kernel_launches", ctypes.c_int64 * K_COUNT),
        ("round_filter_ms", ctypes.c_double * MAX_ROUNDS),
        ("gpu_launches", ctypes.c_int64),
        ("dense_round", ctypes.c_int32),
        ("compacted_mask", ctypes.c_int64),
        ("survival_permille", ctypes.c_int32 * MAX_ROUNDS),
        ("hub_row", ctypes.c_int32),
        ("light_switch_round", ctypes.c_int32),
        ("light_t", ctypes.c_uint32),
        ("member_ends", ctypes.c_int64 * MAX_ROUNDS),
        ("dedup_in", ctypes.c_int64 * MAX_ROUNDS),
        ("layout", ctypes.c_int32),
        ("member_round", ctypes.c_int32 * MAX_ROUNDS),
    ]


# include/mst_debug.h: int (*)(uint64_t* host_buf, int64_t count, void* ctx)
ALLREDUCE_MIN_FN = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.POINTER(ctypes.c_uint64), ctypes.c_int64,
                                    ctypes.c_void_p)


class mst_launch_time(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("sub", ctypes.c_int32), ("round", ctypes.c_int32),
                ("shard", ctypes.c_int32), ("ms", ctypes.c_double)]


class MSTError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status


_lib = None


def lib_path() -> str:
    return _build.LIB


def load(build_if_missing: bool = True):
    """Load libmst.so (building it with nvcc first if it is missing or stale)."""
    global _lib
    if _lib is not None:
        return _lib
    if build_if_missing and _build.needs_build():
        _build.build()
    if not os.path.exists(_build.LIB):
        raise ImportError(f"libmst.so not found at {_build.LIB}; run __graft_entry__.build()")
    L = ctypes.CDLL(_build.LIB)
    p, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int
    pp = ctypes.POINTER(ctypes.c_void_p)
    L.mst_create.argtypes = [i64, i64, p, p, p, pp]
    L.mst_create_host.argtypes = [i64, i64, p, p, p, pp]
    L.mst_create_sim.argtypes = [i64, i64, p, p, p, i32, pp]
    L.mst_create_dist.argtypes = [i64, i64, p, p, p, p, i32, i32, pp]
    L.mst_run.argtypes = [p, p, p, p, p]
    L.mst_run_host.argtypes = [p, p, p, p, p]
    L.mst_solve_host.argtypes = [i64, i64, p, p, p, p, p, p]
    L.mst_destroy.argtypes = [p]
    L.mst_destroy.restype = None
    L.mst_last_error.restype = ctypes.c_char_p
    L.mst_get_stats.argtypes = [p, ctypes.POINTER(mst_stats)]
    L.mst_set_profiling.argtypes = [p, i32]
    L.mst_get_launch_times.argtypes = [p, ctypes.POINTER(mst_launch_time), i64,
                                       ctypes.POINTER(ctypes.c_int64)]
    L.mst_set_option.argtypes = [p, i32, i64]
    L.mst_get_unique_id.argtypes = [p]
    L.mst_version.restype = ctypes.c_char_p
    L.mst_debug_filter_pass.argtypes = [p, p, i32, i64, i32, ctypes.POINTER(ctypes.c_double),
                                        ctypes.POINTER(ctypes.c_int64)]
    L.mst_debug_filter_pass.restype = ctypes.c_int
    L.mst_shard_ranges.argtypes = [p, i64, i32, p, p]
    L.mst_shard_ranges.restype = ctypes.c_int
    L.mst_create_dist_hostx.argtypes = [i64, i64, p, p, p, i32, i32, ALLREDUCE_MIN_FN, p, pp]
    L.mst_create_dist_hostx.restype = ctypes.c_int
    for name in EXPORTS:
        if name not in ("mst_destroy", "mst_last_error", "mst_version"):
            getattr(L, name).restype = ctypes.c_int
    _lib = L
    return L


def _check(st):
    if st != MST_OK:
        raise MSTError(st, load().mst_last_error().decode(errors="replace"))


def _dptr(t):
    """device pointer of a torch CUDA tensor (None for empty)."""
    return t.data_ptr() if t is not None and t.numel() > 0 else None


def _stream_ptr(stream):
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return stream.cuda_stream


def mst_version() -> str:
    return load().mst_version().decode()


def mst_get_unique_id() -> bytes:
    buf = (ctypes.c_uint8 * 128)()
    _check(load().mst_get_unique_id(buf))
    return bytes(buf)


class MSTGraph:
    """Owns one library handle. Construct with device tensors (mst_create), host arrays
    (``host=True``: mst_create_host), ``nshards`` (mst_create_sim), ``dist=(id, rank,
    nranks)`` (mst_create_dist) or ``hostx=(rank, nranks, fn)`` (mst_create_dist_hostx: the
    exchange is ``fn(words)``, which must replace the numpy uint64 array ``words`` in place by
    its element-wise minimum over all ranks)."""

    def __init__(self, n, src, dst, w, *, host=False, nshards=1, dist=None, hostx=None):
        L = load()
        self.n = int(n)
        self.m = int(src.shape[0])
        h = ctypes.c_void_p()
        if host:
            src = np.ascontiguousarray(src, np.int32)
            dst = np.ascontiguousarray(dst, np.int32)
            w = np.ascontiguousarray(w, np.uint32)
            _check(L.mst_create_host(self.n, self.m, src.ctypes.data or None,
                                     dst.ctypes.data or None, w.ctypes.data or None,
                                     ctypes.byref(h)))
        else:
            import torch
            for t, dt in ((src, torch.int32), (dst, torch.int32), (w, torch.int32)):
                if not (t.is_cuda and t.is_contiguous()):
                    raise ValueError("src/dst/w must be contiguous CUDA tensors")
                if t.dtype not in (dt, torch.uint32) or t.element_size() != 4:
                    raise ValueError("src/dst must be int32 and w 32-bit")
            if hostx is not None:
                rank, nranks, fn = hostx

                def _cb(buf, count, _ctx, fn=fn):
                    try:
                        fn(np.ctypeslib.as_array(buf, shape=(int(count),)))
                        return 0
                    except Exception:  # noqa: BLE001 -> MST_ENCCL from mst_run
                        import traceback
                        traceback.print_exc()
                        return 1
                self._xcb = ALLREDUCE_MIN_FN(_cb)  # kept alive with the handle
                _check(L.mst_create_dist_hostx(self.n, self.m, _dptr(src), _dptr(dst), _dptr(w),
                                               int(rank), int(nranks), self._xcb, None,
                                               ctypes.byref(h)))
            elif dist is not None:
                uid, rank, nranks = dist
                idbuf = (ctypes.c_uint8 * 128).from_buffer_copy(uid)
                _check(L.mst_create_dist(self.n, self.m, _dptr(src), _dptr(dst), _dptr(w),
                                         idbuf, int(rank), int(nranks), ctypes.byref(h)))
            elif nshards > 1:
                _check(L.mst_create_sim(self.n, self.m, _dptr(src), _dptr(dst), _dptr(w),
                                        int(nshards), ctypes.byref(h)))
            else:
                _check(L.mst_create(self.n, self.m, _dptr(src), _dptr(dst), _dptr(w),
                                    ctypes.byref(h)))
        self._h = h

    def run(self, out_ids=None, stream=None):
        """mst_run: returns (ids tensor[:count] on device, count, total weight)."""
        import torch
        if out_ids is None:
            out_ids = torch.empty(max(self.n - 1, 1), dtype=torch.int32, device="cuda")
        cnt, tot = ctypes.c_int64(0), ctypes.c_uint64(0)
        _check(load().mst_run(self._h, _stream_ptr(stream), _dptr(out_ids), ctypes.byref(cnt),
                              ctypes.byref(tot)))
        return out_ids[: cnt.value], int(cnt.value), int(tot.value)

    def run_host(self, out=None, stream=None):
        """mst_run_host: ids land in a host (numpy) buffer."""
        if out is None:
            out = np.empty(max(self.n - 1, 1), np.int32)
        cnt, tot = ctypes.c_int64(0), ctypes.c_uint64(0)
        _check(load().mst_run_host(self._h, _stream_ptr(stream), out.ctypes.data,
                                   ctypes.byref(cnt), ctypes.byref(tot)))
        return out[: cnt.value], int(cnt.value), int(tot.value)

    def set_option(self, option: int, value: int):
        """mst_set_option: MST_OPT_DENSE / _KEEP_EDGES / _DEVICE_TAIL / _COMPACT_TAU / _LIGHT_FIRST
        (include/mst.h)."""
        _check(load().mst_set_option(self._h, int(option), int(value)))

    def set_profiling(self, on: bool):
        _check(load().mst_set_profiling(self._h, 1 if on else 0))

    def stats(self) -> dict:
        s = mst_stats()
        _check(load().mst_get_stats(self._h, ctypes.byref(s)))
        R = s.rounds
        return {
            "n": s.n, "m": s.m, "arcs0": s.arcs0, "rounds": R, "nranks": s.nranks,
            "rank": s.rank, "local_arcs0": s.local_arcs0,
            "n_r": list(s.n_r[:R]), "a_r": list(s.a_r[:R]),
            "num_edges": s.num_edges, "total_weight": s.total_weight, "build_ms": s.build_ms,
            "profiling": bool(s.profiling),
            "kernel_ms": {KERNEL_NAMES[i]: s.kernel_ms[i] for i in range(K_COUNT)},
            "kernel_launches": {KERNEL_NAMES[i]: s.kernel_launches[i] for i in range(K_COUNT)},
            "round_filter_ms": list(s.round_filter_ms[:R]),
            "gpu_launches": s.gpu_launches,
            "dense_round": s.dense_round,
            "compacted": [bool((s.compacted_mask >> r) & 1) for r in range(R)],
            "survival_permille": list(s.survival_permille[:R]),
            "hub_row": bool(s.hub_row),
            "light_switch_round": s.light_switch_round,
            "light_t": s.light_t,
            "member_ends": list(s.member_ends[:R]),
            "dedup_in": list(s.dedup_in[:R]),
            "layout": ["caller", "hub-first", "bfs"][s.layout] if 0 <= s.layout < 3 else s.layout,
            "member_round": list(s.member_round[:R]),
        }

    def launch_times(self) -> list:
        """Per-launch event times of the last profiled run: dicts {kind, sub, round, shard, ms}
        (kind/sub as names, include/mst.h MST_K_* / MST_SUB_*)."""
        cnt = ctypes.c_int64(0)
        _check(load().mst_get_launch_times(self._h, None, 0, ctypes.byref(cnt)))
        buf = (mst_launch_time * max(cnt.value, 1))()
        _check(load().mst_get_launch_times(self._h, buf, cnt.value, ctypes.byref(cnt)))
        out = []
        for x in buf[: cnt.value]:
            subs = SUB_NAMES.get(x.kind)
            out.append({"kind": KERNEL_NAMES[x.kind],
                        "sub": subs[x.sub] if subs and x.sub < len(subs) else str(x.sub),
                        "round": x.round, "shard": x.shard, "ms": x.ms})
        return out

    def debug_filter_pass(self, map_kind=0, group=1, iters=5, stream=None):
        """Times the A8 kernel alone on the round-0 arcs (include/mst_debug.h)."""
        ms, surv = ctypes.c_double(0), ctypes.c_int64(0)
        _check(load().mst_debug_filter_pass(self._h, _stream_ptr(stream), int(map_kind),
                                            int(group), int(iters), ctypes.byref(ms),
                                            ctypes.byref(surv)))
        return ms.value, surv.value

    def close(self):
        if getattr(self, "_h", None):
            load().mst_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


def mst_solve_host(n, src, dst, w, out=None):
    """One end-to-end call from host arrays to host results (create + run + destroy)."""
    src = np.ascontiguousarray(src, np.int32)
    dst = np.ascontiguousarray(dst, np.int32)
    w = np.ascontiguousarray(w, np.uint32)
    if out is None:
        out = np.empty(max(int(n) - 1, 1), np.int32)
    cnt, tot = ctypes.c_int64(0), ctypes.c_uint64(0)
    _check(load().mst_solve_host(int(n), src.shape[0], src.ctypes.data or None,
                                 dst.ctypes.data or None, w.ctypes.data or None,
                                 out.ctypes.data, ctypes.byref(cnt), ctypes.byref(tot)))
    return out[: cnt.value], int(cnt.value), int(tot.value)


def mst_shard_ranges(row_offsets, nranks):
    """The edge partition used by mst_create_dist (host only): arc windows (lo, hi) per rank."""
    row = np.ascontiguousarray(row_offsets, np.uint32)
    lo = np.empty(nranks, np.int64)
    hi = np.empty(nranks, np.int64)
    _check(load().mst_shard_ranges(row.ctypes.data, row.shape[0] - 1, int(nranks),
                                   lo.ctypes.data, hi.ctypes.data))
    return lo, hi


def minimum_spanning_forest(n, src, dst, w, stream=None):
    """Convenience: device tensors in, (ids, count, total) out; one handle per call."""
    with MSTGraph(n, src, dst, w) as g:
        return g.run(stream=stream)
