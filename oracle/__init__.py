"""The parity oracle — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline`` leg and
``--impl reference``) may import this package. The product path
(``paper_conf_ppopp_nasrebp13_b200``) never imports it and shares no code with it; both
take their inputs from ``graphgen`` (input generation only).

``kruskal`` returns the unique minimum spanning forest of an undirected multigraph under
the order (w, edge id) — Kruskal's "ordered algorithm" of PAPER.md L219 (§5), which reaches
exactly the forest Boruvka's method computes. See ``kruskal.cpp`` for
the steps and DESIGN.md "Readings" for every point where the paper is silent.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "kruskal.cpp")
_LIB = os.path.join(_HERE, "_oracle.so")
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _L():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        p, i64 = ctypes.c_void_p, ctypes.c_int64
        lib.oracle_kruskal.argtypes = [i64, i64, p, p, p, p, p, p]
        lib.oracle_kruskal.restype = i64
        lib.oracle_components.argtypes = [i64, i64, p, p, p]
        lib.oracle_components.restype = i64
        _lib = lib
    return _lib


def _arr(a, dt):
    return np.ascontiguousarray(np.asarray(a), dtype=dt)


def kruskal(n: int, src, dst, w, with_time: bool = False):
    """Minimum spanning forest under (w, id). Returns (ids ascending int32, total uint64 as
    Python int) — plus the single-thread seconds of the algorithm when ``with_time``."""
    src, dst, w = _arr(src, np.int32), _arr(dst, np.int32), _arr(w, np.uint32)
    m = src.shape[0]
    assert dst.shape[0] == m and w.shape[0] == m
    out = np.empty(max(n - 1, 0) or 1, np.int32)
    total = ctypes.c_uint64(0)
    secs = ctypes.c_double(0.0)
    cnt = _L().oracle_kruskal(n, m, src.ctypes.data, dst.ctypes.data, w.ctypes.data,
                              out.ctypes.data, ctypes.addressof(total), ctypes.addressof(secs))
    if cnt < 0:
        raise ValueError("endpoint out of range")
    ids = out[:cnt].copy()
    if with_time:
        return ids, int(total.value), float(secs.value)
    return ids, int(total.value)


def components(n: int, src, dst):
    """label[v] = smallest vertex id of v's connected component; returns (labels, c)."""
    src, dst = _arr(src, np.int32), _arr(dst, np.int32)
    lab = np.empty(max(n, 1), np.int32)
    c = _L().oracle_components(n, src.shape[0], src.ctypes.data, dst.ctypes.data,
                               lab.ctypes.data)
    if c < 0:
        raise ValueError("endpoint out of range")
    return lab[:n].copy(), int(c)
