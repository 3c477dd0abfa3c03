"""Seeded synthetic graph generators (input generation only; no MST arithmetic).

Shared by the oracle (``oracle/``) and the CUDA path — the only module the two share
(see DESIGN.md §"Input recipe"). Every array is a pure function of the config and seed:

* ``h(seed, i) = mix64(seed*0xD1B54A32D192ED03 + i*0x9E3779B97F4A7C15)``, splitmix64 finaliser.
* per-config field seeds ``16k + f + 65536*s`` with f = 0 (u), 1 (v), 2 (w), 3 (perm),
  4 (rmat), 5 (diag); k = config number (1..5), s = user seed index (0 for the bench).

The configs are BASELINE.json's five workloads; their shapes follow the
paper's MST inputs (Fig. 11). The fast path is C (``gen.c``, OpenMP
over index ranges only); ``*_np`` functions restate the same recipes in numpy for tests.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gen.c")
_LIB = os.path.join(_HERE, "_graphgen.so")
_lib = None

M1 = np.uint64(0xD1B54A32D192ED03)
M2 = np.uint64(0x9E3779B97F4A7C15)


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O3", "-fopenmp", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def _L():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        i64, u64, u32, p = ctypes.c_int64, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_void_p
        lib.gg_hash_fill.argtypes = [u64, i64, i64, p]
        lib.gg_grid_m.argtypes = [i64, i64]; lib.gg_grid_m.restype = i64
        lib.gg_grid.argtypes = [i64, i64, u64, u32, u64, p, p, p]
        lib.gg_road_m.argtypes = [i64, i64, u64, i64]; lib.gg_road_m.restype = i64
        lib.gg_road.argtypes = [i64, i64, u64, u64, i64, p, p, p]
        lib.gg_uniform.argtypes = [i64, i64, u64, u64, u64, u32, u64, p, p, p]
        lib.gg_rmat_perm.argtypes = [i64, u64, p]
        lib.gg_rmat.argtypes = [i64, i64, u64, u64, i64, i64, i64, u32, u64, p, p, p, p]
        _lib = lib
    return _lib


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data


def _alloc(m: int):
    return (np.empty(m, np.int32), np.empty(m, np.int32), np.empty(m, np.uint32))


@dataclass
class Graph:
    """An undirected edge list: edge id i = position (SURVEY.md §8 notation)."""
    n: int
    src: np.ndarray  # int32[m]
    dst: np.ndarray  # int32[m]
    w: np.ndarray    # uint32[m]
    name: str = ""

    @property
    def m(self) -> int:
        return int(self.src.shape[0])


def field_seed(k: int, f: int, s: int = 0) -> int:
    return 16 * k + f + 65536 * s


# --------------------------------------------------------------------------- C fast path
def hash_fill(seed: int, start: int, count: int) -> np.ndarray:
    out = np.empty(count, np.uint64)
    _L().gg_hash_fill(seed, start, count, _ptr(out))
    return out


def grid(W: int, H: int, seed_w: int, wlo: int = 1, wmod: int = 1000, name="grid") -> Graph:
    m = int(_L().gg_grid_m(W, H))
    s, d, w = _alloc(m)
    _L().gg_grid(W, H, seed_w, wlo, wmod, _ptr(s), _ptr(d), _ptr(w))
    return Graph(W * H, s, d, w, name)


def road(W: int, H: int, seed_w: int, seed_diag: int, thresh: int = 414, name="road") -> Graph:
    m = int(_L().gg_road_m(W, H, seed_diag, thresh))
    s, d, w = _alloc(m)
    _L().gg_road(W, H, seed_w, seed_diag, thresh, _ptr(s), _ptr(d), _ptr(w))
    return Graph(W * H, s, d, w, name)


def uniform(n: int, m: int, seed_u: int, seed_v: int, seed_w: int, wlo: int = 1,
            wmod: int = 1000, name="uniform") -> Graph:
    s, d, w = _alloc(m)
    if m:
        _L().gg_uniform(n, m, seed_u, seed_v, seed_w, wlo, wmod, _ptr(s), _ptr(d), _ptr(w))
    return Graph(n, s, d, w, name)


def rmat_perm(n: int, seed_perm: int) -> np.ndarray:
    perm = np.empty(n, np.int32)
    _L().gg_rmat_perm(n, seed_perm, _ptr(perm))
    return perm


def rmat(scale: int, m: int, seed_rmat: int, seed_perm: int | None, seed_w: int,
         a: int = 57, b: int = 19, c: int = 19, wlo: int = 1, wmod: int = 1000,
         name="rmat") -> Graph:
    n = 1 << scale
    perm = rmat_perm(n, seed_perm) if seed_perm is not None else None
    s, d, w = _alloc(m)
    _L().gg_rmat(scale, m, seed_rmat, seed_w, a, b, c, wlo, wmod,
                 _ptr(perm) if perm is not None else None, _ptr(s), _ptr(d), _ptr(w))
    return Graph(n, s, d, w, name)


# --------------------------------------------------------------------------- the 5 configs
CONFIGS = {
    1: "grid64",
    2: "uniform",
    3: "road",
    4: "rmat22",
    5: "dense",
}
NAME_TO_K = {v: k for k, v in CONFIGS.items()}


def config(k, s: int = 0, scale_down: int = 0) -> Graph:
    """BASELINE.json config k (1..5 or name), seed index s.

    ``scale_down`` shrinks the size parameters by 2**scale_down (same recipe; used only for
    parity tests that must finish in seconds on the oracle)."""
    if isinstance(k, str):
        k = NAME_TO_K[k]
    sd = scale_down
    fs = lambda f: field_seed(k, f, s)  # noqa: E731
    if k == 1:
        return grid(64, 64, fs(2), name="grid64")
    if k == 2:
        n = (1 << 22) >> sd
        return uniform(n, 4 * n, fs(0), fs(1), fs(2), name="uniform")
    if k == 3:
        W = 4890 >> (sd // 2) if sd else 4890
        return road(W, W, fs(2), fs(5), 414, name="road")
    if k == 4:
        scale = 22 - sd
        return rmat(scale, 16 << scale, fs(4), fs(3), fs(2), name="rmat22")
    if k == 5:
        n = 65536 >> (sd // 2) if sd else 65536
        m = 2048 * n >> (sd - sd // 2) if sd else 2048 * n
        return uniform(n, m, fs(0), fs(1), fs(2), name="dense")
    raise ValueError(k)


# --------------------------------------------------------------------------- numpy restatement
def mix64_np(x: np.ndarray) -> np.ndarray:
    x = x.astype(np.uint64, copy=True)
    with np.errstate(over="ignore"):
        x ^= x >> np.uint64(30)
        x *= np.uint64(0xBF58476D1CE4E5B9)
        x ^= x >> np.uint64(27)
        x *= np.uint64(0x94D049BB133111EB)
        x ^= x >> np.uint64(31)
    return x


def h_np(seed: int, i) -> np.ndarray:
    i = np.asarray(i, dtype=np.uint64)
    with np.errstate(over="ignore"):
        return mix64_np(np.uint64(seed) * M1 + i * M2)


def grid_np(W, H, seed_w, wlo=1, wmod=1000) -> Graph:
    src, dst = [], []
    for y in range(H):
        for x in range(W):
            v = y * W + x
            if x < W - 1:
                src.append(v); dst.append(v + 1)
            if y < H - 1:
                src.append(v); dst.append(v + W)
    m = len(src)
    w = (wlo + h_np(seed_w, np.arange(m)) % np.uint64(wmod)).astype(np.uint32)
    return Graph(W * H, np.array(src, np.int32), np.array(dst, np.int32), w)


def road_np(W, H, seed_w, seed_diag, thresh=414) -> Graph:
    g = grid_np(W, H, 0)
    mg = g.m
    src, dst = list(g.src), list(g.dst)
    base = [1000] * mg
    for y in range(H - 1):
        for x in range(W - 1):
            v = y * W + x
            if int(h_np(seed_diag, v) % np.uint64(1000)) < thresh:
                src.append(v); dst.append(v + W + 1); base.append(1414)
    m = len(src)
    hw = h_np(seed_w, np.arange(m)) % np.uint64(501)
    w = (np.array(base, np.uint64) * (np.uint64(750) + hw) // np.uint64(1000)).astype(np.uint32)
    return Graph(W * H, np.array(src, np.int32), np.array(dst, np.int32), w)


def uniform_np(n, m, seed_u, seed_v, seed_w, wlo=1, wmod=1000) -> Graph:
    i = np.arange(m)
    s = (h_np(seed_u, i) % np.uint64(n)).astype(np.int32)
    d = (h_np(seed_v, i) % np.uint64(n)).astype(np.int32)
    w = (wlo + h_np(seed_w, i) % np.uint64(wmod)).astype(np.uint32)
    return Graph(n, s, d, w)


def rmat_np(scale, m, seed_rmat, seed_perm, seed_w, a=57, b=19, c=19, wlo=1, wmod=1000):
    n = 1 << scale
    u = np.zeros(m, np.uint64)
    v = np.zeros(m, np.uint64)
    i = np.arange(m, dtype=np.uint64)
    for lev in range(scale):
        q = h_np(seed_rmat, np.uint64(32) * i + np.uint64(lev)) % np.uint64(100)
        bu = (q >= a + b).astype(np.uint64)
        bv = (((q >= a) & (q < a + b)) | (q >= a + b + c)).astype(np.uint64)
        u = (u << np.uint64(1)) | bu
        v = (v << np.uint64(1)) | bv
    if seed_perm is not None:
        perm = np.argsort(h_np(seed_perm, np.arange(n)), kind="stable").astype(np.int32)
        s, d = perm[u.astype(np.int64)], perm[v.astype(np.int64)]
    else:
        s, d = u.astype(np.int32), v.astype(np.int32)
    w = (wlo + h_np(seed_w, i) % np.uint64(wmod)).astype(np.uint32)
    return Graph(n, s.astype(np.int32), d.astype(np.int32), w)
