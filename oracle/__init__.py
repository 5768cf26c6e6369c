"""CPU oracle (TEST INFRASTRUCTURE ONLY).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` / ``--impl
reference`` legs may import this package.  The product path never imports it; it shares no code
with ``paper_conf_ppopp_menglts19_b200``.

Thin ctypes wrapper over ``oracle/oracle.c`` (plain C, see its header for the paper citations of
every function and for the one place OpenMP is used: the per-vertex loops of PR / Delta-PR,
bit-identical to one thread).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_lib = None

P = ctypes.c_void_p


def build() -> str:
    src = os.path.join(_HERE, "oracle.c")
    if not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        # -O2 plain C; no -ffast-math (keeps fp64 order as written); OpenMP only across the
        # vertices of orc_pr / orc_dpr (bit-identical to one thread, see oracle.c's header)
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-o", _SO, src, "-lm"])
    return _SO


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        i64, i32, dbl = ctypes.c_int64, ctypes.c_int32, ctypes.c_double
        lib.orc_bfs.argtypes = [i64, P, P, i32, P]
        lib.orc_bfs_features.argtypes = [i64, P, P, i32, P, P, P, P, i64]
        lib.orc_bfs_features.restype = i64
        lib.orc_sssp.argtypes = [i64, P, P, P, i32, P]
        lib.orc_cc.argtypes = [i64, P, P, P]
        lib.orc_pr.argtypes = [i64, P, P, P, dbl, i32, P]
        lib.orc_dpr.argtypes = [i64, P, P, P, dbl, dbl, i32, P, P]
        lib.orc_bc.argtypes = [i64, P, P, P, i32, P]
        lib.orc_attrs.argtypes = [i64, P, P]
        lib.orc_ratios.argtypes = [i64, i64, i64, i64, i64, i64, P]
        lib.orc_ratios.restype = None
        lib.orc_set_threads.argtypes = [ctypes.c_int]
        lib.orc_set_threads.restype = None
        lib.orc_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def _p(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data)


def _arrs(g):
    off = np.ascontiguousarray(g.off, dtype=np.int64)
    col = np.ascontiguousarray(g.col, dtype=np.int32)
    if col.size == 0:
        col = np.zeros(1, np.int32)
    return off, col


class OracleError(RuntimeError):
    pass


def _check(rc, what):
    if rc == -3:
        raise OverflowError(f"oracle {what}: overflow")
    if rc != 0:
        raise OracleError(f"oracle {what} failed rc={rc}")


def bfs(g, src: int) -> np.ndarray:
    off, col = _arrs(g)
    depth = np.empty(g.n, np.int32)
    _check(_load().orc_bfs(g.n, _p(off), _p(col), src, _p(depth)), "bfs")
    return depth


def bfs_features(g, src: int, max_levels: int = 1 << 20):
    """Per-level (Va, Ea, Via, Eia) arrays of level-synchronous BFS from src."""
    off, col = _arrs(g)
    bufs = [np.zeros(max_levels, np.int64) for _ in range(4)]
    L = _load().orc_bfs_features(g.n, _p(off), _p(col), src, *[_p(b) for b in bufs], max_levels)
    if L < 0:
        raise OracleError(f"bfs_features rc={L}")
    return tuple(b[:L].copy() for b in bufs)


def sssp(g, src: int) -> np.ndarray:
    off, col = _arrs(g)
    if g.w is None:
        raise ValueError("sssp needs weights")
    w = np.ascontiguousarray(g.w, dtype=np.uint32)
    if w.size == 0:
        w = np.zeros(1, np.uint32)
    dist = np.empty(g.n, np.uint32)
    _check(_load().orc_sssp(g.n, _p(off), _p(col), _p(w), src, _p(dist)), "sssp")
    return dist


def cc(g) -> np.ndarray:
    off, col = _arrs(g)
    lab = np.empty(max(g.n, 1), np.int32)
    _check(_load().orc_cc(g.n, _p(off), _p(col), _p(lab)), "cc")
    return lab[:g.n]


def pr(g, damping: float = 0.85, iters: int = 20, csc=None) -> np.ndarray:
    """fp64 power iteration.  csc: optional in-edge graph (default: g itself)."""
    off, col = _arrs(g)
    coff, ccol = (off, col) if csc is None else _arrs(csc)
    out = np.empty(g.n, np.float64)
    _check(_load().orc_pr(g.n, _p(off), _p(coff), _p(ccol), damping, iters, _p(out)), "pr")
    return out


def dpr(g, damping: float = 0.85, eps: float = 1e-6, max_iters: int = 100000, csc=None):
    """fp64 Delta-PageRank (oracle.c orc_dpr, DESIGN R16).  eps is the ABSOLUTE residual threshold.

    Returns (rank, iterations)."""
    off, col = _arrs(g)
    coff, ccol = (off, col) if csc is None else _arrs(csc)
    out = np.empty(g.n, np.float64)
    it = np.zeros(1, np.int32)
    _check(_load().orc_dpr(g.n, _p(off), _p(coff), _p(ccol), damping, eps, max_iters, _p(out), _p(it)), "dpr")
    return out, int(it[0])


def bc(g, sources) -> np.ndarray:
    off, col = _arrs(g)
    s = np.ascontiguousarray(np.asarray(sources, dtype=np.int32))
    if s.size == 0:
        s = np.zeros(1, np.int32)
    out = np.empty(g.n, np.float64)
    _check(_load().orc_bc(g.n, _p(off), _p(col), _p(s), len(sources), _p(out)), "bc")
    return out


def attrs(g) -> dict:
    off, _ = _arrs(g)
    out = np.empty(7, np.float64)
    _check(_load().orc_attrs(g.n, _p(off), _p(out)), "attrs")
    return dict(zip(["N", "M", "dbar", "sigma_d", "r_d", "gini", "h_er"], out.tolist()))


def ratios(N, M, Va, Ea, Via, Eia) -> dict:
    out = np.empty(5, np.float64)
    _load().orc_ratios(N, M, Va, Ea, Via, Eia, _p(out))
    return dict(zip(["Vap", "Eap", "Viap", "Eiap", "cd"], out.tolist()))


def set_threads(k: int) -> None:
    """Threads for the per-vertex loops of pr / dpr (0 = all cores); results do not depend on it."""
    _load().orc_set_threads(int(k))


def threads() -> int:
    return int(_load().orc_threads())
