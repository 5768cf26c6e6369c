"""Parallel CPU baselines timed beside the GPU in bench.py ("an OpenMP
level-synchronous BFS on all host cores").  Context only: not the oracle, not the product path."""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libompbase.so")
_lib = None


def build() -> str:
    src = os.path.join(_HERE, "omp_bfs.c")
    if not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O3", "-fopenmp", "-fPIC", "-shared", "-o", _SO, src])
    return _SO


def _load():
    global _lib
    if _lib is None:
        build()
        _lib = ctypes.CDLL(_SO)
        P = ctypes.c_void_p
        _lib.omp_bfs.argtypes = [ctypes.c_int64, P, P, ctypes.c_int32, P]
        _lib.omp_threads.restype = ctypes.c_int
    return _lib


def bfs(g, src: int) -> np.ndarray:
    off = np.ascontiguousarray(g.off, dtype=np.int64)
    col = np.ascontiguousarray(g.col, dtype=np.int32)
    out = np.empty(g.n, np.int32)
    rc = _load().omp_bfs(g.n, off.ctypes.data, col.ctypes.data, int(src), out.ctypes.data)
    if rc:
        raise RuntimeError(f"omp_bfs rc={rc}")
    return out


def threads() -> int:
    return int(_load().omp_threads())
