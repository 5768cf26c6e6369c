"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

This package holds no arithmetic of the method: it draws graphs (R-MAT / grid / Chung-Lu), edge
weights and source vertices, and builds CSR arrays.  The C implementation is ``gen/gen.c``
(counter-based splitmix64, so draws do not depend on thread count).
and SURVEY.md section 8 (d1-d5, Q5, Q12) for the recipes.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libgswgen.so")


def build() -> str:
    """Compile gen.c into libgswgen.so (gcc, -O3, OpenMP)."""
    src = os.path.join(_HERE, "gen.c")
    if not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O3", "-fopenmp", "-fPIC", "-shared", "-o", _SO, src, "-lm"])
    return _SO


class _Csr(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("nnz", ctypes.c_int64),
                ("off", ctypes.POINTER(ctypes.c_int64)), ("col", ctypes.POINTER(ctypes.c_int32)),
                ("w", ctypes.POINTER(ctypes.c_uint32))]


_lib = None


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_SO)
        lib.gen_rmat.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_double, ctypes.c_double,
                                 ctypes.c_double, ctypes.c_uint64, ctypes.c_int, ctypes.POINTER(_Csr)]
        lib.gen_rmat_slice.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_double, ctypes.c_double,
                                       ctypes.c_double, ctypes.c_uint64, ctypes.c_int, ctypes.c_int64,
                                       ctypes.c_int64, ctypes.POINTER(_Csr)]
        lib.gen_grid.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.POINTER(_Csr)]
        lib.gen_chung_lu.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_double, ctypes.c_double,
                                     ctypes.c_uint64, ctypes.POINTER(_Csr)]
        lib.gen_hash_weights.argtypes = [ctypes.POINTER(_Csr), ctypes.c_uint64, ctypes.c_uint32]
        lib.gen_free.argtypes = [ctypes.POINTER(_Csr)]
        lib.gen_set_threads.argtypes = [ctypes.c_int]
        lib.gen_set_threads.restype = None
        lib.gen_splitmix64.argtypes = [ctypes.c_uint64]
        lib.gen_splitmix64.restype = ctypes.c_uint64
        _lib = lib
    return _lib


@dataclass
class Graph:
    """Host CSR: row offsets (int64, n+1), column indices (int32, nnz), optional uint32 weights."""
    n: int
    off: np.ndarray
    col: np.ndarray
    w: Optional[np.ndarray] = None
    name: str = ""

    @property
    def nnz(self) -> int:
        return int(self.off[-1]) if self.n > 0 else 0

    @property
    def deg(self) -> np.ndarray:
        return np.diff(self.off)


def _take(c: _Csr, name: str) -> Graph:
    lib = _load()
    n, nnz = int(c.n), int(c.nnz)
    off = np.ctypeslib.as_array(c.off, shape=(n + 1,)).copy()
    col = np.ctypeslib.as_array(c.col, shape=(max(nnz, 1),))[:nnz].copy()
    w = None
    if c.w:
        w = np.ctypeslib.as_array(c.w, shape=(max(nnz, 1),))[:nnz].copy()
    lib.gen_free(ctypes.byref(c))
    return Graph(n, off, col, w, name)


def rmat(scale: int, edgefactor: int = 16, a: float = 0.57, b: float = 0.19, c: float = 0.19,
         seed: int = 1, permute: bool = True) -> Graph:
    """Graph500-style R-MAT / Kronecker graph, symmetrised, deduplicated, loop-free."""
    lib, out = _load(), _Csr()
    rc = lib.gen_rmat(scale, edgefactor, a, b, c, seed, int(permute), ctypes.byref(out))
    if rc != 0:
        raise MemoryError(f"gen_rmat failed rc={rc}")
    return _take(out, f"rmat{scale}_ef{edgefactor}_s{seed}")


def rmat_slice(scale: int, vb: int, ve: int, edgefactor: int = 16, a: float = 0.57, b: float = 0.19,
               c: float = 0.19, seed: int = 1, permute: bool = True):
    """Rows [vb, ve) of ``rmat(scale, ...)`` as (offsets rebased to 0, global column ids), built
    without materialising the other rows (gen.c gen_rmat_slice): one rank's share of a 1D
    vertex-partitioned graph, or with [0, 2^scale) the whole graph."""
    lib, out = _load(), _Csr()
    rc = lib.gen_rmat_slice(scale, edgefactor, a, b, c, seed, int(permute), vb, ve, ctypes.byref(out))
    if rc != 0:
        raise MemoryError(f"gen_rmat_slice failed rc={rc}")
    g = _take(out, "")
    return g.off, g.col


def grid(width: int, height: Optional[int] = None) -> Graph:
    """4-neighbour 2D grid (road-like), row-major vertex ids."""
    height = width if height is None else height
    lib, out = _load(), _Csr()
    rc = lib.gen_grid(width, height, ctypes.byref(out))
    if rc != 0:
        raise MemoryError(f"gen_grid failed rc={rc}")
    return _take(out, f"grid{width}x{height}")


def chung_lu(n: int, pairs: int, gamma: float = 2.3, i0: float = 150.0, seed: int = 3) -> Graph:
    """Chung-Lu power-law graph (soc-LiveJournal1-shaped at n=4,847,571, pairs=68,993,773)."""
    lib, out = _load(), _Csr()
    rc = lib.gen_chung_lu(n, pairs, gamma, i0, seed, ctypes.byref(out))
    if rc != 0:
        raise MemoryError(f"gen_chung_lu failed rc={rc}")
    return _take(out, f"chunglu{n}_{pairs}")


def with_hash_weights(g: Graph, seed: int = 12345, maxw: int = 64) -> Graph:
    """Attach symmetric weights w(u,v) = 1 + splitmix64((min*N+max) ^ seed) % maxw."""
    lib = _load()
    c = _Csr(g.n, g.nnz, g.off.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
             g.col.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)), None)
    rc = lib.gen_hash_weights(ctypes.byref(c), seed, maxw)
    if rc != 0:
        raise MemoryError("gen_hash_weights failed")
    w = np.ctypeslib.as_array(c.w, shape=(max(g.nnz, 1),))[:g.nnz].copy()
    # free only the weight buffer (off/col belong to numpy)
    ctypes.CDLL(None).free(ctypes.cast(c.w, ctypes.c_void_p))
    return Graph(g.n, g.off, g.col, w, g.name + f"_w{maxw}")


def set_threads(k: int) -> None:
    """OpenMP threads of the C generators (0 = all cores); draws do not depend on it."""
    _load().gen_set_threads(int(k))


def splitmix64(x: int) -> int:
    return int(_load().gen_splitmix64(x & 0xFFFFFFFFFFFFFFFF))


def sources(g: Graph, count: int, seed: int = 7) -> list[int]:
    """Source stream: v_k = splitmix64((seed << 32) | k) mod N, skipping degree-0
    vertices and repeats."""
    deg = g.deg
    out, seen, k = [], set(), 0
    if int((deg > 0).sum()) < count:
        raise ValueError("not enough non-isolated vertices")
    while len(out) < count:
        v = splitmix64((seed << 32) | k) % g.n
        k += 1
        if deg[v] == 0 or v in seen:
            continue
        seen.add(v)
        out.append(int(v))
    return out


def from_edges(n: int, edges, weights=None, symmetric: bool = True, dedupe: bool = True,
               drop_loops: bool = True) -> Graph:
    """CSR from an explicit edge list (tiny hand-built graphs).  With symmetric=True each (u,v[,w])
    also adds (v,u[,w]).  With dedupe=False parallel edges and self-loops may be kept (multigraph,
    SURVEY Q2)."""
    e = np.asarray(edges, dtype=np.int64).reshape(-1, 2)
    w = None if weights is None else np.asarray(weights, dtype=np.int64).reshape(-1)
    src, dst = e[:, 0], e[:, 1]
    ww = w
    if symmetric:
        src, dst = np.concatenate([e[:, 0], e[:, 1]]), np.concatenate([e[:, 1], e[:, 0]])
        ww = None if w is None else np.concatenate([w, w])
    if drop_loops:
        keep = src != dst
        src, dst = src[keep], dst[keep]
        ww = None if ww is None else ww[keep]
    order = np.lexsort((dst, src))
    src, dst = src[order], dst[order]
    ww = None if ww is None else ww[order]
    if dedupe and src.size:
        keep = np.ones(src.size, bool)
        keep[1:] = (src[1:] != src[:-1]) | (dst[1:] != dst[:-1])
        src, dst = src[keep], dst[keep]
        ww = None if ww is None else ww[keep]
    off = np.zeros(n + 1, np.int64)
    np.add.at(off, src + 1, 1)
    off = np.cumsum(off)
    return Graph(n, off, dst.astype(np.int32), None if ww is None else ww.astype(np.uint32), "edges")


# --- the five BASELINE.json configs (sizes table) ---------------------------------

def config_graph(name: str) -> Graph:
    """C1..C5 inputs.  C1: R-MAT 16; C2: 2048^2 weighted grid; C3: R-MAT 22; C4: Chung-Lu LJ-shaped;
    C5: Kronecker 26."""
    if name == "C1":
        return rmat(16, 16, seed=1)
    if name == "C2":
        return with_hash_weights(grid(2048), seed=12345, maxw=64)
    if name == "C3":
        return rmat(22, 16, seed=1)
    if name == "C4":
        return chung_lu(4_847_571, 68_993_773, gamma=2.3, i0=150.0, seed=3)
    if name == "C5":
        off, col = rmat_slice(26, 0, 1 << 26, 16, seed=1)    # the same graph as rmat(26), built in parallel
        return Graph(1 << 26, off, col, None, "rmat26_ef16_s1")
    raise KeyError(name)
