"""B200-native GSWITCH frontier-step library: thin Python binding over the C ABI (include/gsw.h).

Every step of the hot path (ingest, features, selector, Filter, Expand) runs in the CUDA kernels
of ``libgsw.so``; this module only marshals arguments.  PyTorch provides device memory (the
workspace and output tensors) and the CUDA stream.  There is no CPU fallback.

    g = Graph(row_offsets, col_indices, weights=None)     # numpy / torch (host or device)
    depth, stats = g.bfs(src)                             # torch int32 on the graph's device
    g.force_config(direction="pull", load_balance="twc")  # pin patterns (gsw_force_config)
"""
from __future__ import annotations

import ctypes
from typing import Optional, Sequence

import numpy as np

from . import _lib
from ._lib import (AUTO, BITMAP, DIRECTIONS, FORMATS, FUSED, FUSIONS, LB_CM, LB_STRICT,  # noqa: F401
                   LB_THREAD, LB_TWC, LB_WM, LOAD_BALANCES, PULL, PUSH, QUEUE, SORTED_QUEUE, STANDALONE,
                   STEPPINGS, GswError, check)

__all__ = ["Graph", "GswError", "version", "force_config_struct", "DistGraph", "HostDistGraph",
           "TorchHostExchange", "PartitionedGraph", "dist_slice", "dist_unique_id", "owned_rows"]


def version() -> str:
    return _lib.load().gsw_version().decode()


def _ptr_of(a):
    """(pointer, keepalive, is_device) for a numpy array or torch tensor (contiguous)."""
    import torch
    if isinstance(a, torch.Tensor):
        a = a.contiguous()
        return a.data_ptr(), a, a.is_cuda
    a = np.ascontiguousarray(a)
    return a.ctypes.data, a, False


def _as(a, np_dtype, torch_dtype):
    import torch
    if isinstance(a, torch.Tensor):
        return a.to(torch_dtype).contiguous()
    return np.ascontiguousarray(np.asarray(a, dtype=np_dtype))


def force_config_struct(direction=AUTO, format=AUTO, load_balance=AUTO, stepping=AUTO, fusion=AUTO,
                        delta0=0) -> _lib.gsw_config:
    def enc(v, table):
        if isinstance(v, str):
            return table[v.lower()]
        return int(v)
    return _lib.gsw_config(enc(direction, DIRECTIONS), enc(format, FORMATS),
                           enc(load_balance, LOAD_BALANCES), enc(stepping, STEPPINGS),
                           enc(fusion, FUSIONS), int(delta0))


def _stats_dict(st: _lib.gsw_run_stats, recs) -> dict:
    d = {"iterations": st.iterations, "gpu_ms": st.gpu_ms, "edges_touched": st.edges_touched,
         "bytes_alg": st.bytes_alg}
    if recs is not None:
        n = min(st.iterations, len(recs))
        d["records"] = [{k: getattr(recs[i], k) for k, _ in _lib.gsw_iter_record._fields_} for i in range(n)]
    return d


class Graph:
    """A graph resident in one device workspace (gsw_graph_create)."""

    def __init__(self, row_offsets, col_indices, weights=None, csc: Optional[tuple] = None,
                 device: str | int = "cuda", stream=None):
        import torch
        lib = _lib.load()
        self.device = torch.device(device)
        if self.device.type != "cuda":
            raise ValueError("gsw graphs live on a CUDA device")
        off = _as(row_offsets, np.int64, torch.int64)
        col = _as(col_indices, np.int32, torch.int32)
        w = None if weights is None else _as(weights, np.uint32, torch.int32)
        self.n = int(off.shape[0]) - 1
        self.nnz = int(col.shape[0])
        self.weighted = w is not None
        with torch.cuda.device(self.device):
            self.stream = stream if stream is not None else torch.cuda.current_stream(self.device)
            keep = []

            def mk(o, c, ww):
                po, ko, _ = _ptr_of(o)
                pc, kc, _ = _ptr_of(c) if self.nnz else (None, None, False)
                pw, kw, _ = _ptr_of(ww) if ww is not None else (None, None, False)
                keep.extend([ko, kc, kw])
                return _lib.gsw_csr(self.n, self.nnz, po, pc, pw)

            csr = mk(off, col, w)
            csc_s = None
            if csc is not None:
                coff = _as(csc[0], np.int64, torch.int64)
                ccol = _as(csc[1], np.int32, torch.int32)
                cw = None if len(csc) < 3 or csc[2] is None else _as(csc[2], np.uint32, torch.int32)
                csc_s = mk(coff, ccol, cw)
            nbytes = ctypes.c_size_t()
            check(lib.gsw_workspace_size(self.n, self.nnz, int(self.weighted), int(csc is not None),
                                         ctypes.byref(nbytes)), "gsw_workspace_size")
            self.workspace = torch.empty(nbytes.value, dtype=torch.uint8, device=self.device)
            h = ctypes.c_void_p()
            check(lib.gsw_graph_create(ctypes.byref(csr), ctypes.byref(csc_s) if csc_s is not None else None,
                                       self.workspace.data_ptr(), nbytes.value, self.stream.cuda_stream,
                                       ctypes.byref(h)), "gsw_graph_create")
            self._h = h
            del keep

    # -------------------------------------------------------------------------------------
    def close(self):
        if getattr(self, "_h", None):
            _lib.load().gsw_graph_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def attributes(self) -> dict:
        out = (ctypes.c_double * 7)()
        check(_lib.load().gsw_graph_attributes(self._h, out), "gsw_graph_attributes")
        return dict(zip(["N", "M", "dbar", "sigma_d", "r_d", "gini", "h_er"], list(out)))

    def validate(self) -> None:
        check(_lib.load().gsw_graph_validate(self._h), "gsw_graph_validate")

    def force_config(self, **kw) -> None:
        """Pin patterns: direction, format, load_balance, stepping, fusion, delta0 (None = AUTO)."""
        lib = _lib.load()
        if not kw or all(v in (None, 0, "auto") for v in kw.values()):
            check(lib.gsw_force_config(self._h, None), "gsw_force_config")
            return
        cfg = force_config_struct(**{k: (AUTO if v in (None, "auto") else v) for k, v in kw.items()})
        check(lib.gsw_force_config(self._h, ctypes.byref(cfg)), "gsw_force_config")

    # -------------------------------------------------------------------------------------
    def _stats(self, records: int):
        st = _lib.gsw_run_stats()
        recs = None
        if records:
            recs = (_lib.gsw_iter_record * records)()
            st.records = ctypes.cast(recs, ctypes.POINTER(_lib.gsw_iter_record))
            st.max_records = records
        return st, recs

    def _out(self, out, dtype):
        import torch
        if out is None:
            return torch.empty(getattr(self, "out_len", self.n), dtype=dtype, device=self.device)
        return out

    def bfs(self, source: int, out=None, records: int = 0):
        """Depths from `source` (-1 = unreachable).  `out` may be a host (pinned) or device tensor."""
        import torch
        out = self._out(out, torch.int32)
        st, recs = self._stats(records)
        check(_lib.load().gsw_bfs(self._h, int(source), out.data_ptr(), ctypes.byref(st)), "gsw_bfs")
        return out, _stats_dict(st, recs)

    def sssp(self, source: int, out=None, records: int = 0):
        """Shortest distances (uint32 values in an int32 tensor; 0xFFFFFFFF = unreachable)."""
        import torch
        out = self._out(out, torch.int32)
        st, recs = self._stats(records)
        check(_lib.load().gsw_sssp(self._h, int(source), out.data_ptr(), ctypes.byref(st)), "gsw_sssp")
        return out, _stats_dict(st, recs)

    def cc(self, out=None, records: int = 0):
        import torch
        out = self._out(out, torch.int32)
        st, recs = self._stats(records)
        check(_lib.load().gsw_cc(self._h, out.data_ptr(), ctypes.byref(st)), "gsw_cc")
        return out, _stats_dict(st, recs)

    def cc_hook(self, out=None, records: int = 0):
        """Connected components by hooking + pointer jumping (Soman et al.)."""
        import torch
        out = self._out(out, torch.int32)
        st, recs = self._stats(records)
        check(_lib.load().gsw_cc_hook(self._h, out.data_ptr(), ctypes.byref(st)), "gsw_cc_hook")
        return out, _stats_dict(st, recs)

    def pr(self, damping: float = 0.85, iters: int = 20, out=None, records: int = 0):
        import torch
        out = self._out(out, torch.float64)
        st, recs = self._stats(records)
        check(_lib.load().gsw_pr(self._h, float(damping), int(iters), out.data_ptr(), ctypes.byref(st)), "gsw_pr")
        return out, _stats_dict(st, recs)

    def dpr(self, damping: float = 0.85, tol: float = 1e-6, max_iters: int = 10000, out=None, records: int = 0):
        """Delta-PageRank (gsw_dpr): ||fixed point - rank||_1 <= tol."""
        import torch
        out = self._out(out, torch.float64)
        st, recs = self._stats(records)
        check(_lib.load().gsw_dpr(self._h, float(damping), float(tol), int(max_iters), out.data_ptr(),
                                  ctypes.byref(st)), "gsw_dpr")
        return out, _stats_dict(st, recs)

    def app_bfs(self, source: int, out=None, records: int = 0):
        """BFS written with the user-programmable front-end (include/gsw_app.cuh, gsw_app_bfs)."""
        import torch
        out = self._out(out, torch.int32)
        st, recs = self._stats(records)
        check(_lib.load().gsw_app_bfs(self._h, int(source), out.data_ptr(), ctypes.byref(st)), "gsw_app_bfs")
        return out, _stats_dict(st, recs)

    def app_sssp(self, source: int, out=None, records: int = 0):
        """SSSP written with the user-programmable front-end (include/gsw_app.cuh, gsw_app_sssp)."""
        import torch
        out = self._out(out, torch.int32)
        st, recs = self._stats(records)
        check(_lib.load().gsw_app_sssp(self._h, int(source), out.data_ptr(), ctypes.byref(st)), "gsw_app_sssp")
        return out, _stats_dict(st, recs)

    def bc(self, sources: Sequence[int], out=None, records: int = 0):
        import torch
        out = self._out(out, torch.float64)
        src = np.ascontiguousarray(np.asarray(list(sources), dtype=np.int32))
        st, recs = self._stats(records)
        check(_lib.load().gsw_bc(self._h, src.ctypes.data if src.size else None, int(src.size), out.data_ptr(),
                                 ctypes.byref(st)), "gsw_bc")
        return out, _stats_dict(st, recs)


# ------------------------------------------------------------------------------------------------
# Multi-GPU: 1D vertex partition (include/gsw.h "Multi-GPU").  BFS, PageRank and CC run on these
# handles; outputs cover the owned slice (NCCL / host-staged mode) or all vertices (loopback).

def dist_slice(n: int, nranks: int) -> int:
    """Slice size S: rank r owns vertices [r*S, min(n, (r+1)*S))."""
    return int(_lib.load().gsw_dist_slice(int(n), int(nranks)))


def dist_unique_id() -> bytes:
    """A fresh 128-byte ncclUniqueId (create on one rank, broadcast to the others)."""
    buf = ctypes.create_string_buffer(128)
    check(_lib.load().gsw_dist_unique_id(buf), "gsw_dist_unique_id")
    return buf.raw


class _Handle(Graph):
    """Shared methods of the partitioned handles (bfs, pr, force_config come from Graph)."""

    def __init__(self):   # noqa: D401 -- constructed by the subclasses
        pass


class DistGraph(_Handle):
    """NCCL mode: this process owns rows [rank*S, rank*S + n_owned) of an n_global-vertex
    symmetric graph (global column ids).  Collective: every rank constructs it in the same order."""

    def __init__(self, owned_offsets, owned_cols, n_global: int, nccl_id: bytes, nranks: int, rank: int,
                 device: str | int = "cuda", stream=None, weights=None):
        import torch
        lib = _lib.load()
        self.device = torch.device(device)
        off = _as(owned_offsets, np.int64, torch.int64)
        col = _as(owned_cols, np.int32, torch.int32)
        w = None if weights is None else _as(weights, np.uint32, torch.int32)
        self.n = int(n_global)
        self.out_len = int(off.shape[0]) - 1
        self.nnz = int(col.shape[0])
        self.rank, self.nranks = int(rank), int(nranks)
        with torch.cuda.device(self.device):
            self.stream = stream if stream is not None else torch.cuda.current_stream(self.device)
            po, ko, _ = _ptr_of(off)
            pc, kc, _ = _ptr_of(col) if self.nnz else (None, None, False)
            pw, kw, _ = _ptr_of(w) if w is not None else (None, None, False)
            csr = _lib.gsw_csr(self.out_len, self.nnz, po, pc, pw)
            nbytes = ctypes.c_size_t()
            check(lib.gsw_dist_workspace_size_weighted(self.n, self.nnz, self.nranks, int(w is not None), 0,
                                                       ctypes.byref(nbytes)), "gsw_dist_workspace_size_weighted")
            self.workspace = torch.empty(nbytes.value, dtype=torch.uint8, device=self.device)
            idbuf = ctypes.create_string_buffer(bytes(nccl_id), 128) if nccl_id is not None else None
            h = ctypes.c_void_p()
            check(lib.gsw_graph_create_dist(ctypes.byref(csr), self.n, idbuf, self.nranks, self.rank,
                                            self.workspace.data_ptr(), nbytes.value, self.stream.cuda_stream,
                                            ctypes.byref(h)), "gsw_graph_create_dist")
            self._h = h
            del ko, kc, kw


class TorchHostExchange:
    """Host-staged exchange (gsw_exchange) over a torch.distributed process group -- typically
    gloo, so several processes can share one GPU in tests.  Marshalling only: the callbacks move
    the library's pinned host buffers through the group's all_gather / all_reduce."""

    def __init__(self, group=None):
        import torch.distributed as dist
        self.dist, self.group = dist, group
        self.nranks = dist.get_world_size(group)

        def allgather(_user, send, recv, nbytes):
            try:
                import torch
                src = torch.from_numpy(np.ctypeslib.as_array(ctypes.cast(send, ctypes.POINTER(ctypes.c_uint8)),
                                                             shape=(nbytes,)).copy())
                outs = [torch.empty_like(src) for _ in range(self.nranks)]
                self.dist.all_gather(outs, src, group=self.group)
                dst = np.ctypeslib.as_array(ctypes.cast(recv, ctypes.POINTER(ctypes.c_uint8)),
                                            shape=(nbytes * self.nranks,))
                dst[:] = torch.cat(outs).numpy()
                return 0
            except Exception:                     # noqa: BLE001 -- reported to the library as failure
                return 1

        def allreduce(ctype, np_dtype):
            def fn(_user, buf, count):
                try:
                    import torch
                    arr = np.ctypeslib.as_array(buf, shape=(count,))
                    t = torch.from_numpy(arr.astype(np_dtype))
                    self.dist.all_reduce(t, group=self.group)
                    arr[:] = t.numpy()
                    return 0
                except Exception:                 # noqa: BLE001
                    return 1
            return fn

        self._fns = (_lib.ALLGATHER_FN(allgather), _lib.ALLREDUCE_U64_FN(allreduce(ctypes.c_uint64, np.int64)),
                     _lib.ALLREDUCE_F64_FN(allreduce(ctypes.c_double, np.float64)))
        self.struct = _lib.gsw_exchange(None, *self._fns)


class HostDistGraph(_Handle):
    """Host-staged mode: like DistGraph, but the per-iteration exchange goes through `exchange`
    (a TorchHostExchange) instead of NCCL.  The kernels are the same partitioned kernels."""

    def __init__(self, owned_offsets, owned_cols, n_global: int, exchange: "TorchHostExchange", rank: int,
                 device: str | int = "cuda", stream=None, weights=None):
        import torch
        lib = _lib.load()
        self.device = torch.device(device)
        off = _as(owned_offsets, np.int64, torch.int64)
        col = _as(owned_cols, np.int32, torch.int32)
        w = None if weights is None else _as(weights, np.uint32, torch.int32)
        self.n = int(n_global)
        self.out_len = int(off.shape[0]) - 1
        self.nnz = int(col.shape[0])
        self.rank, self.nranks = int(rank), exchange.nranks
        self._exchange = exchange                 # keeps the callbacks alive
        with torch.cuda.device(self.device):
            self.stream = stream if stream is not None else torch.cuda.current_stream(self.device)
            po, ko, _ = _ptr_of(off)
            pc, kc, _ = _ptr_of(col) if self.nnz else (None, None, False)
            pw, kw, _ = _ptr_of(w) if w is not None else (None, None, False)
            csr = _lib.gsw_csr(self.out_len, self.nnz, po, pc, pw)
            nbytes = ctypes.c_size_t()
            check(lib.gsw_dist_workspace_size_weighted(self.n, self.nnz, self.nranks, int(w is not None), 0,
                                                       ctypes.byref(nbytes)), "gsw_dist_workspace_size_weighted")
            self.workspace = torch.empty(nbytes.value, dtype=torch.uint8, device=self.device)
            h = ctypes.c_void_p()
            check(lib.gsw_graph_create_dist_host(ctypes.byref(csr), self.n, ctypes.byref(exchange.struct),
                                                 self.nranks, self.rank, self.workspace.data_ptr(), nbytes.value,
                                                 self.stream.cuda_stream, ctypes.byref(h)),
                  "gsw_graph_create_dist_host")
            self._h = h
            del ko, kc


class PartitionedGraph(_Handle):
    """Loopback mode: `nparts` virtual ranks of the full graph on this GPU, running the same
    partitioned kernels as DistGraph with the exchange done in device memory."""

    def __init__(self, row_offsets, col_indices, nparts: int, device: str | int = "cuda", stream=None,
                 weights=None):
        import torch
        lib = _lib.load()
        self.device = torch.device(device)
        off = _as(row_offsets, np.int64, torch.int64)
        col = _as(col_indices, np.int32, torch.int32)
        w = None if weights is None else _as(weights, np.uint32, torch.int32)
        self.n = int(off.shape[0]) - 1
        self.out_len = self.n
        self.nnz = int(col.shape[0])
        self.nparts = int(nparts)
        with torch.cuda.device(self.device):
            self.stream = stream if stream is not None else torch.cuda.current_stream(self.device)
            po, ko, _ = _ptr_of(off)
            pc, kc, _ = _ptr_of(col) if self.nnz else (None, None, False)
            pw, kw, _ = _ptr_of(w) if w is not None else (None, None, False)
            csr = _lib.gsw_csr(self.n, self.nnz, po, pc, pw)
            nbytes = ctypes.c_size_t()
            check(lib.gsw_dist_workspace_size_weighted(self.n, self.nnz, self.nparts, int(w is not None), 1,
                                                       ctypes.byref(nbytes)), "gsw_dist_workspace_size_weighted")
            self.workspace = torch.empty(nbytes.value, dtype=torch.uint8, device=self.device)
            h = ctypes.c_void_p()
            check(lib.gsw_graph_create_partitioned(ctypes.byref(csr), self.nparts, self.workspace.data_ptr(),
                                                   nbytes.value, self.stream.cuda_stream, ctypes.byref(h)),
                  "gsw_graph_create_partitioned")
            self._h = h
            del ko, kc, kw


def owned_rows(row_offsets, col_indices, rank: int, nranks: int, weights=None):
    """Rows [rank*S, min(n, (rank+1)*S)) of a CSR as (offsets rebased to 0, global columns[, weights])."""
    off = np.asarray(row_offsets, dtype=np.int64)
    n = off.shape[0] - 1
    S = dist_slice(n, nranks)
    vb, ve = min(n, rank * S), min(n, (rank + 1) * S)
    loc = off[vb:ve + 1] - off[vb]
    if weights is None:
        return loc, np.asarray(col_indices)[off[vb]:off[ve]]
    return loc, np.asarray(col_indices)[off[vb]:off[ve]], np.asarray(weights)[off[vb]:off[ve]]
