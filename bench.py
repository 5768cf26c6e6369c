#!/usr/bin/env python
"""Benchmark of the GSWITCH frontier-step hot path on B200 (BASELINE.json metric, config C3).

Headline workload (north_star: ">=40% of the B200 HBM roofline on RMAT scale-22 BFS at 1 GPU"):
BFS on the C3 graph (Graph500 R-MAT scale 22, edge factor 16, symmetrised), roots from the
SURVEY Q12 source stream.  One step = one autotuned gsw_bfs call (features -> selector -> Filter
-> Expand per level, all inside one persistent kernel) from the next root.

  python bench.py [--gpus N --steps K --warmup W] [--impl reference] [--workload C3|C5]

Prints ONE JSON line on rank 0.  GTEPS = sum over steps of m_cc / device time, with m_cc = the
undirected edges with both endpoints reached.  L2 is flushed (256 MiB write) between
timed steps; each step's device time is the span of the call's device work from the library's
CUDA events on its stream (SURVEY 8(d) timing protocol); the host-inclusive time of the synchronous
call is reported beside it; max over ranks.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

PEAKS_FILE = os.path.join(ROOT, "MEASURED_PEAKS.json")
FALLBACK_HBM = 6650.0   # GB/s, B200_PROFILING.md fallback
# random 4-byte L2 gathers per second (G/s), measured by tools/micro_gather.cu (profiles/r2/micro_gather.txt)
PR_GATHER_PEAK = 356.0


def workload_label(workload, g=None, n=None, nnz=None):
    """The `config.workload` string both arms print for the same graph (the driver compares them)."""
    scale = {"C3": 22, "C5": 26}.get(workload, 22)
    n = g.n if g is not None else n
    nnz = g.nnz if g is not None else nnz
    return (f"{workload}: BFS on R-MAT scale {scale} ef 16 (Graph500 a,b,c=.57,.19,.19), n={n}, nnz={nnz}, "
            "roots per SURVEY Q12")


def csr_hash(g):
    """Content hash of the generated CSR (recorded in every result line), so lines
    from different runs can be checked to have timed the same graph."""
    import hashlib
    h = hashlib.sha256()
    h.update(np.ascontiguousarray(g.off).view(np.uint8))
    h.update(np.ascontiguousarray(g.col).view(np.uint8))
    return "sha256:" + h.hexdigest()[:16]


def hbm_peak():
    try:
        with open(PEAKS_FILE) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return FALLBACK_HBM, "fallback (B200_PROFILING.md)"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.p = None

    def __enter__(self):
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "50"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.p = None
        return self

    def __exit__(self, *a):
        self.out = ""
        if self.p:
            time.sleep(0.12)
            self.p.terminate()
            try:
                self.out, _ = self.p.communicate(timeout=5)
            except Exception:
                self.out = ""

    def summary(self):
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for line in (self.out or "").strip().splitlines():
            parts = [x.strip() for x in line.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                mx = float(parts[1])
            except ValueError:
                continue
            for nm, v in zip(names, parts[3:7]):
                if v.lower() == "active":
                    reasons.add(nm)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": mx, "reasons": sorted(reasons), "samples": 0}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm)}


MAX_FRAC = 1.2


def sane_frac(frac, what):
    """A roofline fraction above 1.2 means the byte model or the run is broken (a
    corrupted SSSP counter reported 8093x peak); refuse to print it."""
    if not (frac == frac) or frac < 0 or frac > MAX_FRAC:
        raise SystemExit(f"bench: roofline fraction {frac!r} for {what} is outside [0, {MAX_FRAC}]: "
                         "the run or its byte model is broken; refusing to report it")
    return frac


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def m_cc(deg, depth):
    return int(deg[depth >= 0].sum()) // 2


def build_graph(name):
    import gen
    t0 = time.time()
    g = gen.config_graph(name)
    return g, time.time() - t0


# --------------------------------------------------------------------------------------------
def run_reference(args, ws, rank):
    """--impl reference: the CPU oracle (plain single-threaded C) on the host cores, on the same
    workload as this arm: C3 BFS at N = 1, the partitioned C5 BFS for N > 1 (rank 0 only; the
    oracle holds the whole graph).  C5 steps are a bounded sample (2 roots, ~40 s each)."""
    if rank != 0:
        return
    import gen
    import oracle
    c5 = (ws > 1 or args.partitioned) and not (args.dist_workload_forced and args.workload == "C3")
    workload = "C5" if c5 else args.workload
    gen.set_threads(0)          # torchrun exports OMP_NUM_THREADS=1: generate with every core
    g, _ = build_graph(workload)
    deg = g.deg
    roots = gen.sources(g, max(64, args.steps + args.warmup))
    nsteps = min(args.steps, 2) if workload == "C5" else args.steps
    if workload != "C5":
        for k in range(args.warmup):
            oracle.bfs(g, roots[k % len(roots)])
    edges, secs = 0, 0.0
    for k in range(nsteps):
        s = roots[(args.warmup + k) % len(roots)]
        t0 = time.perf_counter()
        d = oracle.bfs(g, s)
        secs += time.perf_counter() - t0
        edges += m_cc(deg, d)
    v = edges / secs / 1e9
    line = {"impl": "reference", "metric": "BFS GTEPS", "value": v, "unit": "GTEPS", "n_gpus": ws,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": secs * 1e3 / nsteps,
            "higher_is_better": True, "scaling": "strong" if c5 else "weak", "vs_baseline": None, "dtype": "int32",
            "data": "synthetic",
            "config": ({"workload": workload_label(workload, g)} if c5
                       else {"workload": workload_label(workload, g), "csr_hash": csr_hash(g)}),
            "parallelism": "single host thread",
            "cpu_baseline": {"value": v, "unit": "GTEPS", "cores": 1, "kind": "oracle",
                             "sample": f"{nsteps} BFS roots, full {workload} graph, oracle.bfs (FIFO queue, 1 thread)"},
            "e2e": {"value": v, "unit": "GTEPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# --------------------------------------------------------------------------------------------
def cpu_baseline_sample(g, roots, budget_s=12.0):
    import oracle
    deg = g.deg
    edges, secs, n = 0, 0.0, 0
    for s in roots:
        t0 = time.perf_counter()
        d = oracle.bfs(g, s)
        secs += time.perf_counter() - t0
        edges += m_cc(deg, d)
        n += 1
        if secs > budget_s:
            break
    return {"value": edges / secs / 1e9, "unit": "GTEPS", "cores": 1, "kind": "oracle",
            "sample": f"{n} BFS roots on the full {g.name} graph, single-threaded oracle.bfs, {secs:.1f} s"}


def run_extras(gsw, dev, G3, g3, peak, cpu=True):
    """The other BASELINE.json configs (device time of one autotuned call, best of 3, L2 flushed
    before each): C3 CC, PageRank (20 iterations, d = 0.85) and Delta-PR (tol 1e-6), C2 SSSP, C4 BC
    (16 sources), C1 BFS over 64 roots.  Beside each, the CPU oracle timed on the host cores on a
    bounded sample of the same workload (SURVEY 8(d) "oracle timing beside it"), and for BFS the
    OpenMP level-synchronous baseline on all cores (cpu_baselines/)."""
    import torch
    import gen
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    if cpu:
        import oracle
        import cpu_baselines
        oracle.set_threads(0)

    def best(fn):
        b = None
        for k in range(3):
            flush.fill_(k)
            torch.cuda.synchronize()
            r = fn()
            if b is None or r[1]["gpu_ms"] < b[1]["gpu_ms"]:
                b = r
        return b[1]

    def rec(value, unit, st):
        gbs = st["bytes_alg"] / (st["gpu_ms"] * 1e-3) / 1e9
        return {"value": value, "unit": unit, "gpu_ms": st["gpu_ms"], "iterations": st["iterations"],
                "roofline_frac": sane_frac(gbs / peak, unit), "achieved_gbs": gbs}

    def timed(fn):
        t0 = time.perf_counter()
        r = fn()
        return r, time.perf_counter() - t0

    out = {}
    st = best(lambda: G3.cc())
    out["C3_cc"] = rec(g3.nnz / 2 / (st["gpu_ms"] * 1e-3) / 1e9, "GTEPS", st)
    if cpu:
        _, secs = timed(lambda: oracle.cc(g3))
        out["C3_cc"]["cpu_baseline"] = {"value": g3.nnz / 2 / secs / 1e9, "unit": "GTEPS", "cores": 1,
                                        "kind": "oracle", "sample": f"whole C3, union-find, {secs:.2f} s"}
    st = best(lambda: G3.pr(0.85, 20))
    out["C3_pr"] = rec(20 / (st["gpu_ms"] * 1e-3), "PR iters/s", st)
    if cpu:
        _, secs = timed(lambda: oracle.pr(g3, 0.85, 2))
        out["C3_pr"]["cpu_baseline"] = {"value": 2 / secs, "unit": "PR iters/s", "cores": oracle.threads(),
                                        "kind": "oracle", "sample": f"2 fp64 iterations, per-vertex loop over "
                                                                    f"{oracle.threads()} OpenMP threads, {secs:.2f} s"}
    # PR's Expand is bound by random 4-byte gathers of L2-resident contributions, not by HBM:
    # its ceiling is the measured gather rate of tools/micro_gather.cu
    gps = g3.nnz * 20 / (st["gpu_ms"] * 1e-3) / 1e9
    out["C3_pr"]["gather_roofline"] = {
        "bound": "l2_gather", "achieved": gps, "peak": PR_GATHER_PEAK, "unit": "G gathers/s",
        "frac": gps / PR_GATHER_PEAK,
        "peak_source": "tools/micro_gather.cu on B200: 128M streamed power-law indices gathering 4-byte "
                       "values of a 16.8 MB array with a 28,672-entry shared-memory hub cache "
                       "(profiles/r2/micro_gather.txt; uniform indices without cache: 265)"}
    # hooking + pointer-jumping CC (gsw_cc_hook, Soman et al.) beside the GSWITCH CC
    st = best(lambda: G3.cc_hook())
    out["C3_cc_hook"] = rec(g3.nnz / 2 / (st["gpu_ms"] * 1e-3) / 1e9, "GTEPS", st)
    # Delta-PR (DESIGN R16): tol = 1e-6 in L1; GTEPS over the edges its Expand read
    st = best(lambda: G3.dpr(0.85, 1e-6))
    out["C3_dpr"] = rec(st["edges_touched"] / (st["gpu_ms"] * 1e-3) / 1e9, "GTEPS (edges read)", st)
    g2 = gen.config_graph("C2")
    G2 = gsw.Graph(g2.off, g2.col, g2.w, device=dev)
    st = best(lambda: G2.sssp(0))
    out["C2_sssp"] = rec(g2.nnz / 2 / (st["gpu_ms"] * 1e-3) / 1e9, "GTEPS", st)
    out["C2_sssp"]["us_per_round"] = st["gpu_ms"] * 1e3 / max(1, st["iterations"])
    if cpu:
        _, secs = timed(lambda: oracle.sssp(g2, 0))
        out["C2_sssp"]["cpu_baseline"] = {"value": g2.nnz / 2 / secs / 1e9, "unit": "GTEPS", "cores": 1,
                                          "kind": "oracle", "sample": f"binary-heap Dijkstra from vertex 0, {secs:.2f} s "
                                                                      "(no parallel CPU variant: Dijkstra is serial)"}
    # CC on the road grid: label propagation would need ~4,000 iterations (the grid's diameter); the
    # autotuned gsw_cc hands over to hooking after 12, gsw_cc_hook alone needs 2 sweeps
    G2u = gsw.Graph(g2.off, g2.col, device=dev)
    st = best(lambda: G2u.cc())
    out["C2_cc"] = rec(g2.nnz / 2 / (st["gpu_ms"] * 1e-3) / 1e9, "GTEPS", st)
    st = best(lambda: G2u.cc_hook())
    out["C2_cc_hook"] = rec(g2.nnz / 2 / (st["gpu_ms"] * 1e-3) / 1e9, "GTEPS", st)
    del G2, G2u, g2
    g4 = gen.config_graph("C4")
    G4 = gsw.Graph(g4.off, g4.col, device=dev)
    srcs = gen.sources(g4, 16)
    st = best(lambda: G4.bc(srcs))
    out["C4_bc"] = rec(16 * g4.nnz / 2 / (st["gpu_ms"] * 1e-3) / 1e9, "GTEPS", st)
    if cpu:
        _, secs = timed(lambda: oracle.bc(g4, srcs[:1]))
        out["C4_bc"]["cpu_baseline"] = {"value": g4.nnz / 2 / secs / 1e9, "unit": "GTEPS", "cores": 1,
                                        "kind": "oracle", "sample": f"Brandes from 1 of the 16 sources, {secs:.2f} s"}
    del G4, g4
    g1 = gen.config_graph("C1")
    G1 = gsw.Graph(g1.off, g1.col, device=dev)
    roots1 = gen.sources(g1, 64)
    rates, tot_ms, tot_e = [], 0.0, 0
    for s in roots1:
        d, st1 = G1.bfs(s)
        e = m_cc(g1.deg, d.cpu().numpy())
        rates.append(e / (st1["gpu_ms"] * 1e-3) / 1e9)
        tot_ms += st1["gpu_ms"]
        tot_e += e
    hm = lambda r: len(r) / sum(1.0 / x for x in r)
    out["C1_bfs"] = {"value": hm(rates), "unit": "GTEPS (harmonic mean, 64 roots)",
                     "aggregate_gteps": tot_e / (tot_ms * 1e-3) / 1e9, "gpu_ms_per_root": tot_ms / 64}
    if cpu:
        rs, ro = [], []
        for s in roots1:
            d, secs = timed(lambda: oracle.bfs(g1, s))
            rs.append(m_cc(g1.deg, d) / secs / 1e9)
            d, secs = timed(lambda: cpu_baselines.bfs(g1, s))
            ro.append(m_cc(g1.deg, d) / secs / 1e9)
        out["C1_bfs"]["cpu_baseline"] = {"value": hm(rs), "unit": "GTEPS (harmonic mean, 64 roots)", "cores": 1,
                                         "kind": "oracle", "sample": "the same 64 roots, oracle.bfs"}
        out["C1_bfs"]["cpu_openmp"] = {"value": hm(ro), "unit": "GTEPS (harmonic mean, 64 roots)",
                                       "cores": cpu_baselines.threads(), "kind": "openmp level-synchronous BFS",
                                       "sample": "the same 64 roots, cpu_baselines.bfs"}
    return out


def run_c5_extra(gsw, dev, peak, roots_n=2):
    """C5 (Kronecker scale 26, 2.1e9 entries) on this one GPU, twice: the single-GPU persistent
    engine (gsw.Graph) and the 1D-partitioned path at p = 1 (gsw.DistGraph: NCCL with one rank,
    the same kernels and exchange code as bench.py --gpus N), so the N > 1 lines have their p = 1
    point.  BFS over `roots_n` roots (device span, L2 flushed) and PageRank (20 iterations)."""
    import torch
    import gen
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    t0 = time.time()
    g = gen.config_graph("C5")
    gen_s = time.time() - t0
    roots = gen.sources(g, roots_n)
    deg = g.deg
    out = {"gen_seconds": gen_s, "n": g.n, "nnz": g.nnz, "roots": roots}
    for name, make in (("single_gpu", lambda: gsw.Graph(g.off, g.col, device=dev)),
                       ("partitioned_p1", lambda: gsw.DistGraph(g.off, g.col, g.n, None, 1, 0, device=dev))):
        G = make()
        dd = torch.empty(g.n, dtype=torch.int32, device=dev)
        G.bfs(roots[0], out=dd)                           # warm-up
        ms, edges, bytes_alg = 0.0, 0, 0
        for s in roots:
            flush.fill_(1)
            torch.cuda.synchronize()
            _, st = G.bfs(s, out=dd)
            ms += st["gpu_ms"]
            bytes_alg += st["bytes_alg"]
            edges += m_cc(deg, dd.cpu().numpy())
        flush.fill_(2)
        torch.cuda.synchronize()
        _, stp = G.pr(0.85, 20)
        gbs = bytes_alg / (ms * 1e-3) / 1e9
        out[name] = {"bfs_gteps": edges / (ms * 1e-3) / 1e9, "bfs_ms_per_root": ms / len(roots),
                     "bfs_roofline_frac": sane_frac(gbs / peak, f"C5 {name}"), "pr_iters_per_s": 20 / (stp["gpu_ms"] * 1e-3),
                     "pr_gpu_ms": stp["gpu_ms"]}
        del G, dd
        torch.cuda.empty_cache()
    return out


def dist_sources(gsw, off_local, vb, n, count, dev, seed=7):
    """The SURVEY Q12 root stream (gen.sources) on a partitioned graph: candidate k is
    splitmix64((seed << 32) | k) mod n; its owner says whether it has edges; repeats and
    degree-0 vertices are skipped, as gen.sources does on the whole graph."""
    import torch
    import torch.distributed as dist
    import gen
    ncand = 64 * count + 256
    cand = [gen.splitmix64((seed << 32) | k) % n for k in range(ncand)]
    deg = np.diff(off_local)
    ok = torch.zeros(ncand, dtype=torch.int32, device=dev)
    loc = [1 if vb <= v < vb + deg.size and deg[v - vb] > 0 else 0 for v in cand]
    ok += torch.tensor(loc, dtype=torch.int32, device=dev)
    if dist.is_initialized():
        dist.all_reduce(ok, op=dist.ReduceOp.MAX)
    ok = ok.cpu().numpy()
    out, seen = [], set()
    for v, good in zip(cand, ok):
        if good and v not in seen:
            seen.add(v)
            out.append(int(v))
            if len(out) == count:
                break
    return out


def partition_input(workload, rank, ws):
    """This rank's owned rows of the workload graph, generated directly (gen.rmat_slice)."""
    import gen
    import paper_conf_ppopp_menglts19_b200 as gsw
    scale = {"C5": 26, "C3": 22}[workload]
    n = 1 << scale
    S = gsw.dist_slice(n, ws)
    vb, ve = min(n, rank * S), min(n, (rank + 1) * S)
    # torchrun sets OMP_NUM_THREADS=1; give this rank its share of the node's cores for generation
    local_ws = int(os.environ.get("LOCAL_WORLD_SIZE", ws))
    gen.set_threads(max(1, (os.cpu_count() or 1) // max(1, local_ws)))
    t0 = time.time()
    off, col = gen.rmat_slice(scale, vb, ve, 16, seed=1)
    return n, vb, off, col, time.time() - t0


def run_gsw_dist(args, ws, rank, local):
    """N > 1 (default): C5 (Kronecker scale 26) 1D vertex-partitioned over N ranks, one per GPU
    (BASELINE config 5): BFS with the per-level NCCL bitmap all-gather + feature
    all-reduce and device-side decisions, and PageRank with the fp32 contribution all-gather.
    Strong scaling: the graph is fixed, each rank holds 1/N of it.  --partitioned runs the same at
    N = 1 (NCCL with one rank)."""
    import torch
    import torch.distributed as dist
    import paper_conf_ppopp_menglts19_b200 as gsw

    host_ex = args.exchange == "host"
    if host_ex:
        local = 0        # --exchange host: every rank on GPU 0 (tests the N > 1 logic on one GPU)
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if "RANK" not in os.environ:
        os.environ.update(RANK="0", WORLD_SIZE="1", LOCAL_RANK="0", MASTER_ADDR="127.0.0.1",
                          MASTER_PORT=str(29500 + os.getpid() % 1000))
    if host_ex:
        dist.init_process_group("gloo")
    else:
        dist.init_process_group("nccl", device_id=dev)
    rdev = torch.device("cpu") if host_ex else dev        # device of the bench's own reductions
    workload = args.workload if args.workload != "C3" or args.dist_workload_forced else "C5"
    n, vb, off, col, gen_s = partition_input(workload, rank, ws)
    nroots = args.steps + args.warmup
    roots = dist_sources(gsw, off, vb, n, nroots, rdev)
    ex = gsw.TorchHostExchange() if host_ex else None

    def make_graph(o, c):
        if host_ex:
            return gsw.HostDistGraph(o, c, n, ex, rank, device=dev)
        ids = [gsw.dist_unique_id() if rank == 0 else None]       # an ncclUniqueId serves one communicator
        dist.broadcast_object_list(ids, src=0)
        return gsw.DistGraph(o, c, n, ids[0], ws, rank, device=dev)

    t0 = time.time()
    D = make_graph(off, col)
    create_s = time.time() - t0
    deg = np.diff(off)
    out = torch.empty(max(D.out_len, 1), dtype=torch.int32, device=dev)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)

    def mx(x):
        t = torch.tensor([float(x)], device=rdev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def sm(x):
        t = torch.tensor([float(x)], device=rdev, dtype=torch.float64)
        dist.all_reduce(t)
        return float(t.item())

    for k in range(args.warmup):
        D.bfs(roots[k], out=out)
    torch.cuda.synchronize()
    dist.barrier()
    tot_ms, edges_cc, bytes_alg, levels = 0.0, 0, 0, 0
    with ClockSampler(local) as cs:
        for k in range(args.steps):
            flush.fill_(k & 0xff)
            torch.cuda.synchronize()
            dist.barrier()
            _, st = D.bfs(roots[args.warmup + k], out=out)
            tot_ms += mx(st["gpu_ms"])                   # device span of the call, slowest rank
            bytes_alg += st["bytes_alg"]                 # global (same on every rank)
            levels += st["iterations"]
            d = out[:D.out_len].cpu().numpy()
            edges_cc += int(sm(int(deg[d >= 0].sum()))) // 2
    value = edges_cc / (tot_ms * 1e-3) / 1e9
    # PageRank, 20 iterations (d = 0.85), best of 2
    pr_ms = None
    for _ in range(2):
        flush.fill_(1)
        torch.cuda.synchronize()
        dist.barrier()
        _, st = D.pr(0.85, 20)
        t = mx(st["gpu_ms"])
        pr_ms = t if pr_ms is None else min(pr_ms, t)
    pr_bytes = st["bytes_alg"]
    peak, peak_src = hbm_peak()
    per_gpu_gbs = bytes_alg / ws / (tot_ms * 1e-3) / 1e9
    # e2e: owned CSR from pinned host memory -> DistGraph (H2D + slice build) -> BFS into pinned host
    pin_off = torch.from_numpy(off).pin_memory()
    pin_col = torch.from_numpy(col).pin_memory()
    host_out = torch.empty(max(D.out_len, 1), dtype=torch.int32).pin_memory()
    del D
    torch.cuda.empty_cache()
    e2e_ms, e2e_edges = 0.0, 0
    ke = 2
    for k in range(ke):
        dist.barrier()
        t0 = time.perf_counter()
        D2 = make_graph(pin_off, pin_col)
        D2.bfs(roots[args.warmup + k], out=host_out)
        e2e_ms += mx((time.perf_counter() - t0) * 1e3)
        e2e_edges += int(sm(int(deg[host_out.numpy()[:D2.out_len] >= 0].sum()))) // 2
        del D2
        torch.cuda.empty_cache()
    h2d_all = sm(off.nbytes + col.nbytes)           # collectives on every rank, before the rank-0 print
    d2h_all = sm(4 * max(1, len(host_out)))
    nnz_g = sm(len(col))
    if rank == 0:
        launches_per_level = 4                      # push, push_heavy, pull, decide (+ NCCL kernels)
        line = {
            "metric": "BFS GTEPS", "value": value, "unit": "GTEPS", "n_gpus": ws,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": tot_ms / args.steps, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "config": {"workload": workload_label(workload, n=n, nnz=int(nnz_g))},
            "partition": f"1D vertex partition over {ws} ranks (slice {gsw.dist_slice(n, ws)}), per-level NCCL "
                         "bitmap all-gather",
            "l2": "flushed between steps (256 MiB write outside the timed span)",
            "parallelism": f"1D vertex partition x{ws} " + ("(host-staged exchange over gloo, all ranks on GPU 0: "
                                                     "a logic test, not a measurement)" if host_ex else "(NCCL over NVLink)"),
            "roofline": {"bound": "hbm", "achieved": per_gpu_gbs, "peak": peak, "unit": "GB/s",
                         "frac": sane_frac(per_gpu_gbs / peak, "dist BFS"), "traffic": None,
                         "peak_source": peak_src,
                         "kernel": "gsw k_bfs_push/k_bfs_pull per level (+ NCCL all-gather), per GPU",
                         "bytes_model": "SURVEY 8(d) D0 per-level algorithmic bytes, summed over ranks / N"},
            "gpu_launches": launches_per_level * (levels + 3 * args.steps) + 3 * args.steps,
            "timing": "device span of each gsw_bfs call on the library stream (CUDA events), max over ranks",
            "e2e": {"value": e2e_edges / (e2e_ms * 1e-3) / 1e9, "unit": "GTEPS",
                    "h2d_bytes_per_step": int(h2d_all), "d2h_bytes_per_step": int(d2h_all),
                    "note": "per step, every rank: gsw_graph_create_dist from its pinned host slice (NCCL "
                            "communicator, H2D, column-slice build) + gsw_bfs into pinned host depth (D2H); bytes "
                            "summed over ranks; host wall clock of the slowest rank"},
            "clocks": cs.summary(), "gen_seconds": gen_s, "create_seconds": create_s,
            "extra": {f"{workload}_pr": {"value": 20 / (pr_ms * 1e-3), "unit": "PR iters/s", "gpu_ms": pr_ms,
                                         "achieved_gbs_per_gpu": pr_bytes / (pr_ms * 1e-3) / 1e9,
                                         "bytes_model": "4*nnz_owned + 8*n_owned + 4*N (fp32 all-gather) per "
                                                        "iteration and rank"}},
        }
        print(json.dumps(line), flush=True)
    dist.barrier()
    dist.destroy_process_group()


def run_gsw(args, ws, rank, local):
    import torch
    import torch.distributed as dist
    import gen
    import paper_conf_ppopp_menglts19_b200 as gsw

    if args.partitioned or args.force_dist or (ws > 1 and not args.replicas):
        return run_gsw_dist(args, ws, rank, local)
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    replicas = ws > 1 or args.replicas
    if replicas:
        # N > 1 (default): the BFS roots are independent problems (SURVEY Q12 root stream), so they
        # are sharded over the ranks, each holding its own copy of the graph; no data-path collective
        if "RANK" not in os.environ:
            os.environ.update(RANK="0", WORLD_SIZE="1", LOCAL_RANK="0", MASTER_ADDR="127.0.0.1",
                              MASTER_PORT=str(29500 + os.getpid() % 1000))
        dist.init_process_group("nccl", device_id=dev)
    g, gen_s = build_graph(args.workload)
    deg = g.deg
    nroots = max(64, (args.steps + args.warmup) * ws)
    roots = gen.sources(g, nroots)
    roots = [roots[(k * ws + rank) % nroots] for k in range(nroots)]   # this rank's shard
    G = gsw.Graph(g.off, g.col, device=dev)
    stream = G.stream
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    out = torch.empty(g.n, dtype=torch.int32, device=dev)

    def step(k, timed):
        s = roots[k % nroots]
        flush.fill_(k & 0xff)                     # L2 flush outside the timed span
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        _, st = G.bfs(s, out=out)
        e1.record(stream)
        return e0, e1, st, s

    for k in range(args.warmup):
        step(k, False)
    torch.cuda.synchronize()
    if replicas:
        dist.barrier()
    torch.cuda.synchronize()
    evs, kern_ms, bytes_alg, edges_cc, g500_bytes = [], 0.0, 0, 0, 0
    with ClockSampler(local) as cs:
        for k in range(args.steps):
            e0, e1, st, s = step(args.warmup + k, True)
            evs.append((e0, e1))
            kern_ms += st["gpu_ms"]
            bytes_alg += st["bytes_alg"]
            d = out.cpu().numpy()                             # outside the [e0, e1] span
            mcc = m_cc(deg, d)
            edges_cc += mcc
            g500_bytes += 4 * 2 * mcc + 20 * int((d >= 0).sum())
    torch.cuda.synchronize()
    # The step's device time is the span of the call's device work, measured by the library's CUDA
    # events on its stream (ev0 before the control-block reset, ev1 after the persistent kernel;
    # gsw_run_stats.gpu_ms).  The bench's own events around the synchronous Python call also
    # contain the host round trip of the call (stream sync, stats D2H, Python), reported apart.
    step_ms = [a.elapsed_time(b) for a, b in evs]
    host_ms = sum(step_ms)
    tot_ms = kern_ms
    all_edges = edges_cc
    if replicas:
        t = torch.tensor([tot_ms], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        tot_ms = float(t.item())
        e = torch.tensor([edges_cc], device=dev, dtype=torch.float64)
        dist.all_reduce(e)
        all_edges = float(e.item())
    value = all_edges / (tot_ms * 1e-3) / 1e9

    # ---- roofline of the dominant kernel (the persistent BFS kernel; one launch per step)
    peak, peak_src = hbm_peak()
    achieved = bytes_alg / (kern_ms * 1e-3) / 1e9
    # Graph500-equivalent bytes (full top-down): 4*nnz_cc + 20*N_cc per root (context only)
    g500 = g500_bytes / (kern_ms * 1e-3) / 1e9
    traffic = None
    tf = os.path.join(ROOT, "profiles", "bfs_c3_traffic.json")
    if os.path.exists(tf):
        with open(tf) as f:
            traffic = json.load(f).get("dram_bytes_per_launch")
    extra = (run_extras(gsw, dev, G, g, peak, cpu=not args.no_cpu_baseline)
             if (rank == 0 and ws == 1 and not args.quick and args.workload == "C3") else None)
    if extra is not None and not args.no_c5:
        extra["C5"] = run_c5_extra(gsw, dev, peak)

    # ---- e2e: through the public API from pinned host buffers (graph H2D + BFS + depth D2H)
    e2e = None
    if rank == 0 or ws > 1:
        pin_off = torch.from_numpy(g.off).pin_memory()
        pin_col = torch.from_numpy(g.col).pin_memory()
        host_out = torch.empty(g.n, dtype=torch.int32).pin_memory()
        del G
        torch.cuda.synchronize()
        ke = min(args.steps, 8 if args.workload == "C3" else 2)
        e2e_ms, e2e_edges = 0.0, 0
        for k in range(ke + 1):
            s = roots[k % nroots]
            t0 = time.perf_counter()
            G2 = gsw.Graph(pin_off, pin_col, device=dev)
            G2.bfs(s, out=host_out)
            dt = time.perf_counter() - t0
            if k > 0:                              # first iteration warms the allocator
                e2e_ms += dt * 1e3
                e2e_edges += m_cc(deg, host_out.numpy())
            del G2
        if replicas:                               # whole job: all ranks' edges over the slowest rank
            t = torch.tensor([e2e_ms, float(e2e_edges)], device=dev, dtype=torch.float64)
            mx = t.clone()
            dist.all_reduce(mx, op=dist.ReduceOp.MAX)
            dist.all_reduce(t)
            e2e_ms, e2e_edges = float(mx[0].item()), float(t[1].item())
        e2e = {"value": e2e_edges / (e2e_ms * 1e-3) / 1e9, "unit": "GTEPS",
               "h2d_bytes_per_step": int(g.off.nbytes + g.col.nbytes), "d2h_bytes_per_step": int(g.n * 4),
               "note": "per step: gsw_graph_create from pinned host CSR (H2D) + gsw_bfs into pinned host "
                       "depth (D2H); host wall clock"}

    if rank == 0:
        line = {
            "metric": "BFS GTEPS", "value": value, "unit": "GTEPS", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": tot_ms / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "config": {"workload": workload_label(args.workload, g), "csr_hash": csr_hash(g)},
            "selector": "autotuned (hand-set rules, DESIGN.md R13)",
            "l2": "flushed between steps (256 MiB write outside the timed span)",
            "parallelism": (f"root-sharded replicas x{ws} (one graph copy per GPU, no collective)"
                            if replicas else "single GPU"),
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": sane_frac(achieved / peak, "BFS"), "traffic": traffic, "peak_source": peak_src,
                         "kernel": "gsw::bfs_kernel (persistent, 1 launch/step)",
                         "bytes_model": "SURVEY 8(d) D0 per-level algorithmic bytes of the executed variant",
                         "alg_bytes_per_launch": bytes_alg / args.steps,
                         "traffic_unit": "DRAM bytes per launch (profiles/bfs_c3_traffic.json, ncu --set full)",
                         "graph500_equiv": {"achieved": g500, "frac": g500 / peak,
                                            "bytes_model": "4*nnz_cc + 20*N_cc per root (context)"}},
            "gpu_launches": args.steps,
            "timing": "device span of each gsw_bfs call (library CUDA events on its stream: control-block "
                      "reset + persistent kernel), summed over the timed steps; max over ranks",
            "host_inclusive_ms_per_step": host_ms / args.steps,
            "e2e": e2e,
            "clocks": cs.summary(),
            "gen_seconds": gen_s,
            "extra": extra,
        }
        if not args.no_cpu_baseline and ws == 1:
            line["cpu_baseline"] = cpu_baseline_sample(g, roots[:8 if args.workload == "C3" else 1])
        print(json.dumps(line), flush=True)
    if replicas:
        dist.barrier()
        dist.destroy_process_group()


def main():
    # NCCL writes its banner (NCCL_DEBUG=VERSION, set in this image) and debug log to stdout;
    # keep stdout for the one JSON line
    if os.environ.get("NCCL_DEBUG", "").upper() == "VERSION":
        os.environ.pop("NCCL_DEBUG")
    elif os.environ.get("NCCL_DEBUG") and not os.environ.get("NCCL_DEBUG_FILE"):
        os.environ["NCCL_DEBUG_FILE"] = "/dev/stderr"
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=32)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="gsw", choices=["gsw", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-c5", action="store_true", help="skip the C5 (scale 26) single-GPU / p=1 extra")
    ap.add_argument("--quick", action="store_true", help="headline only (skip the other configs)")
    ap.add_argument("--workload", default="C3", choices=["C3", "C5"],
                    help="C3 (default, the north_star's headline) or C5 (R-MAT scale 26, 1 GPU)")
    ap.add_argument("--force-dist", action="store_true", help="run the partitioned NCCL path even at N=1")
    ap.add_argument("--partitioned", action="store_true",
                    help="the 1D vertex-partitioned graph with NCCL exchange (SURVEY 8(e)); default for N > 1")
    ap.add_argument("--exchange", default="nccl", choices=["nccl", "host"],
                    help="partitioned path: NCCL (one GPU per rank) or the host-staged backend over gloo with every "
                         "rank on GPU 0 (exercises the N > 1 code on one GPU; not a performance number)")
    ap.add_argument("--replicas", action="store_true",
                    help="N > 1: root-sharded replicas of C3 instead of the partitioned C5 (or exercise them at N=1)")
    args = ap.parse_args()
    args.dist_workload_forced = "--workload" in sys.argv
    if args.warmup < 3:
        args.warmup = 3
    ws, rank, local = dist_env()
    if args.impl == "reference":
        run_reference(args, ws, rank)
    else:
        run_gsw(args, ws, rank, local)


if __name__ == "__main__":
    main()
