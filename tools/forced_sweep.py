#!/usr/bin/env python
"""Autotuned vs every forced variant (north_star: "the autotuned path beats the best single forced
variant on both scale-free and road-grid inputs").

Each (algorithm, config) is run with the selector (AUTO) and with every valid forced
(direction, format, LB, fusion[, stepping]) combination pinned for all iterations
(gsw_force_config).  Device time per call from the library's CUDA events, L2
flushed (256 MiB write) before every call, median of --reps calls per root, summed over roots.

  python tools/forced_sweep.py [--json profiles/r1_forced_sweep.json] [--only C3:bfs,C2:sssp]
"""
import argparse
import itertools
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

DIRS = ["push", "pull"]
FMTS = ["bitmap", "queue", "sorted_queue"]
LBS = ["thread", "twc", "wm", "cm", "strict"]
FUS = ["standalone", "fused"]
STEPS = ["increase", "decrease", "remain", "static", "unordered"]

JOBS = {
    "C3:bfs": ("C3", "bfs", 4),
    "C1:bfs": ("C1", "bfs", 8),
    "C2:sssp": ("C2", "sssp", 1),
    "C3:sssp": ("C3w", "sssp", 1),
    "C3:cc": ("C3", "cc", 1),
    "C2:bfs": ("C2", "bfs", 1),
}


def variants(algo):
    yield None
    if algo == "sssp":
        # a forced SSSP variant pins the per-round stepping decision too (P4 candidates
        # Increase / Decrease / Remain, plus static delta-stepping and Bellman-Ford)
        for v in itertools.product(DIRS, FMTS, LBS, FUS, STEPS):
            yield dict(direction=v[0], format=v[1], load_balance=v[2], fusion=v[3], stepping=v[4])
    elif algo in ("bfs", "cc"):
        for v in itertools.product(DIRS, FMTS, LBS, FUS):
            yield dict(direction=v[0], format=v[1], load_balance=v[2], fusion=v[3])
    else:
        for v in itertools.product(DIRS, LBS):
            yield dict(direction=v[0], load_balance=v[1])


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--json", default=None)
    ap.add_argument("--merge", action="store_true", help="update an existing --json file job by job")
    ap.add_argument("--only", default=",".join(["C3:bfs", "C1:bfs", "C2:sssp", "C3:cc"]))
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--sssp-reps", type=int, default=2)
    ap.add_argument("--budget-ms", type=float, default=3000.0,
                    help="skip the remaining reps/roots of a variant slower than this")
    a = ap.parse_args()
    import torch
    import gen
    import paper_conf_ppopp_menglts19_b200 as gsw
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    results = {}
    cache = {}
    for job in a.only.split(","):
        cfg, algo, nroots = JOBS[job]
        if cfg not in cache:
            cache.clear()
            torch.cuda.empty_cache()
            g = gen.with_hash_weights(gen.config_graph("C3")) if cfg == "C3w" else gen.config_graph(cfg)
            G = gsw.Graph(g.off, g.col, g.w) if g.w is not None else gsw.Graph(g.off, g.col)
            cache[cfg] = (g, G)
        g, G = cache[cfg]
        roots = gen.sources(g, nroots) if algo in ("bfs", "sssp") else [None]
        if algo == "sssp" and cfg == "C2":
            roots = [0]

        # warm-up: the first call after graph creation (module load, allocator, clocks) is not timed
        G.force_config()
        for s in roots:
            (G.bfs(s) if algo == "bfs" else G.sssp(s)) if algo in ("bfs", "sssp") else G.cc()
        torch.cuda.synchronize()
        rows = {}
        t_job = time.time()
        for v in variants(algo):
            name = "AUTO" if v is None else "-".join(str(x) for x in v.values())
            G.force_config(**(v or {}))
            tot = 0.0
            for s in roots:
                ms = []
                for r in range(a.sssp_reps if algo == "sssp" else a.reps):
                    flush.fill_(r)
                    torch.cuda.synchronize()
                    if algo == "bfs":
                        st = G.bfs(s)[1]
                    elif algo == "sssp":
                        st = G.sssp(s)[1]
                    elif algo == "cc":
                        st = G.cc()[1]
                    ms.append(st["gpu_ms"])
                    if st["gpu_ms"] > a.budget_ms:
                        break
                tot += statistics.median(ms)
            rows[name] = tot
            print(f"{job:8s} {name:40s} {tot:10.3f} ms", flush=True)
        G.force_config()
        forced = {k: v for k, v in rows.items() if k != "AUTO"}
        bk = min(forced, key=forced.get)
        results[job] = {"graph": cfg, "algo": algo, "roots": [int(r) for r in roots if r is not None],
                        "auto_ms": rows["AUTO"], "best_forced": bk, "best_forced_ms": forced[bk],
                        "auto_over_best": rows["AUTO"] / forced[bk], "auto_beats_best": rows["AUTO"] < forced[bk],
                        "n_forced": len(forced), "sweep_s": time.time() - t_job, "all_ms": rows}
        print(f"== {job}: AUTO {rows['AUTO']:.3f} ms, best forced {bk} {forced[bk]:.3f} ms "
              f"(ratio {rows['AUTO'] / forced[bk]:.3f})", flush=True)
    if a.json:
        if a.merge and os.path.exists(a.json):
            old = json.load(open(a.json))
            old.update(results)
            results = old
        with open(a.json, "w") as f:
            json.dump(results, f, indent=1)


if __name__ == "__main__":
    main()
