#!/usr/bin/env python
"""Device time of every algorithm on its BASELINE.json config (autotuned), with per-iteration
records summarised.  Diagnostic companion of bench.py (which reports the headline line)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import gen
import paper_conf_ppopp_menglts19_b200 as gsw


def best(fn, reps=3):
    b = None
    for _ in range(reps):
        r = fn()
        if b is None or r[1]["gpu_ms"] < b[1]["gpu_ms"]:
            b = r
    return b


def summarize(name, st, extra=""):
    recs = st.get("records", [])
    cfgs = {}
    for r in recs:
        k = (r["direction"], r["format"], r["load_balance"], r["fusion"])
        cfgs[k] = cfgs.get(k, 0) + 1
    print(f"{name:28s} {st['gpu_ms']:9.3f} ms  iters={st['iterations']:6d}  GB/s(alg)={st['bytes_alg'] / st['gpu_ms'] / 1e6:8.1f} "
          f"{extra}  cfgs={dict(list(cfgs.items())[:6])}", flush=True)


def main():
    which = sys.argv[1:] or ["C3", "C2", "C4"]
    if "C3" in which:
        g = gen.config_graph("C3")
        G = gsw.Graph(g.off, g.col)
        roots = gen.sources(g, 8)
        tot_ms, tot_e = 0.0, 0
        for s in roots:
            d, st = best(lambda: G.bfs(s, records=64))
            dd = d.cpu().numpy()
            m = int(g.deg[dd >= 0].sum()) // 2
            tot_ms += st["gpu_ms"]; tot_e += m
        summarize("C3 BFS (8 roots, last)", st, f"GTEPS={tot_e / tot_ms / 1e6:.1f} avg_ms={tot_ms / len(roots):.3f}")
        _, st = best(lambda: G.cc(records=256))
        summarize("C3 CC", st, f"GTEPS={g.nnz / 2 / st['gpu_ms'] / 1e6:.1f}")
        _, st = best(lambda: G.pr(0.85, 20, records=64))
        summarize("C3 PR x20", st, f"iters/s={20 / st['gpu_ms'] * 1e3:.0f}")
        for lb in ["thread", "twc", "wm", "cm", "strict"]:
            for d in ["pull", "push"]:
                G.force_config(direction=d, load_balance=lb)
                _, st = best(lambda: G.pr(0.85, 20), 2)
                summarize(f"  PR {d}-{lb}", st, f"iters/s={20 / st['gpu_ms'] * 1e3:.0f}")
        G.force_config()
        del G
    if "C2" in which:
        g = gen.config_graph("C2")
        G = gsw.Graph(g.off, g.col, g.w)
        for step in ["auto", "static", "unordered"]:
            for fus in ["auto", "fused", "standalone"]:
                G.force_config(stepping=step, fusion=fus)
                d, st = best(lambda: G.sssp(0, records=1 << 15), 2)
                summarize(f"C2 SSSP {step}/{fus}", st, f"GTEPS={g.nnz / 2 / st['gpu_ms'] / 1e6:.2f}")
        G.force_config()
        _, st = best(lambda: G.bfs(0, records=8192), 2)
        summarize("C2 BFS", st, "")
        del G
    if "C4" in which:
        g = gen.config_graph("C4")
        G = gsw.Graph(g.off, g.col)
        srcs = gen.sources(g, 16)
        _, st = best(lambda: G.bc(srcs, records=4096), 2)
        summarize("C4 BC x16", st, f"GTEPS={16 * g.nnz / 2 / st['gpu_ms'] / 1e6:.1f}")


if __name__ == "__main__":
    main()
