#!/usr/bin/env python
"""Per-iteration strategy search table (the methodology of PAPER.md Fig. 14):
run BFS with every forced (direction, format, LB, fusion) variant and with the autotuner, and
print each iteration's device time per variant.  BFS levels are unique, so iteration t processes
the same active set under every variant and the per-iteration times are comparable.

  python tools/strategy_table.py --graph C3 --roots 2 [--json out.json]
"""
import argparse
import itertools
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--graph", default="C3")
    ap.add_argument("--roots", type=int, default=1)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--json", default=None)
    ap.add_argument("--algo", default="bfs")
    a = ap.parse_args()
    import torch
    import gen
    import paper_conf_ppopp_menglts19_b200 as gsw
    g = gen.config_graph(a.graph)
    G = gsw.Graph(g.off, g.col, g.w) if g.w is not None else gsw.Graph(g.off, g.col)
    roots = gen.sources(g, a.roots)
    variants = [None] + list(itertools.product(["push", "pull"], ["bitmap", "queue", "sorted_queue"],
                                               ["thread", "twc", "wm", "cm", "strict"], ["standalone", "fused"]))
    out = {}
    for v in variants:
        if v is None:
            G.force_config()
            name = "AUTO"
        else:
            G.force_config(direction=v[0], format=v[1], load_balance=v[2], fusion=v[3])
            name = "-".join(v)
        runs = []
        for s in roots:
            best = None
            for _ in range(a.reps):
                _, st = G.bfs(s, records=4096)
                if best is None or st["gpu_ms"] < best["gpu_ms"]:
                    best = st
            runs.append({"root": s, "gpu_ms": best["gpu_ms"],
                         "iters": [{"t": r["iteration"], "Va": r["Va"], "Ea": r["Ea"], "Eia": r["Eia"],
                                    "edges": r["edges"], "cfg": [r["direction"], r["format"], r["load_balance"],
                                                                 r["fusion"]],
                                    "us": r["filter_us"] + r["expand_us"]} for r in best["records"]]})
        out[name] = runs
        tot = sum(r["gpu_ms"] for r in runs)
        per = " ".join(f"{it['us']:8.1f}" for it in runs[0]["iters"])
        print(f"{name:32s} total {tot:8.3f} ms | {per}", flush=True)
    # best fixed vs per-iteration oracle
    fixed = {k: sum(r["gpu_ms"] for r in v) for k, v in out.items() if k != "AUTO"}
    bk = min(fixed, key=fixed.get)
    print(f"best fixed: {bk} {fixed[bk]:.3f} ms ; AUTO {sum(r['gpu_ms'] for r in out['AUTO']):.3f} ms")
    L = len(out["AUTO"][0]["iters"])
    for t in range(L):
        cand = {k: v[0]["iters"][t]["us"] for k, v in out.items() if k != "AUTO" and len(v[0]["iters"]) > t}
        kb = min(cand, key=cand.get)
        it = out["AUTO"][0]["iters"][t]
        print(f"  iter {t}: Va={it['Va']} Ea={it['Ea']} Eia={it['Eia']} auto={it['us']:.1f}us cfg={it['cfg']} "
              f"best={kb} {cand[kb]:.1f}us")
    if a.json:
        with open(a.json, "w") as f:
            json.dump(out, f)


if __name__ == "__main__":
    main()
