#!/usr/bin/env python
"""Delta-PR on a config graph: autotuned vs forced push / pull, best of 3; per-iteration records."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen
import paper_conf_ppopp_menglts19_b200 as gsw
g = gen.config_graph(sys.argv[1] if len(sys.argv) > 1 else "C3")
tol = float(sys.argv[2]) if len(sys.argv) > 2 else 1e-6
G = gsw.Graph(g.off, g.col)
out = {}
for name, cfg in [("auto", dict()), ("push", dict(direction="push")), ("pull", dict(direction="pull"))]:
    G.force_config(**cfg)
    G.dpr(0.85, tol)
    best = min((G.dpr(0.85, tol, records=4096)[1] for _ in range(3)), key=lambda s: s["gpu_ms"])
    out[name] = dict(ms=best["gpu_ms"], iters=best["iterations"], edges=best["edges_touched"],
                     alg_gbs=best["bytes_alg"] / best["gpu_ms"] / 1e6,
                     dirs="".join("P" if r["direction"] == 2 else "p" for r in best["records"]),
                     va=[r["Va"] for r in best["records"]][:40])
    print(name, json.dumps({k: v for k, v in out[name].items() if k != "va"}), flush=True)
print(json.dumps(out))
