#!/usr/bin/env python
"""Per-round breakdown (Filter/Expand microseconds, active-set sizes) of one SSSP/BFS run."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import gen
import paper_conf_ppopp_menglts19_b200 as gsw
cfg, algo = sys.argv[1], sys.argv[2]
kw = dict(a.split("=") for a in sys.argv[3:])
g = gen.config_graph(cfg)
G = gsw.Graph(g.off, g.col, g.w) if g.w is not None else gsw.Graph(g.off, g.col)
if kw: G.force_config(**kw)
for _ in range(2):
    _, st = (G.sssp(0, records=1 << 15) if algo == "sssp" else G.bfs(0, records=1 << 15))
r = st["records"]
f = np.array([x["filter_us"] for x in r]); e = np.array([x["expand_us"] for x in r])
va = np.array([x["Va"] for x in r]); ed = np.array([x["edges"] for x in r]); th = np.array([x["theta"] for x in r])
print(f"rounds={len(r)} gpu_ms={st['gpu_ms']:.2f} filter_us mean={f.mean():.2f} expand_us mean={e.mean():.2f} "
      f"Va mean={va.mean():.0f} max={va.max()} edges mean={ed.mean():.0f} theta changes={np.count_nonzero(np.diff(th))}")
for q in (10, 50, 90, 99):
    print(f"  p{q}: filter {np.percentile(f, q):.2f} expand {np.percentile(e, q):.2f} Va {np.percentile(va, q):.0f}")
big = np.argsort(-(f + e))[:5]
for i in big:
    print("  slow round", i, r[i])
ct = np.array([x.get("ctas", 0) for x in r])
for name, m in (("solo (ctas=1)", ct == 1), ("grid", ct != 1)):
    if m.any():
        print(f"  {name}: rounds={m.sum()} filter_us mean={f[m].mean():.2f} expand_us mean={e[m].mean():.2f} "
              f"Va mean={va[m].mean():.0f} edges mean={ed[m].mean():.0f}")
        for lo, hi in ((0, 16), (16, 128), (128, 512), (512, 1024), (1024, 1 << 30)):
            mm = m & (va >= lo) & (va < hi)
            if mm.any():
                print(f"     Va in [{lo},{hi}): n={mm.sum()} us/round={(f[mm] + e[mm]).mean():.2f}")
