#!/usr/bin/env python
"""Per-level breakdown of C3 BFS (autotuned and forced push/pull), for a few roots:
config chosen, Va, Ea, Via, Eia, edges scanned, Filter/Expand microseconds."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen
import paper_conf_ppopp_menglts19_b200 as gsw

cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
nroots = int(sys.argv[2]) if len(sys.argv) > 2 else 3
g = gen.config_graph(cfg)
G = gsw.Graph(g.off, g.col)
roots = gen.sources(g, nroots)
D = {v: k for k, v in gsw.DIRECTIONS.items()}
L = {v: k for k, v in gsw.LOAD_BALANCES.items()}
F = {v: k for k, v in gsw.FORMATS.items()}
U = {v: k for k, v in gsw.FUSIONS.items()}
forces = [dict()] if (len(sys.argv) > 3 and sys.argv[3] == 'auto') else [dict(), dict(direction="push"), dict(direction="pull")]
for force in forces:
    G.force_config(**force)
    for s in roots:
        best = None
        for _ in range(3):
            _, st = G.bfs(s, records=64)
            best = st if best is None or st["gpu_ms"] < best["gpu_ms"] else best
        print(f"force={force} root={s} gpu_ms={best['gpu_ms']:.4f} levels={best['iterations']} "
              f"bytes_alg={best['bytes_alg']}", flush=True)
        for r in best["records"]:
            print(f"   it={r['iteration']:2d} {D.get(r['direction'])}/{F.get(r['format'])}/"
                  f"{L.get(r['load_balance'])}/{U.get(r['fusion'])} Va={r['Va']:8d} Ea={r['Ea']:10d} "
                  f"Via={r['Via']:8d} Eia={r['Eia']:10d} edges={r['edges']:10d} "
                  f"filter_us={r['filter_us']:7.2f} expand_us={r['expand_us']:7.2f}", flush=True)
G.force_config()
