#!/usr/bin/env python
"""Calibration of the CTA-resident (solo) tier thresholds: device time of
autotuned BFS / SSSP / CC / BC runs with GSW_SOLO_E / GSW_SOLO_V set per run (0 disables the tier).

  python tools/solo_sweep.py [C2:bfs,C2:sssp,C3:bfs,C1:bfs]
"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import gen
import paper_conf_ppopp_menglts19_b200 as gsw

jobs = (sys.argv[1] if len(sys.argv) > 1 else "C2:bfs,C2:sssp,C3:bfs,C1:bfs").split(",")
SETTINGS = [(0, 0), (512, 256), (1024, 512), (2048, 512), (2048, 1024), (4096, 512), (4096, 768), (8192, 768), (16384, 768)]
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
cache = {}
for job in jobs:
    cfg, algo = job.split(":")
    if cfg not in cache:
        cache.clear()
        g = gen.config_graph(cfg)
        cache[cfg] = (g, gsw.Graph(g.off, g.col, g.w) if g.w is not None else gsw.Graph(g.off, g.col))
    g, G = cache[cfg]
    roots = [0] if cfg == "C2" else gen.sources(g, 4)
    for e, v in SETTINGS:
        os.environ["GSW_SOLO_E"] = str(e)
        os.environ["GSW_SOLO_V"] = str(v)
        tot, solo_it, its = 0.0, 0, 0
        for s in roots:
            ms = []
            for r in range(3):
                flush.fill_(r)
                torch.cuda.synchronize()
                if algo == "bfs":
                    _, st = G.bfs(s, records=1 << 16)
                elif algo == "sssp":
                    _, st = G.sssp(s, records=1 << 16)
                elif algo == "cc":
                    _, st = G.cc(records=1 << 16)
                else:
                    _, st = G.bc(gen.sources(g, 4), records=1 << 16)
                ms.append(st["gpu_ms"])
            tot += statistics.median(ms)
            solo_it += sum(1 for x in st["records"] if x["ctas"] == 1)
            its += st["iterations"]
        print(f"{job:8s} solo_e={e:6d} solo_v={v:6d}  {tot:9.3f} ms  iters={its:6d} solo_iters={solo_it:6d}", flush=True)
os.environ.pop("GSW_SOLO_E", None)
os.environ.pop("GSW_SOLO_V", None)
