#!/usr/bin/env python
"""AUTO with the hand-set rules vs AUTO with the learned trees (GSW_SELECTOR=trees) on the
evaluation configs (none of which is in the training corpus): device time per BFS root, L2
flushed before each call, median of 3, summed over roots."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import gen
import paper_conf_ppopp_menglts19_b200 as gsw

flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
out = {}
for cfg, nroots in (("C1", 16), ("C3", 8), ("C2", 1), ("C4", 4)):
    g = gen.config_graph(cfg)
    G = gsw.Graph(g.off, g.col)
    roots = [0] if cfg == "C2" else gen.sources(g, nroots)
    res = {}
    for sel in ("rules", "trees"):
        os.environ["GSW_SELECTOR"] = sel
        tot = 0.0
        for s in roots:
            G.bfs(s)
            ms = []
            for r in range(3):
                flush.fill_(r)
                torch.cuda.synchronize()
                ms.append(G.bfs(s)[1]["gpu_ms"])
            tot += statistics.median(ms)
        res[sel] = tot
    os.environ.pop("GSW_SELECTOR")
    out[cfg] = res
    print(f"{cfg}: rules {res['rules']:.3f} ms  trees {res['trees']:.3f} ms  trees/rules {res['trees'] / res['rules']:.3f}", flush=True)
    del G
if len(sys.argv) > 1:
    json.dump(out, open(sys.argv[1], "w"), indent=1)
