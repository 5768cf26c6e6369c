"""C5 single-GPU BFS (2 roots, L2 flushed, best of 2) -- for residency A/B on the big graph."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_ppopp_menglts19_b200 as gsw  # noqa: E402

g = gen.config_graph("C5")
G = gsw.Graph(g.off, g.col)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
deg = g.deg
out = torch.empty(g.n, dtype=torch.int32, device="cuda")
for s in gen.sources(g, 2):
    best = None
    for r in range(2):
        flush.fill_(r)
        torch.cuda.synchronize()
        _, st = G.bfs(s, out=out)
        best = st if best is None or st["gpu_ms"] < best["gpu_ms"] else best
    m = int(deg[out.cpu().numpy() >= 0].sum()) // 2
    print(f"C5 root {s}: {best['gpu_ms']:.3f} ms  {m / best['gpu_ms'] / 1e6:.1f} GTEPS  levels {best['iterations']}", flush=True)
