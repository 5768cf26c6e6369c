"""A/B of the PageRank paths on one config: the edge-tiled stream kernel at several shared-memory
hub-cache sizes (entries; the rest of the 256 KB L1/smem array is L1 for the gathers) and the
row-tier kernel (pr_blocked.cu, B source blocks).  Device time of 20 iterations, best of 3.
  python tools/pr_ab.py C3 [caches...]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402
import paper_conf_ppopp_menglts19_b200 as gsw  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
caches = sys.argv[2:] or ["0", "8192", "12288", "16384", "20480", "24576", "28672", "32768", "40960", "1000000"]
g = gen.config_graph(cfg)
G = gsw.Graph(g.off, g.col)


def run(tag, env):
    for k in ("GSW_PR_CACHE", "GSW_PR_BLOCKED", "GSW_PR_BLOCKS"):
        os.environ.pop(k, None)
    os.environ.update(env)
    best = min(G.pr(0.85, 20)[1]["gpu_ms"] for _ in range(3))
    print(f"{cfg} {tag:28s} {best:9.3f} ms  {20 / best * 1e3:8.1f} it/s", flush=True)


run("AUTO", {})
for k in caches:
    run(f"stream cache={k}", {"GSW_PR_CACHE": k, "GSW_PR_BLOCKED": "0"})
run("row tiers B=1", {"GSW_PR_BLOCKED": "1", "GSW_PR_BLOCKS": "1"})
