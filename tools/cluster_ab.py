#!/usr/bin/env python
"""A/B of the grid shape of the latency-bound level loops on the road grid C2 (DESIGN.md 2,
VERDICT r1 item 7): the default cooperative grid (software flip-bit barrier) vs a reduced grid
(GSW_GRID_CTAS=k, same barrier) vs ONE k-CTA thread-block cluster (GSW_CLUSTER=k, hardware
barrier.cluster).  Results must stay bit-identical to the default run.

    python tools/cluster_ab.py [C2] [C1] ...
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import gen
import paper_conf_ppopp_menglts19_b200 as gsw

VARIANTS = [("team_off", {"GSW_TEAM": "0"}),
            ("default", {}),
            ("team8", {"GSW_TEAM": "8"}),
            ("team4", {"GSW_TEAM": "4"}),
            ("team16_e4096", {"GSW_TEAM_E": "4096"}),
            ("team_off_grid16", {"GSW_TEAM": "0", "GSW_GRID_CTAS": "16"}),
            ("team_off_cluster16", {"GSW_TEAM": "0", "GSW_CLUSTER": "16"})]
KEYS = ("GSW_GRID_CTAS", "GSW_CLUSTER", "GSW_SOLO_E", "GSW_TEAM", "GSW_TEAM_E")


def run(label, fn, reps=3):
    best = None
    for _ in range(reps):
        out, st = fn()
        if best is None or st["gpu_ms"] < best[1]["gpu_ms"]:
            best = (out.cpu().numpy(), st)
    return best


def main():
    which = sys.argv[1:] or ["C2"]
    for cfg in which:
        g = gen.config_graph(cfg)
        weighted = cfg == "C2"
        G = gsw.Graph(g.off, g.col, g.w if weighted else None)
        src = 0 if cfg == "C2" else int(gen.sources(g, 1)[0])
        algos = [("bfs", lambda: G.bfs(src, records=1 << 15))]
        if weighted:
            algos.append(("sssp", lambda: G.sssp(src, records=1 << 15)))
        for name, fn in algos:
            ref = None
            for label, env in VARIANTS:
                for k in KEYS:
                    os.environ.pop(k, None)
                os.environ.update(env)
                try:
                    out, st = run(label, fn)
                except Exception as e:  # noqa: BLE001 - report and continue the sweep
                    print(f"{cfg} {name:5s} {label:18s} FAILED: {e}", flush=True)
                    continue
                if ref is None:
                    ref = out
                same = bool(np.array_equal(out, ref))
                recs = st.get("records", [])
                ct = [x.get("ctas", 0) for x in recs]
                print(f"{cfg} {name:5s} {label:18s} {st['gpu_ms']:9.3f} ms  iters={st['iterations']:6d}  "
                      f"grid={max(ct) if ct else 0} team_levels={sum(1 for c in ct if 1 < c <= 16)} "
                      f"us/iter={st['gpu_ms'] * 1e3 / max(1, st['iterations']):6.2f}  identical={same}", flush=True)
        for k in KEYS:
            os.environ.pop(k, None)
        del G


if __name__ == "__main__":
    main()
