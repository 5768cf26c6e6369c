#!/usr/bin/env python
"""C5 (BASELINE.json config 5) on ONE B200: Kronecker/R-MAT scale 26, edge factor 16
(67,108,864 vertices, ~2.1e9 directed CSR entries), BFS from the SURVEY Q12 roots and PageRank
(20 iterations, d = 0.85) through the C ABI, checked against the CPU oracle at full size:
BFS depths bit-exact, PR max relative error <= 1e-5 (R10).  Device times from the
library's CUDA events, L2 flushed before each call.  Writes one JSON object (stdout and --json).

  python tools/c5_check.py [--roots 2] [--no-pr-oracle] [--json gpurun_out/c5_check.json]
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--roots", type=int, default=2)
    ap.add_argument("--no-pr-oracle", action="store_true")
    ap.add_argument("--json", default=None)
    a = ap.parse_args()
    import torch
    import gen
    import oracle
    import paper_conf_ppopp_menglts19_b200 as gsw

    out = {"config": "C5: R-MAT scale 26 ef 16 (Graph500 a,b,c = .57,.19,.19), symmetrised, deduped, "
                     "loop-free, ids permuted; 1 GPU"}
    t0 = time.time()
    g = gen.config_graph("C5")
    out["gen_s"] = time.time() - t0
    out["n"], out["nnz"] = int(g.n), int(g.nnz)
    out["max_deg"], out["isolated"] = int(g.deg.max()), int((g.deg == 0).sum())
    t0 = time.time()
    G = gsw.Graph(g.off, g.col, device="cuda")
    torch.cuda.synchronize()
    out["ingest_s"] = time.time() - t0
    out["device_mem_gb"] = torch.cuda.memory_allocated() / 1e9
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    roots = gen.sources(g, a.roots)
    bfs = []
    for s in roots:
        G.bfs(s)                                   # warm-up
        flush.fill_(1)
        torch.cuda.synchronize()
        d, st = G.bfs(s)
        got = d.cpu().numpy()
        t0 = time.time()
        ref = oracle.bfs(g, s)
        osec = time.time() - t0
        reached = ref >= 0
        mcc = int(g.deg[reached].sum()) // 2
        bfs.append({"root": int(s), "gpu_ms": st["gpu_ms"], "levels": st["iterations"], "m_cc": mcc,
                    "gteps": mcc / (st["gpu_ms"] * 1e-3) / 1e9, "bytes_alg": st["bytes_alg"],
                    "parity_bit_exact": bool(np.array_equal(got, ref)),
                    "mismatches": int((got != ref).sum()), "oracle_s": osec,
                    "oracle_gteps": mcc / osec / 1e9})
        print(json.dumps(bfs[-1]), flush=True)
    out["bfs"] = bfs
    flush.fill_(2)
    torch.cuda.synchronize()
    x, st = G.pr(0.85, 20)
    pr = {"gpu_ms": st["gpu_ms"], "iters_per_s": 20 / (st["gpu_ms"] * 1e-3), "bytes_alg": st["bytes_alg"],
          "achieved_gbs": st["bytes_alg"] / (st["gpu_ms"] * 1e-3) / 1e9}
    xv = x.cpu().numpy()
    pr["mass"] = float(xv.sum())
    pr["min_over_floor"] = float(xv.min() / ((1 - 0.85) / g.n))
    if not a.no_pr_oracle:
        t0 = time.time()
        r = oracle.pr(g, 0.85, 20)
        pr["oracle_s"] = time.time() - t0
        pr["max_rel_err"] = float((np.abs(xv - r) / r).max())
        pr["parity_1e-5"] = pr["max_rel_err"] <= 1e-5
    out["pr"] = pr
    print(json.dumps(pr), flush=True)
    if a.json:
        with open(a.json, "w") as f:
            json.dump(out, f, indent=1)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
