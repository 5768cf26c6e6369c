#!/usr/bin/env python
"""gpurun_out/forced_sweep.json -> profiles/<tag>_forced_sweep.{json,md} (committed evidence for the
north_star target "the autotuned path beats the best single forced variant")."""
import json
import os
import shutil
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag = sys.argv[1] if len(sys.argv) > 1 else "r1"
src = os.path.join(ROOT, "gpurun_out", "forced_sweep.json")
d = json.load(open(src))
shutil.copy(src, os.path.join(ROOT, "profiles", f"{tag}_forced_sweep.json"))
lines = [f"# Autotuned vs every forced variant ({tag})", "",
         "`tools/forced_sweep.py` on one B200: device time (library CUDA events, L2 flushed before every call), "
         "median of 3 calls per root (SSSP: 1), summed over the roots. A forced variant pins every pattern "
         "(direction, format, LB, fusion; SSSP also stepping) for all iterations (`gsw_force_config`).", "",
         "| job | graph | roots | AUTO ms | best forced variant | its ms | AUTO / best | forced variants |",
         "|---|---|---|---|---|---|---|---|"]
for job, r in d.items():
    lines.append(f"| {job} | {r['graph']} | {len(r['roots']) or '-'} | {r['auto_ms']:.3f} | `{r['best_forced']}` | "
                 f"{r['best_forced_ms']:.3f} | {r['auto_over_best']:.3f} | {r['n_forced']} |")
open(os.path.join(ROOT, "profiles", f"{tag}_forced_sweep.md"), "w").write("\n".join(lines) + "\n")
print("\n".join(lines))
