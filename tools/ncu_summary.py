#!/usr/bin/env python
"""Key --set full metrics of one ncu capture as a markdown table:
python tools/ncu_summary.py gpurun_out/x.ncu-rep "title" > profiles/.../x.md"""
import csv
import io
import subprocess
import sys

sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.abspath(__file__)))
from summarize_profiles import METRICS  # noqa: E402

rep, title = sys.argv[1], sys.argv[2]
txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
h, u = rows[0], rows[1]
print(f"# ncu --set full: {title}\n")
for r in rows[2:]:
    print(f"kernel `{r[h.index('Kernel Name')][:90]}`\n")
    print("| metric | value | unit |\n|---|---|---|")
    for k, name in METRICS:
        if k in h:
            print(f"| {name} (`{k}`) | {r[h.index(k)]} | {u[h.index(k)]} |")
    print()
