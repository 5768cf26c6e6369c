#!/usr/bin/env python
"""Hot SASS instructions of an ncu --set full --import-source capture by warp-stall samples, and the
kernel's stall-reason totals: python tools/ncu_hotspots.py gpurun_out/x.ncu-rep [N]"""
import csv
import io
import subprocess
import sys
from collections import Counter

rep = sys.argv[1]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 25
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
hdr_i = next(i for i, r in enumerate(rows) if "Warp Stall Sampling (All Samples)" in r)
h = rows[hdr_i]
col = {c: i for i, c in enumerate(h)}
samp = col["Warp Stall Sampling (All Samples)"]
stalls = [c for c in h if c.startswith("stall_")]
tot_st = Counter()
out = []
for r in rows[hdr_i + 1:]:
    if len(r) != len(h):
        continue
    try:
        v = float(r[samp] or 0)
    except ValueError:
        continue
    st = {}
    for c in stalls:
        try:
            x = float(r[col[c]] or 0)
        except ValueError:
            x = 0.0
        st[c] = x
        tot_st[c] += x
    top = sorted(st.items(), key=lambda kv: -kv[1])[:2]
    out.append((v, r[col["Address"]][-5:], r[col["Source"]].strip()[:60], top))
tot = sum(v for v, *_ in out) or 1.0
print(f"total stall samples {tot:.0f}")
print("stall reasons: " + ", ".join(f"{k[6:]} {100 * v / max(1, sum(tot_st.values())):.1f}%"
                                     for k, v in tot_st.most_common(8)))
for v, a, s, top in sorted(out, key=lambda x: -x[0])[:N]:
    print(f"{100 * v / tot:5.1f}%  {a}  {s:<60} " + " ".join(f"{k[6:]}={int(x)}" for k, x in top if x))
