#!/usr/bin/env python
"""Summarise gpurun_out/ ncu captures into profiles/ (committed evidence):
  profiles/<tag>_launches.csv      the launch list of `bench.py` (gpu__time_duration per launch)
  profiles/<tag>_launch_shares.md  time share per kernel of that list
  profiles/<tag>_<kernel>.md       key --set full metrics per captured kernel
  profiles/bfs_c3_traffic.json     DRAM bytes per bfs_kernel launch (read by bench.py as `traffic`)
"""
import csv
import io
import json
import os
import shutil
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")
TAG = sys.argv[1] if len(sys.argv) > 1 else "r1"

METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput % of peak"),
    ("lts__t_sector_hit_rate.pct", "L2 hit rate"),
    ("l1tex__t_sector_hit_rate.pct", "L1 hit rate"),
    ("lts__t_sectors_op_read.sum", "L2 read sectors"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM throughput %"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("smsp__warp_issue_stalled_long_scoreboard_per_warp_active.pct", "stall: long scoreboard %"),
    ("smsp__warp_issue_stalled_barrier_per_warp_active.pct", "stall: CTA barrier %"),
    ("smsp__warp_issue_stalled_lg_throttle_per_warp_active.pct", "stall: LG throttle %"),
]


def raw(rep):
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    if len(rows) < 3:
        return {}, {}
    h, units, v = rows[0], rows[1], rows[2]
    return {k: v[i] for i, k in enumerate(h)}, {k: units[i] for i, k in enumerate(h)}


def bytes_of(val, unit):
    x = float(val.replace(",", ""))
    return x * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(unit, 1)


def main():
    os.makedirs(PROF, exist_ok=True)
    lst = os.path.join(OUT, "launches_bench.csv")
    if os.path.exists(lst):
        shutil.copy(lst, os.path.join(PROF, f"{TAG}_launches.csv"))
        agg = defaultdict(lambda: [0, 0.0])
        for r in csv.reader(open(lst)):
            if len(r) > 14 and r[0] != "ID" and r[12] == "gpu__time_duration.sum":
                k = r[4].split("(")[0]
                agg[k][0] += 1
                agg[k][1] += float(r[14].replace(",", ""))
        tot = sum(v[1] for v in agg.values())
        with open(os.path.join(PROF, f"{TAG}_launch_shares.md"), "w") as f:
            f.write(f"# Launch list of `bench.py --steps 8 --warmup 3 --quick` under ncu ({TAG})\n\n")
            f.write("Cold-cache, serialised replay: compare shares, not absolute times. Graph creation "
                    "(gsw_graph_create: offsets, attributes) runs once before the timed steps.\n\n")
            f.write("| kernel | launches | total us | share |\n|---|---|---|---|\n")
            for k, (n, ns) in sorted(agg.items(), key=lambda x: -x[1][1]):
                f.write(f"| `{k}` | {n} | {ns / 1e3:.1f} | {ns / tot * 100:.1f}% |\n")
            # the timed region of a step holds exactly one persistent-kernel launch (the L2 flush
            # runs before the start event); everything else is graph creation (warm-up, e2e leg)
            bfs = [(k, v) for k, v in agg.items() if "bfs_kernel" in k]
            if bfs:
                k, (n, ns) = bfs[0]
                f.write(f"\n**Timed region of a step** (between the CUDA events): one `{k}` launch = 100% of the "
                        f"step's device work; under ncu its mean duration is {ns / n / 1e3:.1f} us per launch "
                        f"({n} launches: warm-up + timed steps + e2e leg).\n")
    for rep, kernel in [("bfs_c3_full", "bfs_kernel"), ("pr_c3_full", "pr_kernel"), ("sssp_c2_full", "sssp_kernel"),
                        ("bfs_c2_full", "bfs_kernel_c2"), ("dpr_pull_c3_full", "dpr_pull"),
                        ("dpr_push_c3_full", "dpr_push"), ("dpr_filter_c3_full", "dpr_filter")]:
        path = os.path.join(OUT, rep + ".ncu-rep")
        if not os.path.exists(path):
            continue
        vals, units = raw(path)
        with open(os.path.join(PROF, f"{TAG}_{kernel}.md"), "w") as f:
            f.write(f"# ncu --set full: `{kernel}` ({rep}, one launch, {TAG})\n\n| metric | value | unit |\n|---|---|---|\n")
            for m, name in METRICS:
                if m in vals:
                    f.write(f"| {name} (`{m}`) | {vals[m]} | {units.get(m, '')} |\n")
        if kernel == "bfs_kernel" and "dram__bytes_read.sum" in vals:
            rd = bytes_of(vals["dram__bytes_read.sum"], units["dram__bytes_read.sum"])
            wr = bytes_of(vals["dram__bytes_write.sum"], units["dram__bytes_write.sum"])
            dur = float(vals["gpu__time_duration.sum"].replace(",", ""))
            json.dump({"dram_bytes_per_launch": rd + wr, "dram_read": rd, "dram_write": wr,
                       "duration": dur, "duration_unit": units["gpu__time_duration.sum"],
                       "source": f"profiles/{TAG}_bfs_kernel.md (ncu --set full, one C3 BFS launch)"},
                      open(os.path.join(PROF, "bfs_c3_traffic.json"), "w"), indent=1)
    print(open(os.path.join(PROF, f"{TAG}_launch_shares.md")).read() if os.path.exists(lst) else "")


if __name__ == "__main__":
    main()
