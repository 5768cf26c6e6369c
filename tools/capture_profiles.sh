#!/bin/bash
# Run on the GPU box (gpurun): launch lists + one --set full capture per hot kernel.
set -x
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_bench.csv \
    python bench.py --steps 8 --warmup 3 --quick --no-cpu-baseline > gpurun_out/launches_bench.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:bfs_kernel -s 3 -c 1 -o gpurun_out/bfs_c3_full \
    python bench.py --steps 1 --warmup 3 --quick --no-cpu-baseline > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:pr_ -s 1 -c 1 -o gpurun_out/pr_c3_full \
    python tools/prof_one.py pr C3 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:sssp_kernel -s 1 -c 1 -o gpurun_out/sssp_c2_full \
    python tools/prof_one.py sssp C2 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:bfs_kernel -s 1 -c 1 -o gpurun_out/bfs_c2_full \
    python tools/prof_one.py bfs C2 > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -c 1200 --csv --log-file gpurun_out/launches_dpr_c3.csv \
    python tools/prof_one.py dpr C3 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_dpr_pull -s 5 -c 1 -o gpurun_out/dpr_pull_c3_full \
    python tools/prof_one.py dpr C3 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_dpr_push -s 5 -c 1 -o gpurun_out/dpr_push_c3_full \
    python tools/prof_one.py dpr C3 direction=push > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:k_dpr_filter -s 5 -c 1 -o gpurun_out/dpr_filter_c3_full \
    python tools/prof_one.py dpr C3 > /dev/null 2>&1
ls -la gpurun_out
