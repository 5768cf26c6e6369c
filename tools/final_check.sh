#!/bin/bash
# One gpurun call at the end of a session: GPU parity suite, smoke, the bench line, and ncu
# --set full captures of the BC and CC kernels (the BFS one is in tools/capture_profiles.sh).
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q --durations=10 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as e; e.smoke()" > gpurun_out/smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 600 ncu --set full --clock-control none --import-source on -k regex:bc_kernel -s 1 -c 1 -o gpurun_out/bc_c4_full \
    python tools/prof_one.py bc C4 > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:cc_kernel -s 1 -c 1 -o gpurun_out/cc_c3_full \
    python tools/prof_one.py cc C3 > /dev/null 2>&1
tail -3 gpurun_out/pytest_gpu.log; cat gpurun_out/smoke.log; tail -c 600 gpurun_out/bench.json; ls -la gpurun_out
