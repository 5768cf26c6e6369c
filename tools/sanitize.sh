#!/bin/bash
# compute-sanitizer over every libgsw kernel: memcheck, racecheck, initcheck
# and synccheck on the tools/sanitize_run.py workload; logs -> gpurun_out/sanitize_<tool>.log.
# Usage (on the GPU box): bash tools/sanitize.sh [small|c1]
set -u
SIZE=${1:-small}
CS=/usr/local/cuda/bin/compute-sanitizer
mkdir -p gpurun_out
for tool in memcheck racecheck initcheck synccheck; do
  sz=$SIZE
  [ "$tool" = racecheck ] && sz=small     # racecheck serialises shared-memory accesses: small graphs
  extra=""
  [ "$tool" = memcheck ] && extra="--leak-check full"
  echo "== $tool ($sz)"
  timeout 1500 $CS --tool $tool $extra --kernel-name kns=gsw --print-limit 50 \
      --log-file gpurun_out/sanitize_${tool}.log python tools/sanitize_run.py $sz \
      > gpurun_out/sanitize_${tool}.out 2>&1
  echo "rc=$?"
  tail -3 gpurun_out/sanitize_${tool}.out
  tail -3 gpurun_out/sanitize_${tool}.log
done
