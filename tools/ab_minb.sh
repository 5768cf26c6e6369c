set -x
mkdir -p gpurun_out
for V in default m4; do
  if [ $V = m4 ]; then export GSW_LIB_PATH=$PWD/build/var_m4/libgsw.so; else unset GSW_LIB_PATH; fi
  echo "== $V"
  timeout 300 python tools/perf_all.py C3 C2 2>&1 | grep -E "BFS|SSSP"
  timeout 300 python bench.py --quick --no-cpu-baseline --steps 20 --warmup 5 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('bench', d['value'], d['ms_per_step'])"
  timeout 600 python tools/bfs_c5.py
done
