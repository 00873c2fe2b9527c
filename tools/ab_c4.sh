#!/bin/bash
# A/B of C2 push BFS (bench) and the C4-shape BFS (10M vertices, ~500 levels) for compile variants.
out=gpurun_out; mkdir -p $out
for d in base "$@"; do
  envs=(); if [ "$d" != "base" ]; then IFS=',' read -ra kv <<< "$d"; for x in "${kv[@]}"; do envs+=("SAGE_DEF_${x%%=*}=${x#*=}"); done; fi
  env "${envs[@]}" python tools/build.py --force > /dev/null
  for r in 1 2; do
    v=$(python bench.py --no-extras 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().splitlines()[-1]); print(round(d['value'],2), round(d['roofline']['kernel_ms'],3))")
    u=$(LEVELS=0 python tools/prof_run.py --graph uk --n 10000000 --reps 3 --op bfs_push 2>/dev/null | grep "^bfs_push 2" | python -c "import sys,ast; l=sys.stdin.read(); print(round(ast.literal_eval(l[l.index('{'):])['kernel_ms'],3))")
    echo "variant $d rep $r: C2 $v | C4-shape ms $u"
  done
done
