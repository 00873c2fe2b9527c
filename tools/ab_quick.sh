#!/bin/bash
# Quick A/B session (under gpurun): targeted tests on the default build, then alternating
# bench runs (push BFS, --no-extras) and per-level records for the default build and each
# variant given as "DEF=VAL[,DEF=VAL]" (SAGE_DEF_* compile definitions).
# Usage: bash tools/ab_quick.sh <tag> "<pytest -k expr or ''>" VARIANT...
tag=${1:-q}; kexpr=$2; shift 2
out=gpurun_out; mkdir -p $out
trap 'python tools/build.py > /dev/null' EXIT
python tools/build.py > /dev/null || exit 1
if [ -n "$kexpr" ]; then
  timeout 900 python -m pytest tests -m gpu -q -x -k "$kexpr" > $out/pytest_$tag.txt 2>&1; tail -3 $out/pytest_$tag.txt
fi
i=0; for d in base "$@"; do
  envs=(); if [ "$d" != "base" ]; then IFS=',' read -ra kv <<< "$d"; for x in "${kv[@]}"; do envs+=("SAGE_DEF_${x%%=*}=${x#*=}"); done; fi
  env "${envs[@]}" python tools/build.py > /dev/null || exit 1
  mkdir -p /tmp/v_$i; cp paper_conf_sigmod_00020t21_b200/libsage.so /tmp/v_$i/; i=$((i+1))
done
for rep in 1 2; do
  i=0; for d in base "$@"; do
    cp /tmp/v_$i/libsage.so paper_conf_sigmod_00020t21_b200/libsage.so
    v=$(timeout 300 python bench.py --no-extras 2>>$out/bench_$tag.err | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), round(d['roofline']['kernel_ms'],3), round(d['ms_per_step'],3))")
    echo "rep $rep variant $d: GTEPS kernel_ms step_ms = $v"
    if [ $rep == 1 ]; then timeout 300 python tools/prof_run.py --scale 24 --reps 3 --op bfs_push > $out/levels_${tag}_$i.txt 2>&1; tail -8 $out/levels_${tag}_$i.txt; fi
    i=$((i+1))
  done
done
