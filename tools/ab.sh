#!/bin/bash
# A/B timing session (under gpurun): default build + tests, then variants given as
# "NAME=VALUE[,NAME=VALUE]" compile definitions (SAGE_DEF_*), each with a short push-BFS bench.
# Usage: bash tools/ab.sh <tag> [DEF=VAL ...]
tag=${1:-ab}; shift
out=gpurun_out; mkdir -p $out
# leave the default library in the tree whatever happens (the stamp makes this a real rebuild)
trap 'python tools/build.py > /dev/null' EXIT
python tools/build.py > /dev/null || exit 1
timeout 900 python -m pytest tests -m gpu -q -x > $out/pytest_gpu_$tag.txt 2>&1
tail -2 $out/pytest_gpu_$tag.txt
timeout 300 python bench.py --no-extras > $out/bench_${tag}_base.json 2>&1
timeout 300 python tools/prof_run.py --scale 24 --reps 3 --op bfs_push > $out/levels_${tag}_base.txt 2>&1
echo base; cut -c1-200 $out/bench_${tag}_base.json
for d in "$@"; do
  envs=(); IFS=',' read -ra kv <<< "$d"; for x in "${kv[@]}"; do envs+=("SAGE_DEF_${x%%=*}=${x#*=}"); done
  env "${envs[@]}" python tools/build.py --force > /dev/null || continue
  timeout 300 python bench.py --no-extras > $out/bench_${tag}_$d.json 2>&1
  timeout 300 python tools/prof_run.py --scale 24 --reps 3 --op bfs_push > $out/levels_${tag}_$d.txt 2>&1
  echo $d; cut -c1-200 $out/bench_${tag}_$d.json
done
