#!/bin/bash
# Repeated A/B of push-BFS kernel time (median over 3 bench runs per variant, alternating).
# Usage: bash tools/ab_reps.sh "DEF=VAL[,DEF=VAL]" ...   (first variant = default build)
out=gpurun_out; mkdir -p $out
# leave the default library in the tree whatever happens (the stamp makes this a real rebuild)
trap 'python tools/build.py > /dev/null' EXIT
build_variant() {
  local d=$1; envs=()
  if [ "$d" != "base" ]; then IFS=',' read -ra kv <<< "$d"; for x in "${kv[@]}"; do envs+=("SAGE_DEF_${x%%=*}=${x#*=}"); done; fi
  env "${envs[@]}" python tools/build.py --force > /dev/null
  mkdir -p /tmp/v_$2; cp paper_conf_sigmod_00020t21_b200/libsage.so /tmp/v_$2/
}
i=0; for d in base "$@"; do build_variant "$d" $i; i=$((i+1)); done
for rep in 1 2 3; do
  i=0; for d in base "$@"; do
    cp /tmp/v_$i/libsage.so paper_conf_sigmod_00020t21_b200/libsage.so
    v=$(python bench.py --no-extras 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().splitlines()[-1]); print(round(d['value'],2), round(d['roofline']['kernel_ms'],3))")
    echo "rep $rep variant $d: $v"
    i=$((i+1))
  done
done
