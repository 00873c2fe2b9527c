mkdir -p gpurun_out
for v in base SAGE_SPLIT_K=4 SAGE_LOGALL=65536 SAGE_SPLIT_K=4,SAGE_LOGALL=65536 SAGE_SPLIT_K=16,SAGE_LOGALL=65536; do
  envs=(); if [ "$v" != "base" ]; then IFS=',' read -ra kv <<< "$v"; for x in "${kv[@]}"; do envs+=("SAGE_DEF_${x%%=*}=${x#*=}"); done; fi
  env "${envs[@]}" python tools/build.py > /dev/null
  echo "== $v" >> gpurun_out/ab17.txt
  timeout 300 python tools/c1_sweep.py 2>&1 | head -2 >> gpurun_out/ab17.txt
  timeout 300 python bench.py --no-extras 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C2', round(d['value'],2), round(d['roofline']['kernel_ms'],3))" >> gpurun_out/ab17.txt
done
python tools/build.py > /dev/null
