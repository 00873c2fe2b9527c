mkdir -p gpurun_out
for v in base SAGE_WIN_HOTLG=13 SAGE_WIN_HALO=2048,SAGE_WIN_HOTLG=13 SAGE_WIN_HOTLG=10; do
  envs=(); if [ "$v" != "base" ]; then IFS=',' read -ra kv <<< "$v"; for x in "${kv[@]}"; do envs+=("SAGE_DEF_${x%%=*}=${x#*=}"); done; fi
  env "${envs[@]}" python tools/build.py > /dev/null
  echo "$v $(PR_WIN_ONLY=1 timeout 400 python tools/pr_c4.py 5 2>&1 | tail -1)" >> gpurun_out/ab23.txt
done
python tools/build.py > /dev/null
