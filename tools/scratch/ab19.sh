mkdir -p gpurun_out
for v in base SAGE_SPLIT_K=0 SAGE_WARP_RANK_LINEAR=1; do
  if [ $v == base ]; then python tools/build.py > /dev/null; else env SAGE_DEF_$v python tools/build.py > /dev/null; fi
  echo "$v $(timeout 400 python tools/cfg_bfs.py C4 2>&1 | tail -1)" >> gpurun_out/ab19.txt
  echo "$v C2 $(timeout 300 python bench.py --no-extras 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), round(d['roofline']['kernel_ms'],3))")" >> gpurun_out/ab19.txt
done
python tools/build.py > /dev/null
