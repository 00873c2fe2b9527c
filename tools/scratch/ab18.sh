mkdir -p gpurun_out
for v in base SAGE_FUSED_LOGC=1; do
  if [ $v == base ]; then python tools/build.py > /dev/null; else env SAGE_DEF_$v python tools/build.py > /dev/null; fi
  echo "$v $(timeout 400 python tools/cfg_bfs.py C4 2>&1 | tail -1)" >> gpurun_out/ab18.txt
done
python tools/build.py > /dev/null
