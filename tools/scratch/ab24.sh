mkdir -p gpurun_out
python tools/build.py > /dev/null
timeout 900 python -m pytest tests -m gpu -q -x -k "traversal or configs or fullsize or reorder or outofcore" > gpurun_out/ab24_pytest.txt 2>&1
for v in base SAGE_FUSED_PACK_SMALL=0; do
  if [ $v == base ]; then python tools/build.py > /dev/null; else env SAGE_DEF_$v python tools/build.py > /dev/null; fi
  echo "== $v" >> gpurun_out/ab24.txt
  timeout 300 python tools/c1_sweep.py 2>&1 | head -2 >> gpurun_out/ab24.txt
  LEVELS=0 timeout 300 python tools/prof_run.py --scale 20 --reps 3 --op bfs_push 2>&1 | grep "^bfs_push" >> gpurun_out/ab24.txt
done
python tools/build.py > /dev/null
