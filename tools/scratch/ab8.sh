mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_traversal.py -q -x -k "pagerank" > gpurun_out/ab8_pytest.txt 2>&1
for v in base SAGE_WIN_MODE=1 SAGE_WIN_MODE=2 SAGE_WIN_GPOL=1; do
  if [ $v == base ]; then python tools/build.py > /dev/null; else env SAGE_DEF_$v python tools/build.py > /dev/null; fi
  echo "$v $(PR_WIN_ONLY=1 timeout 400 python tools/pr_c4.py 5 2>&1 | tail -1)" >> gpurun_out/ab8_pr.txt
done
python tools/build.py > /dev/null
