mkdir -p gpurun_out
python tools/build.py > /dev/null
timeout 900 python -m pytest tests -m gpu -q -x -k "sssp or SSSP or smoke or fullsize" > gpurun_out/ab22_pytest.txt 2>&1
for v in base SAGE_SSSP_SHADOW=0; do
  if [ $v == base ]; then python tools/build.py > /dev/null; else env SAGE_DEF_$v python tools/build.py > /dev/null; fi
  echo "== $v" >> gpurun_out/ab22.txt
  LEVELS=0 timeout 300 python tools/prof_run.py --scale 24 --reps 4 --op sssp 2>&1 | grep -v "^   L" >> gpurun_out/ab22.txt
done
python tools/build.py > /dev/null
