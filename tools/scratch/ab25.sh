mkdir -p gpurun_out
python tools/build.py > /dev/null
timeout 900 python -m pytest tests -m gpu -q -x -k "traversal or configs or bc" > gpurun_out/ab25_pytest.txt 2>&1
for v in base SAGE_SPLIT_PROP=0 SAGE_SPLIT_PROP=4096; do
  if [ $v == base ]; then python tools/build.py > /dev/null; else env SAGE_DEF_$v python tools/build.py > /dev/null; fi
  echo "== $v" >> gpurun_out/ab25.txt
  timeout 300 python tools/c1_sweep.py 2>&1 | head -2 >> gpurun_out/ab25.txt
  timeout 300 python bench.py 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C2', round(d['value'],2), round(d['roofline']['kernel_ms'],3), 'DO', round(d['bfs_do']['ms'],3), 'SSSP', round(d['sssp']['ms'],2), 'BC', round(d['bc']['ms_per_source'],2), 'PR', round(d['pagerank']['pull']['ms_20_iter'],1), round(d['pagerank']['push']['ms_20_iter'],1), 'C4s', round(d['c4_shape']['bfs_ms'],3), 'C1', round(d['c1']['push']['us_median']), round(d['c1']['do']['us_median']))" >> gpurun_out/ab25.txt
done
python tools/build.py > /dev/null
