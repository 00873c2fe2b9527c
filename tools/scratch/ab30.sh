mkdir -p gpurun_out
python tools/build.py > /dev/null
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/ab30_pytest.txt 2>&1
timeout 300 python tools/c1_sweep.py 2>&1 | head -2 > gpurun_out/ab30.txt
timeout 400 python bench.py 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C2', round(d['value'],2), round(d['roofline']['kernel_ms'],3), 'DO', round(d['bfs_do']['ms'],3), 'SSSP', round(d['sssp']['ms'],2), 'BC', round(d['bc']['ms_per_source'],2), 'C1', round(d['c1']['push']['us_median']), round(d['c1']['do']['us_median']))" >> gpurun_out/ab30.txt
