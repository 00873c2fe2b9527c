mkdir -p gpurun_out
python tools/build.py > /dev/null
timeout 600 python -m pytest tests -m gpu -q -x -k "bc or BC or smoke" > gpurun_out/ab32_pytest.txt 2>&1
timeout 300 python bench.py 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C2', round(d['value'],2), 'BC', round(d['bc']['ms_per_source'],2), 'reorder', round(d['reorder']['round_ms'],1))" > gpurun_out/ab32.txt
timeout 900 python tools/c3_reorder.py 5 > gpurun_out/ab32_c3.json 2>&1
timeout 600 python tools/reorder_round_profile.py >> gpurun_out/ab32.txt 2>&1
