mkdir -p gpurun_out
python tools/build.py > /dev/null
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/ab31_pytest.txt 2>&1
timeout 300 python tools/c1_sweep.py 2>&1 | head -2 > gpurun_out/ab31.txt
timeout 300 python tools/prof_run.py --scale 16 --reps 4 --op bfs_push 2>&1 | tail -8 >> gpurun_out/ab31.txt
timeout 300 python bench.py --no-extras 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C2', round(d['value'],2), round(d['roofline']['kernel_ms'],3))" >> gpurun_out/ab31.txt
echo "C4 $(timeout 400 python tools/cfg_bfs.py C4 2>&1 | tail -1)" >> gpurun_out/ab31.txt
