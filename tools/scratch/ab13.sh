mkdir -p gpurun_out
python tools/build.py > /dev/null
timeout 600 python -m pytest tests/test_gpu_traversal.py -q -x -k "pagerank" > gpurun_out/ab13_pytest.txt 2>&1
timeout 400 python tools/pr_c4.py 5 > gpurun_out/ab13_pr.txt 2>&1
timeout 900 python tools/c3_reorder.py 5 > gpurun_out/ab13_c3.txt 2>&1
