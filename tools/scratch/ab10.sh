mkdir -p gpurun_out
python tools/build.py > /dev/null
timeout 600 python -m pytest tests/test_gpu_traversal.py -q -x -k "pagerank" > gpurun_out/ab10_pytest.txt 2>&1
timeout 300 python tools/pr_c4.py 5 10000000 >> gpurun_out/ab10_pr.txt 2>&1
PR_WIN_ONLY=1 timeout 400 python tools/pr_c4.py 5 >> gpurun_out/ab10_pr.txt 2>&1
SAGE_DEF_SAGE_WIN_MODE=2 python tools/build.py > /dev/null
PR_WIN_ONLY=1 timeout 400 python tools/pr_c4.py 5 >> gpurun_out/ab10_pr.txt 2>&1
python tools/build.py > /dev/null
