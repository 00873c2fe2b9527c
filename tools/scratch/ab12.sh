mkdir -p gpurun_out
python tools/build.py > /dev/null
timeout 600 python -m pytest tests/test_gpu_traversal.py -q -x -k "pagerank" > gpurun_out/ab12_pytest.txt 2>&1
echo "hot+bins $(timeout 400 python tools/pr_c4.py 5 2>&1 | tail -1)" >> gpurun_out/ab12_pr.txt
SAGE_DEF_SAGE_WIN_BINS=0 python tools/build.py > /dev/null
echo "hot+direct $(PR_WIN_ONLY=1 timeout 400 python tools/pr_c4.py 5 2>&1 | tail -1)" >> gpurun_out/ab12_pr.txt
SAGE_DEF_SAGE_WIN_BINS=0 SAGE_DEF_SAGE_WIN_HOT=0 python tools/build.py > /dev/null
echo "direct $(PR_WIN_ONLY=1 timeout 400 python tools/pr_c4.py 5 2>&1 | tail -1)" >> gpurun_out/ab12_pr.txt
python tools/build.py > /dev/null
