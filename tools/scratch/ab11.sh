mkdir -p gpurun_out
for v in 3 4; do
SAGE_DEF_SAGE_WIN_MODE=$v python tools/build.py > /dev/null
echo "mode $v $(PR_WIN_ONLY=1 timeout 400 python tools/pr_c4.py 5 2>&1 | tail -1)" >> gpurun_out/ab11_pr.txt
done
python tools/build.py > /dev/null
