mkdir -p gpurun_out
for v in 48 96 128 192; do
SAGE_DEF_SAGE_PASS_MB=$v python tools/build.py > /dev/null
echo "pass_mb $v $(timeout 600 python tools/reorder_round_profile.py 2>&1 | tr '\n' ' ')" >> gpurun_out/ab15.txt
done
python tools/build.py > /dev/null
