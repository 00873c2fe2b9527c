mkdir -p gpurun_out
python tools/build.py > /dev/null
timeout 900 python -m pytest tests -m gpu -q -x -k "reorder or online" > gpurun_out/ab16_pytest.txt 2>&1
echo "$(timeout 600 python tools/reorder_round_profile.py 2>&1 | tr '\n' ' ')" >> gpurun_out/ab16.txt
echo "$(timeout 600 python tools/reorder_round_profile.py 2>&1 | tr '\n' ' ')" >> gpurun_out/ab16.txt
