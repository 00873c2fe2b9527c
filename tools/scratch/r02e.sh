python tools/build.py > /dev/null
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_multi_loopback.py -q -x > gpurun_out/pytest_loop_r02e.txt 2>&1; tail -3 gpurun_out/pytest_loop_r02e.txt
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_reorder_r02e.csv python tools/prof_run.py --scale 24 --reps 2 --op reorder > gpurun_out/reorder_r02e.txt 2>&1
timeout 300 python tools/prof_run.py --scale 24 --reps 3 --op reorder > gpurun_out/reorder_plain_r02e.txt 2>&1
SAGE_DEF_SAGE_PASS_MB=100000 python tools/build.py > /dev/null
timeout 300 python tools/prof_run.py --scale 24 --reps 3 --op reorder > gpurun_out/reorder_1pass_r02e.txt 2>&1
python tools/build.py > /dev/null
bash tools/level_isolate.sh r02e
