# final round-2 evidence run (one B200): tests, smoke, bench, launch list, ncu captures, full configs
mkdir -p gpurun_out
bash tools/gpu_round.sh r02i > gpurun_out/gpu_round_r02i.txt 2>&1
bash tools/prof_round.sh r02i sssp pr_win > gpurun_out/prof_round_r02i.txt 2>&1
timeout 1500 python tools/full_configs.py C3 C4 > gpurun_out/full_configs_r02i.json 2> gpurun_out/full_configs_r02i.err
timeout 900 python tools/c3_reorder.py 5 > gpurun_out/c3_reorder_r02i.json 2> gpurun_out/c3_reorder_r02i.err
