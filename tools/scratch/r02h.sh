# round-2 evidence run (one B200): tests, smoke, bench, launch list, ncu captures, sanitizers, full configs
mkdir -p gpurun_out
bash tools/gpu_round.sh r02h > gpurun_out/gpu_round_r02h.txt 2>&1
bash tools/prof_round.sh r02h sssp pr_pull pr_win sample bc > gpurun_out/prof_round_r02h.txt 2>&1
bash tools/sanitize.sh r02h > gpurun_out/sanitize_r02h.txt 2>&1
timeout 1500 python tools/full_configs.py C3 C4 > gpurun_out/full_configs_r02h.json 2> gpurun_out/full_configs_r02h.err
