#!/bin/bash
# One GPU session: tests, bench, launch list and a full ncu capture of the dominant kernel.
# Usage (under gpurun): bash tools/gpu_round.sh <tag>
tag=${1:-r01}
out=gpurun_out
mkdir -p $out
python tools/build.py > /dev/null
timeout 1200 python -m pytest tests -m gpu -q > $out/pytest_gpu_$tag.txt 2>&1
timeout 300 python __graft_entry__.py smoke > $out/smoke_$tag.txt 2>&1
timeout 900 python bench.py > $out/bench_$tag.json 2> $out/bench_$tag.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file $out/launches_$tag.csv python bench.py --steps 2 --warmup 1 --no-extras > $out/bench_ncu_$tag.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_bfs -s 2 -c 1 \
    -o $out/prof_bfs_$tag python tools/prof_run.py --scale 24 --reps 3 --op bfs_push > $out/ncu_bfs_$tag.log 2>&1
# Table 3-style Tiled Partitioning share: warp-time in classification (enqueue flushes) over all
# warp-time of the push BFS kernel (SAGE_PROF build, separate library)
SAGE_PROF=1 python tools/build.py > /dev/null
SAGE_PROF=1 SAGE_LIB=libsage_prof.so timeout 300 python tools/prof_run.py --scale 24 --reps 3 --op bfs_push \
    > $out/tp_share_$tag.txt 2>&1
tail -3 $out/pytest_gpu_$tag.txt; cat $out/smoke_$tag.txt | tail -2
