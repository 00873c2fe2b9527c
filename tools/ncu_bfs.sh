python tools/build.py > /dev/null
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_bfs -s 2 -c 1 -o gpurun_out/prof_bfs_p2 python tools/prof_run.py --scale 24 --reps 3 --op bfs_push > gpurun_out/ncu_bfs_p2.log 2>&1
tail -2 gpurun_out/ncu_bfs_p2.log
