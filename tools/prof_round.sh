#!/bin/bash
# ncu evidence for one round (under gpurun): the launch list of the bench command, then one
# `--set full` capture per product kernel family on C2 (RMAT-24).  Read them here with
# `ncu -i gpurun_out/prof_<k>_<tag>.ncu-rep --page raw --csv` (tools/summarize_profiles.py).
# Usage: bash tools/prof_round.sh <tag> [kernels...]   (default: all)
tag=${1:-r02}; shift
ks=${@:-"bfs sssp pr_pull pr_push pr_win sample bc"}
out=gpurun_out; mkdir -p $out
python tools/build.py > /dev/null
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file $out/launches_$tag.csv python bench.py --steps 2 --warmup 1 --no-extras > $out/bench_ncu_$tag.txt 2>&1
full="ncu --set full --clock-control none --import-source on"
for k in $ks; do
  case $k in
    bfs)     timeout 900 $full -k regex:k_bfs -s 2 -c 1 -o $out/prof_bfs_$tag python tools/prof_run.py --scale 24 --reps 3 --op bfs_push > $out/ncu_bfs_$tag.log 2>&1 ;;
    sssp)    timeout 900 $full -k regex:k_sssp -s 1 -c 1 -o $out/prof_sssp_$tag python tools/prof_run.py --scale 24 --reps 2 --op sssp > $out/ncu_sssp_$tag.log 2>&1 ;;
    pr_pull) timeout 900 $full -k regex:k_pagerank_pull -s 1 -c 1 -o $out/prof_pr_pull_$tag python tools/prof_run.py --scale 24 --reps 2 --op pr > $out/ncu_pr_pull_$tag.log 2>&1 ;;
    pr_push) timeout 900 $full -k regex:"k_pagerank<" -s 1 -c 1 -o $out/prof_pr_push_$tag python tools/prof_run.py --scale 24 --reps 2 --op pr_push > $out/ncu_pr_push_$tag.log 2>&1 ;;
    sample)  timeout 900 $full -k regex:k_sample -s 3 -c 3 -o $out/prof_sample_$tag python tools/prof_run.py --scale 24 --reps 1 --op reorder > $out/ncu_sample_$tag.log 2>&1 ;;
    pr_win)  timeout 900 $full -k regex:k_pagerank_win -s 1 -c 1 -o $out/prof_pr_win_$tag python tools/prof_run.py --graph uk --n 10000000 --reps 2 --op pr_push > $out/ncu_pr_win_$tag.log 2>&1 ;;
    bc)      timeout 900 $full -k regex:k_bc -s 2 -c 2 -o $out/prof_bc_$tag python tools/prof_run.py --scale 24 --reps 2 --op bc > $out/ncu_bc_$tag.log 2>&1 ;;
  esac
  echo "$k done rc=$?"
done
