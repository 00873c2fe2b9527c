for mb in 3 5 6 4; do
  SAGE_DEF_SAGE_BFS_MINB=$mb python tools/build.py --force > /dev/null 2>&1
  echo "minb=$mb"; timeout 300 python tools/prof_run.py --scale 24 --reps 3 --op bfs_push | grep -E "kernel_ms" | tail -2
done
