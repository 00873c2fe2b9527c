for v in 1 0; do
  SAGE_DEF_SAGE_STATUS_NC=$v python tools/build.py --force > /dev/null 2>&1
  echo "status_nc=$v"; timeout 300 python tools/prof_run.py --scale 24 --reps 4 --op bfs_push | grep -E "kernel_ms" | tail -3
done
