python tools/build.py > /dev/null
SAGE_PROF=1 python tools/build.py > /dev/null
for ml in 1 2 3; do
  echo "== max levels $ml"
  SAGE_DEBUG_MAX_LEVELS=$ml SAGE_PROF=1 SAGE_LIB=libsage_prof.so python tools/prof_run.py --scale 24 --reps 2 --op bfs_push 2>&1 | grep -v "^ *L dir" | tail -3
done
echo "== full"; SAGE_PROF=1 SAGE_LIB=libsage_prof.so python tools/prof_run.py --scale 24 --reps 2 --op bfs_push 2>&1 | tail -12
