python tools/build.py > /dev/null
timeout 600 python -m pytest tests -m gpu -q -x -k "pagerank or nccl or bfs_random or bc" 2>&1 | tail -2
for pf in 4 2 8; do
  SAGE_DEF_SAGE_PR_PREFETCH=$pf python tools/build.py --force > /dev/null
  echo "== prefetch $pf"
  python tools/prof_run.py --graph uk --n 105000000 --op pr --reps 2 2>&1 | tail -1
  python tools/prof_run.py --scale 24 --op pr --reps 2 2>&1 | tail -1
  python -c "
import sys; sys.argv=['x']
" 
done
python tools/build.py --force > /dev/null
python bench.py --no-extras 2>&1 | cut -c1-220
