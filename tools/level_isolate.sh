#!/bin/bash
# The heavy levels of the C2 push BFS in isolation.  The fused kernel runs a
# whole BFS in one launch, so ncu cannot range one level; instead build the kernel to stop after
# level L (SAGE_BFS_STOP_AFTER, a profiling-only define) for L = 1, 2, 3, collect raw counters
# and their per-cycle peaks for each build on the same source, and let tools/level_isolate.py
# difference consecutive builds: level L = build(L) - build(L-1).
# Usage (under gpurun): bash tools/level_isolate.sh <tag>
tag=${1:-r02}
out=gpurun_out; mkdir -p $out
C="l1tex__t_requests_pipe_lsu_mem_global_op_ld l1tex__t_sectors_pipe_lsu_mem_global_op_ld
   l1tex__t_requests_pipe_lsu_mem_global_op_red l1tex__t_requests_pipe_lsu_mem_global_op_atom
   l1tex__t_requests l1tex__t_sectors l1tex__lsuin_requests l1tex__data_pipe_lsu_wavefronts
   l1tex__data_pipe_lsu_wavefronts_mem_lgds_cmd_read l1tex__m_xbar2l1tex_read_sectors
   l1tex__m_l1tex2xbar_req_cycles_active l1tex__lsu_writeback_active l1tex__f_wavefronts
   lts__t_requests lts__t_sectors lts__t_tag_requests lts__d_sectors lts__t_sectors_srcunit_tex_op_read
   lts__t_sectors_lookup_hit lts__t_sectors_lookup_miss lts__xbar2lts_cycles_active lts__lts2xbar_cycles_active
   dram__bytes_read dram__bytes_write sm__inst_executed_pipe_lsu smsp__inst_executed smsp__issue_active
   smsp__inst_executed_op_global_ld"
M="gpu__time_duration.sum,sm__cycles_elapsed.avg,l1tex__cycles_elapsed.avg,lts__cycles_elapsed.avg,dram__cycles_elapsed.avg"
for c in $C; do M="$M,$c.sum,$c.sum.peak_sustained"; done
for L in 1 2 3 -1; do
  SAGE_DEF_SAGE_BFS_STOP_AFTER=$L python tools/build.py > /dev/null || exit 1
  timeout 900 ncu --metrics $M --clock-control none -k regex:k_bfs -s 2 -c 1 --csv \
      python tools/prof_run.py --scale 24 --reps 3 --op bfs_push > $out/level_iso_${tag}_L$L.csv 2> $out/level_iso_${tag}_L$L.err
  echo "stop=$L rc=$?"
done
python tools/build.py > /dev/null
python tools/level_isolate.py $out/level_iso_${tag} > $out/level_iso_${tag}.md
cat $out/level_iso_${tag}.md
