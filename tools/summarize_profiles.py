"""Summarise a gpu_round.sh session into profiles/: ncu --set full of the dominant kernel,
the launch list shares, the bench line, and profiles/traffic.json (read by bench.py)."""
import csv
import io
import json
import shutil
import subprocess
import sys
from collections import defaultdict

tag = sys.argv[1] if len(sys.argv) > 1 else "r01"
rep = f"gpurun_out/prof_bfs_{tag}.ncu-rep"
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(raw)))
h, u, v = r[0], r[1], r[2]
d = dict(zip(h, v))
un = dict(zip(h, u))
keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_sector_hit_rate.pct",
        "l1tex__t_sector_hit_rate.pct", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "l1tex__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "lts__t_sectors_srcunit_tex_op_read.sum",
        "lts__t_sectors_srcunit_tex_op_atom.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
        "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum"]
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
rd = float(d["dram__bytes_read.sum"]) * scale.get(un["dram__bytes_read.sum"], 1)
wr = float(d["dram__bytes_write.sum"]) * scale.get(un["dram__bytes_write.sum"], 1)
stalls = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): float(x) for k, x in d.items()
          if k.startswith("smsp__pcsamp_warps_issue_stalled") and not k.endswith("not_issued") and x}
tot = sum(stalls.values())
json.dump({"kernel": d.get("Kernel Name", "?").split("(")[0] + " push-only (SAGE_F_PUSH_ONLY), RMAT-24 sym, 1 launch = 1 BFS",
           "source": f"profiles/{tag}_bfs_push_ncu.md (ncu --set full --clock-control none)",
           "bfs_push_bytes_per_launch": rd + wr, "dram_read_bytes": rd, "dram_write_bytes": wr,
           "lts_hit_rate_pct": float(d["lts__t_sector_hit_rate.pct"]),
           "ncu_duration_ms": float(d["gpu__time_duration.sum"])}, open("profiles/traffic.json", "w"), indent=1)
with open(f"profiles/{tag}_bfs_push_ncu.md", "w") as f:
    f.write(f"# {tag} — ncu --set full of the persistent push BFS kernel ({d.get('Kernel Name', '?').split('(')[0]})\n\n")
    f.write("`ncu --set full --clock-control none --import-source on -k regex:k_bfs -s 2 -c 1 python tools/prof_run.py "
            "--scale 24 --reps 3 --op bfs_push` on one B200 (RMAT-24 symmetric, push-only; one launch = one BFS).\n\n")
    f.write("| metric | value | unit |\n|---|---|---|\n")
    for k in keys:
        f.write(f"| {k} | {d.get(k)} | {un.get(k)} |\n")
    f.write("\n| warp stall | share of samples |\n|---|---|\n")
    for k, x in sorted(stalls.items(), key=lambda kv: -kv[1])[:8]:
        f.write(f"| {k} | {x / tot * 100:.1f}% |\n")
    f.write(f"\nDRAM traffic per launch {(rd + wr) / 1e9:.2f} GB (read {rd / 1e9:.2f}, write {wr / 1e9:.2f}); "
            "algorithmic (model) bytes 4.41 GB.\n")
rows = [x for x in csv.reader(open(f"gpurun_out/launches_{tag}.csv")) if len(x) > 10]
hh = rows[0]
iK, iV, iU = hh.index("Kernel Name"), hh.index("Metric Value"), hh.index("Metric Unit")
totk, cnt = defaultdict(float), defaultdict(int)
for x in rows[1:]:
    t = float(x[iV].replace(",", ""))
    t = {"nsecond": t / 1e3, "ns": t / 1e3, "usecond": t, "us": t, "msecond": t * 1e3, "ms": t * 1e3}.get(x[iU], t)
    k = x[iK].split("(")[0]
    totk[k] += t
    cnt[k] += 1
T = sum(totk.values())
with open(f"profiles/{tag}_launches.md", "w") as f:
    f.write(f"# {tag} — launch list of `bench.py --steps 2 --warmup 1 --no-extras` under ncu\n\n"
            "`ncu --metrics gpu__time_duration.sum --clock-control none` (cold-cache, serialised: compare shares). "
            "Includes graph validation at load and the warm-up/timed BFS steps.\n\n"
            "| kernel | launches | total us | share |\n|---|---|---|---|\n")
    for k, t in sorted(totk.items(), key=lambda kv: -kv[1]):
        f.write(f"| {k} | {cnt[k]} | {t:.1f} | {t / T * 100:.1f}% |\n")
shutil.copy(f"gpurun_out/launches_{tag}.csv", f"profiles/{tag}_launches.csv")
shutil.copy(f"gpurun_out/bench_{tag}.json", f"profiles/{tag}_bench.json")
print(open(f"profiles/{tag}_bfs_push_ncu.md").read())
print(open(f"profiles/{tag}_launches.md").read())
