"""profiles/traffic.json (read by bench.py for the roofline's `traffic`) from an ncu --set full
capture of the push BFS kernel:  python tools/update_traffic.py <report.ncu-rep> <profiles md name>"""
import csv
import io
import json
import subprocess
import sys

rep, md = sys.argv[1], sys.argv[2]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(raw)))
d, u = dict(zip(r[0], r[2])), dict(zip(r[0], r[1]))
sc = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
rd = float(d["dram__bytes_read.sum"]) * sc[u["dram__bytes_read.sum"]]
wr = float(d["dram__bytes_write.sum"]) * sc[u["dram__bytes_write.sum"]]
out = {"kernel": d.get("Kernel Name", "?") + " push-only (SAGE_F_PUSH_ONLY), RMAT-24 sym, 1 launch = 1 BFS",
       "source": f"profiles/{md} (ncu --set full --clock-control none)",
       "bfs_push_bytes_per_launch": rd + wr, "dram_read_bytes": rd, "dram_write_bytes": wr,
       "lts_hit_rate_pct": float(d["lts__t_sector_hit_rate.pct"]),
       "ncu_duration_ms": float(d["gpu__time_duration.sum"])}
json.dump(out, open("profiles/traffic.json", "w"), indent=1)
print(json.dumps(out, indent=1))
