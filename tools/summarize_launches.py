"""Launch list (ncu --metrics gpu__time_duration.sum --csv) -> markdown table of per-kernel shares.

    python tools/summarize_launches.py <launches.csv> <out.md> "<title / command>"
"""
import csv
import io
import sys
from collections import defaultdict

src, out, title = sys.argv[1], sys.argv[2], sys.argv[3]
lines = [ln for ln in open(src).read().splitlines() if ln.startswith('"')]
r = list(csv.reader(io.StringIO("\n".join(lines))))
h = r[0]
ik, iu, iv = h.index("Kernel Name"), h.index("Metric Unit"), h.index("Metric Value")
sc = {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3, "s": 1e6, "second": 1e6}
tot, cnt = defaultdict(float), defaultdict(int)
for x in r[1:]:
    if len(x) != len(h):
        continue
    name = x[ik].split("(")[0]
    tot[name] += float(x[iv].replace(",", "")) * sc.get(x[iu], 1.0)
    cnt[name] += 1
s = sum(tot.values()) or 1.0
txt = [f"# {title}\n", "`ncu --metrics gpu__time_duration.sum --clock-control none` (cold-cache, serialised: "
       "compare shares, not absolute times).\n", "| kernel | launches | total us | share |", "|---|---|---|---|"]
for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
    txt.append(f"| {k} | {cnt[k]} | {v:.1f} | {100 * v / s:.1f}% |")
open(out, "w").write("\n".join(txt) + "\n")
print("\n".join(txt))
