"""Difference the counters of tools/level_isolate.sh's builds into per-level rates.

    python tools/level_isolate.py gpurun_out/level_iso_<tag>   (reads <prefix>_L{1,2,3,-1}.csv)

For every counter X, level L's utilisation of the unit is
    (X(L) - X(L-1)) / (X.sum.peak_sustained * (unit cycles(L) - unit cycles(L-1)))
i.e. the same ratio ncu's pct_of_peak_sustained_elapsed reports, restricted to one level.
"""
import csv
import io
import sys

SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "ns": 1, "us": 1e3, "ms": 1e6, "nsecond": 1, "usecond": 1e3,
         "msecond": 1e6, "second": 1e9}


def load(path):
    txt = open(path).read()
    lines = [ln for ln in txt.splitlines() if ln.startswith('"')]
    r = list(csv.reader(io.StringIO("\n".join(lines))))
    hdr = r[0]
    ci = {k: hdr.index(k) for k in ("Metric Name", "Metric Unit", "Metric Value")}
    out = {}
    for x in r[1:]:
        try:
            v = float(x[ci["Metric Value"]].replace(",", "")) * SCALE.get(x[ci["Metric Unit"]], 1)
        except ValueError:
            continue
        out[x[ci["Metric Name"]]] = v
    return out


def unit_cycles(name):
    for u in ("l1tex", "lts", "dram"):
        if name.startswith(u + "__"):
            return f"{u}__cycles_elapsed.avg"
    return "sm__cycles_elapsed.avg"


def main():
    pre = sys.argv[1]
    runs = {L: load(f"{pre}_L{L}.csv") for L in (1, 2, 3, -1)}
    names = sorted({k[:-len(".sum")] for k in runs[1] if k.endswith(".sum") and not k.startswith("gpu__")})
    cols = [("level 2", runs[2], runs[1]), ("level 3", runs[3], runs[2]), ("levels 2+3", runs[3], runs[1]),
            ("whole BFS", runs[-1], None)]
    print("# C2 push BFS, heavy levels in isolation (counter differences of stop-after-level builds)\n")
    print("| | " + " | ".join(c[0] for c in cols) + " |")
    print("|---|" + "---|" * len(cols))

    def d(a, b, k):
        return a.get(k, 0.0) - (b.get(k, 0.0) if b else 0.0)
    print("| duration (us) | " + " | ".join(f"{d(a, b, 'gpu__time_duration.sum') / 1e3:.0f}" for _, a, b in cols) + " |")
    print("| SM cycles | " + " | ".join(f"{d(a, b, 'sm__cycles_elapsed.avg'):.3g}" for _, a, b in cols) + " |")
    for nm in names:
        cells = []
        for _, a, b in cols:
            cnt = d(a, b, nm + ".sum")
            pk = a.get(nm + ".sum.peak_sustained", 0.0)
            cyc = d(a, b, unit_cycles(nm))
            pct = 100.0 * cnt / (pk * cyc) if pk and cyc > 0 else float("nan")
            cells.append(f"{cnt:.3g} ({pct:.0f}%)")
        print(f"| {nm} | " + " | ".join(cells) + " |")
    print("\nEach cell: the counter's increment over the level(s), and in brackets its share of the unit's "
          "sustained peak over those cycles (ncu's pct_of_peak_sustained_elapsed, per level).")


if __name__ == "__main__":
    main()
