"""Summarise one `ncu --set full --import-source on` capture into a markdown file under profiles/.

    python tools/summarize_ncu.py <report.ncu-rep> <out.md> "<title / command>" [model_bytes]

Writes: the headline metrics (duration, DRAM bytes, L2 / L1 hit rates, issue activity), the
L1TEX / LTS sub-unit utilisations (to name the unit that bounds a kernel), the top warp-stall
reasons, and the SASS lines that move the most L2 sectors with their stall samples (to attribute
the traffic to an array of the method).  Prints the markdown.
"""
import csv
import io
import subprocess
import sys

KEYS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "lts__t_sector_hit_rate.pct", "l1tex__t_sector_hit_rate.pct",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "smsp__inst_executed.sum", "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed", "l1tex__throughput.avg.pct_of_peak_sustained_elapsed",
    "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
    "l1tex__m_l1tex2xbar_req_cycles_active.avg.pct_of_peak_sustained_elapsed",
    "l1tex__lsu_writeback_active.avg.pct_of_peak_sustained_elapsed",
    "l1tex__lsuin_requests.avg.pct_of_peak_sustained_elapsed",
    "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
    "l1tex__t_requests_pipe_lsu_mem_global_op_atom.sum",
    "lts__t_sectors_srcunit_tex_op_read.sum", "lts__t_sectors_srcunit_tex_op_atom.sum",
    "lts__t_sectors_srcunit_tex_op_red.sum", "lts__t_sectors_srcunit_tex_op_write.sum",
    "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
    "smsp__inst_executed_op_global_ld.sum", "smsp__inst_executed_op_shared_ld.sum",
]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}


def main():
    rep, out, title = sys.argv[1], sys.argv[2], sys.argv[3]
    model = float(sys.argv[4]) if len(sys.argv) > 4 else None
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(raw)))
    h, u, v = r[0], r[1], r[2]
    d, un = dict(zip(h, v)), dict(zip(h, u))
    kname = d.get("Kernel Name", "?")

    def val(k):
        try:
            return float(str(d[k]).replace(",", "")) * SCALE.get(un.get(k, ""), 1)
        except (KeyError, ValueError):
            return None

    rd, wr = val("dram__bytes_read.sum") or 0.0, val("dram__bytes_write.sum") or 0.0
    lines = [f"# {title}\n", f"Kernel: `{kname}`.\n", "| metric | value | unit |", "|---|---|---|"]
    for k in KEYS:
        if k in d:
            lines.append(f"| {k} | {d[k]} | {un.get(k, '')} |")
    lines.append(f"\nDRAM traffic per launch {(rd + wr) / 1e9:.3f} GB (read {rd / 1e9:.3f}, write {wr / 1e9:.3f})"
                 + (f"; algorithmic (model) bytes {model / 1e9:.3f} GB, amplification {(rd + wr) / model:.2f}x."
                    if model else "."))
    stalls = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): float(x) for k, x in d.items()
              if k.startswith("smsp__pcsamp_warps_issue_stalled") and not k.endswith("not_issued") and x
              and x.replace(".", "").isdigit()}
    tot = sum(stalls.values()) or 1.0
    lines += ["\n| warp stall | share of samples |", "|---|---|"]
    for k, x in sorted(stalls.items(), key=lambda kv: -kv[1])[:8]:
        lines.append(f"| {k} | {x / tot * 100:.1f}% |")
    src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(src)))
    hdr = next((i for i, x in enumerate(rows) if x and x[0] == "Address"), None)
    if hdr is not None:
        H = rows[hdr]
        ci = {k: H.index(k) for k in ("Source", "L2 Theoretical Sectors Global", "Warp Stall Sampling (All Samples)",
                                      "Instructions Executed") if k in H}
        body = [x for x in rows[hdr + 1:] if len(x) == len(H)]

        def num(x, k):
            try:
                return float(x[ci[k]].replace(",", ""))
            except (KeyError, ValueError):
                return 0.0
        tsec = sum(num(x, "L2 Theoretical Sectors Global") for x in body) or 1.0
        tsmp = sum(num(x, "Warp Stall Sampling (All Samples)") for x in body) or 1.0
        top = sorted(body, key=lambda x: -num(x, "L2 Theoretical Sectors Global"))[:12]
        lines += ["\nSASS lines moving the most L2 sectors (share of the kernel's L2 sectors / stall samples):\n",
                  "| SASS | L2 sectors | share | stall samples share |", "|---|---|---|---|"]
        for x in top:
            lines.append(f"| `{x[ci['Source']].strip()}` | {num(x, 'L2 Theoretical Sectors Global'):.3g} | "
                         f"{num(x, 'L2 Theoretical Sectors Global') / tsec * 100:.1f}% | "
                         f"{num(x, 'Warp Stall Sampling (All Samples)') / tsmp * 100:.1f}% |")
    txt = "\n".join(lines) + "\n"
    open(out, "w").write(txt)
    print(txt)


if __name__ == "__main__":
    main()
