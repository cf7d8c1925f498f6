"""Summarise ncu CSV exports (no GPU, no .ncu-rep needed): key raw metrics and per-opcode warp
stall samples.  The CSVs come from the GPU box:
    ncu -i X.ncu-rep --page raw --csv > raw.csv
    ncu -i X.ncu-rep --page source --csv --print-source sass > source.csv
Usage: python tools/ncu_csv_summary.py raw.csv [source.csv] [top_n]"""
import csv
import sys
from collections import defaultdict

KEYS = ["gpu__time_duration.sum", "launch__grid_size", "launch__registers_per_thread",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__t_sector_hit_rate.pct", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smsp__inst_executed.sum", "dram__bytes_read.sum",
        "dram__bytes_write.sum", "sm__warps_active.avg.per_cycle_active", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"]


def raw_summary(path):
    rows = list(csv.reader(open(path)))
    h = rows[0]
    units = rows[1]
    for v in rows[2:]:
        print("-- kernel:", v[h.index("Kernel Name")][:110] if "Kernel Name" in h else "?")
        for i, n in enumerate(h):
            if n in KEYS or ("average_warps_issue_stalled" in n and n.endswith("per_issue_active.ratio")):
                try:
                    if "stalled" in n and float(v[i].replace(",", "")) < 0.02:
                        continue
                except Exception:
                    pass
                print("  %-88s %s %s" % (n, v[i], units[i] if i < len(units) else ""))


def source_summary(path, top):
    rows = list(csv.reader(open(path)))
    hi = next(i for i, r in enumerate(rows) if "Source" in r and "Address" in r)
    hh = rows[hi]
    idx = {n: i for i, n in enumerate(hh)}
    agg = defaultdict(lambda: [0, 0])
    stall_cols = [n for n in hh if n.startswith("stall_") and "Not Issued" not in n]
    stalls = defaultdict(float)
    for r in rows[hi + 1:]:
        if len(r) < len(hh):
            continue
        s = r[idx["Source"]].strip()
        if not s:
            continue
        t = s.split()
        op = t[1] if t[0].startswith("@") else t[0]
        try:
            a = agg[op]
            a[0] += int(r[idx["Instructions Executed"]] or 0)
            a[1] += int(r[idx["Warp Stall Sampling (All Samples)"]] or 0)
            for c in stall_cols:
                stalls[(op, c)] += float(r[idx[c]] or 0)
        except Exception:
            pass
    tot = sum(a[1] for a in agg.values()) or 1
    for op, a in sorted(agg.items(), key=lambda x: -x[1][1])[:top]:
        top3 = sorted(((stalls[(op, c)], c) for c in stall_cols), reverse=True)[:3]
        print("  %-26s inst %12d samples %6.2f%%  %s" % (op, a[0], 100.0 * a[1] / tot,
              ", ".join("%s %.0f%%" % (c.replace("stall_", ""), 100.0 * x / max(a[1], 1)) for x, c in top3 if x)))


if __name__ == "__main__":
    raw_summary(sys.argv[1])
    if len(sys.argv) > 2:
        source_summary(sys.argv[2], int(sys.argv[3]) if len(sys.argv) > 3 else 15)
