"""Summarise an ncu report here (no GPU): key raw metrics + per-opcode stall samples."""
import csv, subprocess, sys
from collections import defaultdict
rep = sys.argv[1]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(raw.splitlines()))
h, v = rows[0], rows[2]
keys = ["gpu__time_duration.sum", "launch__grid_size", "launch__registers_per_thread",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smsp__inst_executed.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "sm__warps_active.avg.per_cycle_active"]
for i, n in enumerate(h):
    if n in keys or ("average_warps_issue_stalled" in n and n.endswith("per_issue_active.ratio")):
        try:
            if "stalled" in n and float(v[i]) < 0.02: continue
        except Exception: pass
        print("%-90s %s" % (n, v[i]))
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(src.splitlines()))
hh = rows[1]; idx = {n: i for i, n in enumerate(hh)}
agg = defaultdict(lambda: [0, 0, 0])
for r in rows[2:]:
    s = r[idx["Source"]].strip()
    if not s: continue
    t = s.split()
    op = t[1] if t[0].startswith("@") else t[0]
    try:
        a = agg[op]; a[0] += int(r[idx["Instructions Executed"]]); a[1] += int(r[idx["Warp Stall Sampling (All Samples)"]])
        a[2] += int(r[idx["L1 Wavefronts Shared"]] or 0)
    except Exception: pass
tot = sum(a[1] for a in agg.values()) or 1
for op, a in sorted(agg.items(), key=lambda x: -x[1][1])[:int(sys.argv[2]) if len(sys.argv) > 2 else 15]:
    print("%-28s inst %12d samples %6.2f%% smem_wf %12d" % (op, a[0], 100 * a[1] / tot, a[2]))
