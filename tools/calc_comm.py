"""Fig. 5 analog: calculation vs communication time of the partitioned factorization.

    python tools/calc_comm.py [--out profiles/r02_calc_comm.json]

For C2 / C3 / C5 with G = 2, 4, 8 column owners (cyclic guide array, Eq. 12) the plan is run with
profile = 1 and the library's CUDA-event statistics (tqr_kernel_stats) give the device-busy time of
the update kernels (which = 0), the panel kernels (1), the layout passes (2) and the panel transfers
(3: from the start of a step's copies to their completion), plus the bytes transferred.  With one
GPU the owners are logical (every owner on cuda:0), so a transfer is an HBM-to-HBM copy, not an
NVLink one: the byte counts are the multi-GPU ones, the times are a lower bound.  The NVLink time
at the nominal 900 GB/s per direction is reported beside them.
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_icpp_kimp13_b200 as tqr  # noqa: E402
from bench import CONFIGS  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="C2,C3,C5")
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    res = {}
    for cfg in args.configs.split(","):
        m, n, nb, ib, seed = CONFIGS[cfg]
        g = torch.Generator(device="cuda").manual_seed(seed)
        A0 = torch.randn((n, m), dtype=torch.float64, device="cuda", generator=g).t()
        for G in (2, 4, 8):
            plan = tqr.Plan(m, n, nb, ib, ndev=G, logical_devices=True, profile=True)
            plan.load(A0)
            plan.factor_tiles()
            for w in range(4):
                plan.kernel_stats(w, reset=True)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            plan.load(A0)
            plan.factor_tiles()
            e1.record()
            torch.cuda.synchronize()
            st = [plan.kernel_stats(w, reset=True) for w in range(4)]
            plan.close()
            total = e0.elapsed_time(e1)
            row = {"total_ms": round(total, 3),
                   "update_busy_ms": round(st[0][1], 3), "panel_busy_ms": round(st[1][1], 3),
                   "layout_ms": round(st[2][1], 3), "transfer_busy_ms": round(st[3][1], 3),
                   "transfers": st[3][0], "transfer_bytes": st[3][2],
                   "transfer_ms_at_900GBs": round(st[3][2] / 900e9 * 1e3, 3)}
            row["comm_share_at_900GBs"] = round(row["transfer_ms_at_900GBs"] / total, 4)
            res["%s_G%d" % (cfg, G)] = row
            print(cfg, "G=%d" % G, json.dumps(row), flush=True)
        del A0
        torch.cuda.empty_cache()
    if args.out:
        with open(args.out, "w") as f:
            json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
