"""Critical-path probe (diagnostic): TQR_CRITICAL_PATH_PROBE=1 skips the bulk trailing updates, so
a factorization runs only the panels, the lookahead updates and the panel transfers -- the chain no
number of GPUs can shorten.  Logical owners on one GPU reproduce the multi-GPU ownership pattern
(peer copies stand in for the NCCL broadcast).  Usage: python tools/cp_probe.py C5 8"""
import os
import sys

os.environ["TQR_CRITICAL_PATH_PROBE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icpp_kimp13_b200 as tqr  # noqa: E402
from bench import CONFIGS  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C5"
G = int(sys.argv[2]) if len(sys.argv) > 2 else 8
m, n, nb, ib, seed = CONFIGS[cfg]
g = torch.Generator(device="cuda").manual_seed(seed)
A0 = torch.randn((n, m), dtype=torch.float64, device="cuda", generator=g).t()
guides = {"cyclic": list(range(G)), "pairs": [d for d in range(G) for _ in range(2)],
          "quads": [d for d in range(G) for _ in range(4)],
          "snake": list(range(G)) + list(range(G - 1, -1, -1))}
for name, guide in guides.items():
    plan = tqr.Plan(m, n, nb, ib, ndev=G, guide=guide, logical_devices=True)
    plan.load(A0)
    plan.factor_tiles()
    torch.cuda.synchronize()
    best = 1e30
    for _ in range(3):
        plan.load(A0)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        plan.factor_tiles()
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    plan.close()
    print("%s G=%d guide=%s critical path %.1f ms" % (cfg, G, name, best), flush=True)
