"""One tiled QR of a BASELINE config through the C ABI (for ncu / compute-sanitizer runs)."""
import argparse, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_icpp_kimp13_b200 as tqr
from bench import CONFIGS
ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C3")
ap.add_argument("--reps", type=int, default=1)
args = ap.parse_args()
m, n, nb, ib, seed = CONFIGS[args.config]
g = torch.Generator(device="cuda").manual_seed(seed)
A = torch.randn((n, m), dtype=torch.float64, device="cuda", generator=g).t()
R = torch.empty((n, m), dtype=torch.float64, device="cuda").t()
with tqr.Plan(m, n, nb, ib) as p:
    for _ in range(args.reps):
        p.load(A); p.factor_tiles(); p.store_r(R)
torch.cuda.synchronize()
print("done", args.config)
