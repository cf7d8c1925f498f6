"""Full-size elementwise parity at bench configurations (test infrastructure, GPU box):
the GPU factorization in the bench launch configuration (tqr_load + tqr_factor_tiles +
tqr_store_r on the device, inputs = bench.py's seeded torch.randn matrix) against the CPU oracle
(Algorithm 1, all host cores) on the SAME matrix, every entry of R compared (sign-normalised,
column-norm relative, reading Q16), plus ||A - QR||_F / ||A||_F via tqr_apply_qt('N') (GPU).

    python tools/full_parity.py C3 C4 [--out profiles/r01_full_parity.json]
"""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_icpp_kimp13_b200 as tqr  # noqa: E402
from bench import CONFIGS  # noqa: E402


def main():
    args = [a for a in sys.argv[1:] if not a.startswith("--")]
    out = sys.argv[sys.argv.index("--out") + 1] if "--out" in sys.argv else None
    if out in args:
        args.remove(out)
    res = {}
    for cfg in args:
        m, n, nb, ib, seed = CONFIGS[cfg]
        g = torch.Generator(device="cuda").manual_seed(seed)
        A0 = torch.randn((n, m), dtype=torch.float64, device="cuda", generator=g).t()
        R = torch.empty((n, m), dtype=torch.float64, device="cuda").t()
        plan = tqr.Plan(m, n, nb, ib)
        plan.load(A0)
        plan.factor_tiles()
        plan.store_r(R)
        torch.cuda.synchronize()
        # residual on the GPU: Q [R; 0] vs A
        QR = R.clone()
        plan.apply_qt(QR, "N")
        res_gpu = float((QR - A0).norm() / A0.norm())
        del QR
        Rg = np.triu(R[:n].cpu().numpy())
        A = np.asfortranarray(A0.cpu().numpy())
        plan.close()
        del R, A0
        torch.cuda.empty_cache()
        t0 = time.time()
        Ro = oracle.qr(A).R
        t_or = time.time() - t0
        d1 = np.where(np.diag(Rg) < 0, -1.0, 1.0)
        d2 = np.where(np.diag(Ro) < 0, -1.0, 1.0)
        cn = np.linalg.norm(Ro, axis=0)
        err = float(np.max(np.abs(Rg * d1[:, None] - Ro * d2[:, None]) / cn[None, :]))
        res[cfg] = {"m": m, "n": n, "nb": nb, "ib": ib, "seed": seed, "entries_compared": n * (n + 1) // 2,
                    "R_colnorm_rel_err_max": err, "R_tol": 1e-10, "residual_gpu": res_gpu, "residual_tol": 1e-13,
                    "oracle_seconds": round(t_or, 1), "oracle_threads": oracle.num_threads(),
                    "pass": bool(err <= 1e-10 and res_gpu <= 1e-13)}
        print(cfg, json.dumps(res[cfg]), flush=True)
    if out:
        with open(out, "w") as f:
            json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
