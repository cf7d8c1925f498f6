"""Full-size parity at the bench configurations (test infrastructure, GPU box).

The GPU factorization in the bench launch configuration (tqr_load + tqr_factor_tiles +
tqr_store_r on the device; input = bench.py's own seeded torch.randn matrix, FP64 or FP32) is
checked against:
  * the CPU oracle (Algorithm 1, all host cores) on the SAME matrix: every entry of R
    (sign-normalised, column-norm relative, reading Q16; FP32: the FP64 oracle on the FP32 input);
  * the residual ||A - QR||_F / ||A||_F and the thin-Q orthogonality ||Q^T Q - I||_F (Q = Q [I; 0]
    through tqr_apply_qt('N'), reading Q18), each next to cuSOLVER's Householder QR
    (torch.linalg.qr) on the same matrix, and ||Q^T Q - I||_F / (sqrt(n) eps) (reading Q19).

    python tools/full_parity.py C2 C3 C5 [--f32 C5] [--out profiles/r02_full_parity.json]
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

BARS = {"f64": (1e-10, 1e-13, 1e-13), "f32": (1e-3, 1e-5, 1e-5)}


def orth_of(Q):
    n = Q.shape[1]
    G = Q.t() @ Q
    G.diagonal().sub_(1.0)
    return float(G.norm())


def one(cfg, dts):
    m, n, nb, ib, seed = CONFIGS[cfg]
    f32 = dts == "f32"
    tdt = torch.float32 if f32 else torch.float64
    eps = float(torch.finfo(tdt).eps)
    g = torch.Generator(device="cuda").manual_seed(seed)
    A0 = torch.randn((n, m), dtype=tdt, device="cuda", generator=g).t()        # exactly bench.py's input
    R = torch.empty((n, m), dtype=tdt, device="cuda").t()
    out = {"m": m, "n": n, "nb": nb, "ib": ib, "seed": seed, "dtype": dts}
    plan = tqr.Plan(m, n, nb, ib, dtype=tqr.TQR_F32 if f32 else tqr.TQR_F64)
    t0 = time.time()
    plan.load(A0)
    plan.factor_tiles()
    plan.store_r(R)
    torch.cuda.synchronize()
    out["gpu_seconds"] = round(time.time() - t0, 3)
    A64 = A0.double()
    # residual: Q [R; 0] vs A (GPU apply, norms in FP64)
    QR = R.clone()
    plan.apply_qt(QR, "N")
    out["residual"] = float((QR.double() - A64).norm() / A64.norm())
    del QR
    # thin Q and its orthogonality (FP64 Gram of the stored Q)
    E = torch.zeros((n, m), dtype=tdt, device="cuda").t()
    E[:n, :n] = torch.eye(n, dtype=tdt, device="cuda")
    plan.apply_qt(E, "N")
    out["orth"] = orth_of(E.double())
    del E
    plan.close()
    torch.cuda.empty_cache()
    # cuSOLVER (LAPACK-style blocked Householder) on the same matrix
    Ql, Rl = torch.linalg.qr(A0)
    out["orth_cusolver"] = orth_of(Ql.double())
    out["residual_cusolver"] = float((Ql.double() @ Rl.double() - A64).norm() / A64.norm())
    del Ql, Rl
    torch.cuda.empty_cache()
    out["orth_over_sqrt_n_eps"] = out["orth"] / (np.sqrt(n) * eps)
    out["orth_cusolver_over_sqrt_n_eps"] = out["orth_cusolver"] / (np.sqrt(n) * eps)
    Rg = np.triu(R[:n].double().cpu().numpy())
    A = np.asfortranarray(A64.cpu().numpy())
    del R, A0, A64
    torch.cuda.empty_cache()
    t0 = time.time()
    Ro = oracle.qr(A).R
    out["oracle_seconds"] = round(time.time() - t0, 1)
    out["oracle_threads"] = oracle.num_threads()
    d1 = np.where(np.diag(Rg) < 0, -1.0, 1.0)
    d2 = np.where(np.diag(Ro) < 0, -1.0, 1.0)
    cn = np.linalg.norm(Ro, axis=0)
    cn[cn == 0] = 1.0
    out["entries_compared"] = n * (n + 1) // 2
    out["R_colnorm_rel_err_max"] = float(np.max(np.abs(Rg * d1[:, None] - Ro * d2[:, None]) / cn[None, :]))
    rt, st, ot = BARS[dts]
    out["bars"] = {"R": rt, "residual": st, "orth": ot}
    out["pass_R"] = out["R_colnorm_rel_err_max"] <= rt
    out["pass_residual"] = out["residual"] <= st
    out["pass_orth_absolute"] = out["orth"] <= ot
    out["orth_vs_cusolver"] = out["orth"] / out["orth_cusolver"]
    return out


def main():
    out_path = sys.argv[sys.argv.index("--out") + 1] if "--out" in sys.argv else None
    jobs = []
    argv = sys.argv[1:]
    i = 0
    while i < len(argv):
        a = argv[i]
        if a == "--out":
            i += 2
            continue
        if a == "--f32":
            jobs.append((argv[i + 1], "f32"))
            i += 2
            continue
        jobs.append((a, "f64"))
        i += 1
    res = {}
    if out_path and os.path.exists(out_path):
        with open(out_path) as f:
            res = json.load(f)
    for cfg, dts in jobs:
        key = cfg if dts == "f64" else cfg + "_f32"
        res[key] = one(cfg, dts)
        print(key, json.dumps(res[key]), flush=True)
        if out_path:
            with open(out_path, "w") as f:
                json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
