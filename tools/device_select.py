"""Measure the paper's per-tile operation times on this B200 and run the device selection
(Alg. 2 main device, Alg. 3 + Eqs. 10-11 number of devices) for the BASELINE configs.

    python tools/device_select.py [--link-gbs 700] [--out profiles/r01_device_select.json]

time(T), time(E): a p x 1 tile column factored with the flat chain (tree_domain = -1):
    t(p) = time(T) + (p - 1) time(E), from p = 2 and p = 16 (two solves, least squares).
time(UT), time(UE): the whole-GPU throughput of the update kernel -- Q^T applied to a 16 x 1
    factorisation's right-hand side of 18 tile columns (n_rhs = 18 nb): 18 (UT + 15 UE);
    UT = UE / 2 by the flop ratio (2 nb^3 vs 4 nb^3).
The NVLink speed cannot be measured on one GPU: --link-gbs (default 700 GB/s, the NCCL broadcast
bandwidth SURVEY 8(a7) assumes) is an input, stated in the output.
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


def timed(fn, reps=5):
    fn()
    torch.cuda.synchronize()
    best = 1e30
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1) * 1e-3)
    return best


def tile_times(nb, ib):
    g = torch.Generator(device="cuda").manual_seed(1)
    tp = {}
    for p in (2, 16):
        m = p * nb
        A0 = torch.randn((nb, m), dtype=torch.float64, device="cuda", generator=g).t()
        plan = tqr.Plan(m, nb, nb, ib, tree_domain=-1)

        def f():
            plan.load(A0)
            plan.factor_tiles()
        # factor_tiles alone: the load is a separate phase, subtract it
        t_all = timed(f)
        t_load = timed(lambda: plan.load(A0))
        tp[p] = t_all - t_load
        if p == 16:
            f()
            B0 = torch.randn((18 * nb, m), dtype=torch.float64, device="cuda", generator=g).t()
            B = B0.clone()
            t_app = timed(lambda: plan.apply_qt(B, "T"))
            t_copy = 0.0
        plan.close()
    tE = (tp[16] - tp[2]) / 14.0
    tT = max(tp[2] - tE, 0.0)
    # 18 tile columns x (UT + 15 UE), UT = UE / 2
    tUE = (t_app - t_copy) / (18.0 * (0.5 + 15.0))
    return {"T": tT, "E": tE, "UT": 0.5 * tUE, "UE": tUE}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--link-gbs", type=float, default=700.0)
    ap.add_argument("--ndev", type=int, default=8)
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    res = {"link_gbs": args.link_gbs, "ndev": args.ndev, "configs": {}}
    cache = {}
    for name in ("C1", "C2", "C3", "C4", "C5"):
        m, n, nb, ib, _ = CONFIGS[name]
        if (nb, ib) not in cache:
            cache[(nb, ib)] = tile_times(nb, ib)
        t = cache[(nb, ib)]
        times = [(t["T"], t["E"], t["UT"], t["UE"])] * args.ndev
        speed = [[args.link_gbs * 1e9] * args.ndev for _ in range(args.ndev)]
        main_dev = tqr.tqr_select_main(times)
        M, N = -(-m // nb), -(-n // nb)
        order, Tp, pb = tqr.tqr_select_ndev(M, N, nb, 8, times, speed, main_dev)
        res["configs"][name] = {"nb": nb, "ib": ib, "M": M, "N": N,
                                "tile_times_us": {k: round(v * 1e6, 3) for k, v in t.items()},
                                "main": main_dev, "order": order,
                                "T_p_ms": [round(x * 1e3, 4) for x in Tp], "p_best": pb}
        print(name, "M x N = %d x %d" % (M, N), "tile us", res["configs"][name]["tile_times_us"],
              "T(p) ms", res["configs"][name]["T_p_ms"], "-> p =", pb, flush=True)
    if args.out:
        with open(args.out, "w") as f:
            json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
