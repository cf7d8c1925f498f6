"""NEXT-2: the paper's per-tile operation times measured on this B200 (Fig. 4 analog),
the device selection they drive (Alg. 2 main device P:L747-768, Alg. 3 + Eqs. 10-11 number of
devices P:L811-995), and the predicted-vs-actual table (Table III analog).

    python tools/device_select.py [--ncols 148] [--out profiles/r02_device_select.json]

Every time is a CUDA-event device time of the library's own kernels (no host overhead):
  T  (GEQRT)  panel kernel of a 1 x 1 tile plan (tqr_kernel_stats which = 1)
  E  (TSQRT)  (panel(p = 16) - panel(p = 1)) / 15: the per-tile increment of the TS chain
  UT (UNMQR)  update kernel applying one diagonal tile's Q^T to ncols tile columns, / ncols
  UE (TSMQR)  (update(p = 16) - update(p = 1)) / (15 ncols): the per-tile increment of the chain
UT and UE are throughput times with the GPU full (ncols tile columns x nb/32 CTAs in flight), the
way the bulk trailing update runs; T and E are latencies (one panel at a time, the way the
critical path runs).  The update kernel is timed through tqr_apply_qt on a device B (the same
launch the trailing update uses); the staging copies apply_qt adds are timed separately with
the same byte counts and subtracted.
Link speed speed(x, y) of Eq. 11: measured peer-to-peer copy bandwidth when this process sees
>= 2 GPUs; otherwise the NVLink 5 nominal 900 GB/s per direction, stated as such in the output.
"actual": best GPU count measured by the driver's SCALE_rNN.json when present (else null).
"""
import argparse
import glob
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_icpp_kimp13_b200 as tqr  # noqa: E402
from bench import CONFIGS, flops  # noqa: E402


def ev_time(fn, reps=5):
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


def panel_time(p, nb, ib, g, reps=5):
    m = p * nb
    A0 = torch.randn((nb, m), dtype=torch.float64, device="cuda", generator=g).t()
    plan = tqr.Plan(m, nb, nb, ib, tree_domain=-1, profile=True)
    best = 1e30
    for _ in range(reps + 1):
        plan.load(A0)
        plan.kernel_stats(1, reset=True)
        plan.factor_tiles()
        c, ms, _ = plan.kernel_stats(1, reset=True)
        best = min(best, ms * 1e-3 / max(c, 1))
    return plan, A0, best


def update_time(plan, m, nb, ncols, g):
    B = torch.randn((ncols * nb, m), dtype=torch.float64, device="cuda", generator=g).t()
    t_apply = ev_time(lambda: plan.apply_qt(B, "T"))
    # apply_qt's own staging: memset + copy in + copy out of an (p nb) x (ncols nb) block
    W = torch.empty_like(B)
    t_stage = ev_time(lambda: (W.zero_(), W.copy_(B), B.copy_(W)))
    return max(t_apply - t_stage, 1e-9)


def tile_times(nb, ib, ncols):
    g = torch.Generator(device="cuda").manual_seed(1)
    plan1, _, t_p1 = panel_time(1, nb, ib, g)
    plan16, _, t_p16 = panel_time(16, nb, ib, g)
    u1 = update_time(plan1, nb, nb, ncols, g)
    u16 = update_time(plan16, 16 * nb, nb, ncols, g)
    plan1.close()
    plan16.close()
    return {"T": t_p1, "E": max((t_p16 - t_p1) / 15.0, 0.0), "UT": u1 / ncols,
            "UE": max((u16 - u1) / (15.0 * ncols), 0.0)}


def link_speed():
    if torch.cuda.device_count() >= 2:
        x = torch.empty(256 << 20, dtype=torch.uint8, device="cuda:0")
        y = torch.empty(256 << 20, dtype=torch.uint8, device="cuda:1")
        t = ev_time(lambda: y.copy_(x, non_blocking=True))
        return x.numel() / t, "measured cuda:0 -> cuda:1 copy, 256 MiB"
    return 900e9, "nominal NVLink 5, 900 GB/s per direction (one GPU visible: not measurable here)"


def actual_best():
    """{config: best N} from the driver's scaling runs, if any were recorded."""
    out = {}
    for f in sorted(glob.glob(os.path.join(ROOT, "SCALE_r*.json"))):
        try:
            d = json.load(open(f))
        except Exception:
            continue
        runs = d.get("runs") or d.get("results") or []
        for r in runs if isinstance(runs, list) else []:
            try:
                line = r.get("parsed") or r
                cfg, n, v = line["config"]["workload"], line["n_gpus"], line["value"]
                if cfg not in out or v > out[cfg][1]:
                    out[cfg] = (n, v)
            except Exception:
                continue
    return {k: v[0] for k, v in out.items()}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--ncols", type=int, default=148)
    ap.add_argument("--ndev", type=int, default=8)
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    speed, speed_src = link_speed()
    res = {"link_bytes_per_s": speed, "link_source": speed_src, "ndev": args.ndev, "ncols": args.ncols,
           "method": __doc__.strip().split("\n\n")[1], "configs": {}}
    actual = actual_best()
    cache = {}
    for name in ("C1", "C2", "C3", "C4", "C5"):
        m, n, nb, ib, _ = CONFIGS[name]
        if (nb, ib) not in cache:
            cache[(nb, ib)] = tile_times(nb, ib, args.ncols)
        t = cache[(nb, ib)]
        times = [(t["T"], t["E"], t["UT"], t["UE"])] * args.ndev
        sp = [[speed] * args.ndev for _ in range(args.ndev)]
        main_dev = tqr.tqr_select_main(times)
        M, N = -(-m // nb), -(-n // nb)
        order, Tp, pb = tqr.tqr_select_ndev(M, N, nb, 8, times, sp, main_dev)
        res["configs"][name] = {
            "m": m, "n": n, "nb": nb, "ib": ib, "M": M, "N": N,
            "tile_times_us": {k: round(v * 1e6, 3) for k, v in t.items()},
            "tile_tflops": {"T": round(4.0 / 3.0 * nb ** 3 / t["T"] / 1e12, 3),
                            "E": round(2.0 * nb ** 3 / max(t["E"], 1e-12) / 1e12, 3),
                            "UT": round(2.0 * nb ** 3 / max(t["UT"], 1e-12) / 1e12, 3),
                            "UE": round(4.0 * nb ** 3 / max(t["UE"], 1e-12) / 1e12, 3)},
            "main": main_dev, "order": order,
            "predicted_first_iteration_ms": {str(p + 1): round(x * 1e3, 4) for p, x in enumerate(Tp)},
            "predicted_best_ndev": pb,
            "actual_best_ndev": actual.get(name),
            "flops": flops(m, n),
        }
        print(name, "M x N = %d x %d" % (M, N), "tile us", res["configs"][name]["tile_times_us"],
              "tile TF", res["configs"][name]["tile_tflops"], "T(p) ms",
              res["configs"][name]["predicted_first_iteration_ms"], "-> p =", pb, "actual", actual.get(name),
              flush=True)
    if args.out:
        with open(args.out, "w") as f:
            json.dump(res, f, indent=1)


if __name__ == "__main__":
    main()
