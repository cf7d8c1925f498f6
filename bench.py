#!/usr/bin/env python
"""bench.py -- tiled-QR throughput on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C5] [--dtype f64|f32]
                    [--impl ours|reference]

metric : tiled QR GFLOP/s = (2mn^2 - 2n^3/3) / t, whole job, plus % of the FP64 tensor peak.
step   : one pass of the whole hot path over the config's matrix:
         tqr_load (col-major -> tiles) + tqr_factor_tiles (GEQRT/TSQRT panels, UNMQR/TSMQR
         updates, lookahead, broadcasts) + tqr_store_r (R out).  Input resident in HBM.
e2e    : the same through tqr_factor on a PINNED HOST A (H2D of A and D2H of R inside the
         timed region, pipelined with the factorization by the library).
N > 1  : one process per GPU (bench.py starts the N ranks itself with torchrun when WORLD_SIZE is
         unset), column tiles partitioned by a guide array (Eq. 12; --guide: cyclic {0..N-1}, or
         pairs {0,0,1,1,..} -- default for N >= 8); each panel travels from its owner to the other
         ranks by the library's CUDA-IPC transport (device-to-device copies into the receivers'
         IPC-mapped slots over NVLink, ordered by stream flags; --transport nccl: ncclBroadcast);
         a single column tile (C4) is split by rows instead (row split).  Strong scaling (same
         matrix).  More ranks than GPUs (testing on one GPU): ranks share GPUs, n_gpus counts GPUs.
--impl reference : the CPU oracle (Algorithm 1, oracle/) timed on this host's cores on a
         bounded sample of the same workload (first 2048 columns of the config's matrix).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

CONFIGS = {
    # name: (m, n, nb, ib, seed)  -- BASELINE.json configs
    "C1": (256, 256, 64, 16, 101),
    "C2": (4096, 4096, 256, 32, 102),
    "C3": (16384, 16384, 512, 32, 103),
    "C4": (1048576, 512, 512, 32, 104),
    "C5": (32768, 32768, 512, 32, 105),
}
DEFAULT_CONFIG = "C5"
L2_BYTES = 126 * 2 ** 20
SAMPLE_COLS = int(os.environ.get("TQR_ORACLE_SAMPLE_COLS", "2048"))


METRIC = "tiled QR GFLOP/s (2mn^2-2n^3/3) at 1/2/4/8 B200, % of FP64 tensor peak"


def flops(m, n):
    return 2.0 * m * n * n - 2.0 * n ** 3 / 3.0


def fp64_peak_tflops():
    """Measured DMMA.8x8x4 peak (profiles/fp64_peak.json, own microbenchmark on this pool)."""
    try:
        with open(os.path.join(ROOT, "profiles", "fp64_peak.json")) as f:
            d = json.load(f)
        return float(d["dmma_tflops"]), d.get("source", "profiles/fp64_peak.json")
    except Exception:
        return 37.2, "nominal 148 SM x 64 FMA/clk x 2 x 1.965 GHz"


def fp32_peak_tflops():
    """FFMA peak (FP32 SIMT pipe): measured by tools/probes/fp32_peak.cu if recorded, else derived
    from the unit counts: 148 SM x 4 SMSP x 32 lanes x 2 flop x 1.965 GHz = 74.4 TFLOP/s."""
    try:
        with open(os.path.join(ROOT, "profiles", "fp32_peak.json")) as f:
            d = json.load(f)
        return float(d["ffma_tflops"]), d.get("source", "profiles/fp32_peak.json")
    except Exception:
        return 148 * 4 * 32 * 2 * 1.965e-3, "derived: 148 SM x 128 FP32 lanes x 2 x 1.965 GHz"


def load_profile_summary(cfg):
    """ncu summary of the dominant kernel for this config (profiles/ncu_update_<cfg>.json)."""
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_update_%s.json" % cfg)) as f:
            return json.load(f)
    except Exception:
        return {}


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), "--query-gpu=" + self.Q,
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in self.rows:
            try:
                sm.append(float(r[1]))
                mx = float(r[2])
                for i, nm in enumerate(names):
                    if r[5 + i].lower().startswith("active"):
                        reasons.add(nm)
            except Exception:
                continue
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


def oracle_sample(cfg_name, nthreads=0, ncols=None):
    """Bounded CPU-oracle sample of the config: Algorithm 1 on the first min(n, 2048) (or ncols)
    columns of the config's own matrix (same generator, same rows; ~10 s of host work for C5).
    Returns (GFLOP/s, seconds, desc)."""
    import numpy as np
    import oracle
    import synthetic
    m, n, nb, ib, seed = CONFIGS[cfg_name]
    ns = min(n, SAMPLE_COLS if ncols is None else ncols)
    rows = np.arange(m, dtype=np.uint64)
    A = np.empty((m, ns), order="F")
    for j in range(ns):
        A[:, j] = synthetic.gaussian_entries(m, rows, np.full(m, j, dtype=np.uint64), seed)
    t0 = time.perf_counter()
    oracle.qr(A, nthreads=nthreads)
    dt = time.perf_counter() - t0
    return flops(m, ns) / dt / 1e9, dt, "oracle.qr on A[:, :%d] of %s (%dx%d), %s, %.2f s" % (
        ns, cfg_name, m, ns, "1 thread" if nthreads == 1 else "all host cores", dt)


def run_reference(args):
    """--impl reference: the CPU oracle as it stands, on this host's cores."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import oracle
    cores = oracle.num_threads()
    for _ in range(args.warmup):
        oracle_sample(args.config)
    vals, times = [], []
    for _ in range(args.steps):
        v, dt, desc = oracle_sample(args.config)
        vals.append(v)
        times.append(dt)
    m, n, nb, ib, seed = CONFIGS[args.config]
    value = statistics.median(vals)
    line = {
        "impl": "reference", "metric": METRIC, "value": round(value, 3),
        "unit": "GFLOP/s", "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(1e3 * statistics.median(times), 3), "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": args.config, "m": m, "n": n, "nb": nb, "ib": ib, "seed": seed,
                   "parallelism": "oracle on the host cores (rank 0 only)",
                   "sample": "first %d columns" % min(n, SAMPLE_COLS)},
        "cpu_baseline": {"value": round(value, 3), "unit": "GFLOP/s", "cores": cores, "kind": "oracle",
                         "sample": desc},
        "e2e": {"value": round(value, 3), "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "gpu_launches": 0,
    }
    print(json.dumps(line), flush=True)
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default=DEFAULT_CONFIG, choices=sorted(CONFIGS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--dtype", default="f64", choices=["f64", "f32"],
                    help="f32: the C5 FP32 configuration (FFMA updates)")
    ap.add_argument("--ib", type=int, default=0,
                    help="inner block ib (default: the config's; C3-C5 leave ib open, SURVEY 8)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-lookahead", action="store_true")
    ap.add_argument("--tree", type=int, default=0,
                    help="elimination tree: 0 auto (tree for q == 1), -1 flat TS, L > 0 TS domains of L tiles")
    ap.add_argument("--guide", default="auto", choices=["auto", "cyclic", "pairs", "snake"],
                    help="N > 1 column distribution (Eq. 12 guide array): cyclic {0..N-1}; pairs "
                         "{0,0,1,1,..}; snake {0..N-1, N-1..0} (balances the trailing work, which grows "
                         "with the column index: max/mean per-GPU work 1.008 at C5 on 8 GPUs vs 1.082 "
                         "cyclic and 1.158 pairs); auto = snake")
    ap.add_argument("--solve", type=int, default=0,
                    help="also time tqr_solve_ls with this many right-hand sides (NEXT-3; 'solve' key)")
    ap.add_argument("--tree-group", type=int, default=0,
                    help="tree merge: 0 auto (two-level for >= 16 domains), -1 flat chain, G > 1 groups of G")
    ap.add_argument("--transport", default="ipc", choices=["ipc", "nccl"],
                    help="N > 1 panel transport: ipc = the library's own CUDA-IPC peer copies + stream "
                         "flags (default); nccl = ncclBroadcast")
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)

    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world == 1 and args.gpus > 1:
        # started without torchrun: launch the N ranks ourselves (one process per GPU), rank 0
        # prints the JSON line
        import socket
        with socket.socket() as sk:
            sk.bind(("127.0.0.1", 0))
            port = sk.getsockname()[1]
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes", "1", "--nproc-per-node", str(args.gpus),
               "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
        return subprocess.call(cmd)

    import torch
    import paper_conf_icpp_kimp13_b200 as tqr

    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    ndevices = torch.cuda.device_count()
    device = local_rank % ndevices          # more ranks than GPUs: ranks share GPUs (tests / smoke)
    torch.cuda.set_device(device)
    shared = world > ndevices
    n_gpus = min(world, ndevices)
    dist = None
    if world > 1:
        import torch.distributed as dist
        if shared or args.transport == "ipc":
            dist.init_process_group("gloo")          # host-side handshake + barriers only
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", device))

    m, n, nb, ib, seed = CONFIGS[args.config]
    if args.ib:
        ib = args.ib
    f32 = args.dtype == "f32"
    tdt = torch.float32 if f32 else torch.float64
    es = 4 if f32 else 8
    W = max(args.warmup, 3)
    K = max(args.steps, 1)

    # ---- inputs (seeded synthetic N(0,1), generated on the device; identical on every rank)
    gen = torch.Generator(device="cuda").manual_seed(seed)
    A0 = torch.randn((n, m), dtype=tdt, device="cuda", generator=gen).t()   # column-major m x n
    Rout = torch.empty((n, m), dtype=tdt, device="cuda").t()

    nccl_id = None
    if world > 1 and args.transport == "nccl":
        obj = [tqr.tqr_nccl_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0)
        nccl_id = obj[0]
    gmode = args.guide if args.guide != "auto" else "snake"
    if world == 1:
        guide = [0]
    elif gmode == "snake":
        guide = list(range(world)) + list(range(world - 1, -1, -1))
    else:
        guide = [d for d in range(world) for _ in range(2 if gmode == "pairs" else 1)]
    plan = tqr.Plan(m, n, nb, ib, dtype=tqr.TQR_F32 if f32 else tqr.TQR_F64, ndev=world, guide=guide,
                    rank=rank, world=world, nccl_id=nccl_id,
                    transport=("nccl" if args.transport == "nccl" else "ipc") if world > 1 else "auto",
                    lookahead=not args.no_lookahead, profile=True, tree_domain=args.tree,
                    tree_group=args.tree_group)
    if world > 1 and args.transport == "ipc":
        plan.connect()
    pflags = plan.flags()

    def step(Ain, Aout):
        plan.load(Ain)
        plan.factor_tiles()
        plan.store_r(Aout)

    def barrier():
        if dist is not None:
            dist.barrier()

    def max_over_ranks(x):
        if dist is None:
            return x
        t = torch.tensor([x], dtype=torch.float64)
        if dist.get_backend() == "nccl":
            t = t.cuda()
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    for _ in range(W):
        step(A0, Rout)
    torch.cuda.synchronize()
    plan.kernel_stats(0, reset=True)
    plan.kernel_stats(1, reset=True)
    plan.launch_count()

    stream = torch.cuda.current_stream()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(device) as clk:
        barrier()
        torch.cuda.synchronize()
        ev0.record(stream)
        for _ in range(K):
            step(A0, Rout)
        ev1.record(stream)
        torch.cuda.synchronize()
        barrier()
    ms = ev0.elapsed_time(ev1) / K
    ms = max_over_ranks(ms)
    launches = plan.launch_count() // K
    ucount, ums, uflops = plan.kernel_stats(0, reset=True)
    pcount, pms, pflops = plan.kernel_stats(1, reset=True)
    fl = flops(m, n)
    value = fl / (ms * 1e-3) / 1e9
    peak, peak_src = fp32_peak_tflops() if f32 else fp64_peak_tflops()

    # ---- e2e: the public call a user makes, tqr_factor on a pinned host A (in place: A <- R).
    # The library pipelines the host->device column loads and the device->host R stores with the
    # factorization; both copies are inside the timed region.  A is restored from the pristine
    # copy between iterations (untimed).
    e2e = None
    if not args.no_e2e:
        Ah = torch.empty((n, m), dtype=tdt, pin_memory=True).t()
        Ah.copy_(A0)
        plan.factor(Ah)
        torch.cuda.synchronize()
        ke = max(1, min(K, 2))
        tot = 0.0
        for _ in range(ke):
            Ah.copy_(A0)
            torch.cuda.synchronize()
            barrier()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            plan.factor(Ah)
            e1.record(stream)
            torch.cuda.synchronize()
            tot += e0.elapsed_time(e1)
        ems = max_over_ranks(tot / ke)
        e2e = {"value": round(fl / (ems * 1e-3) / 1e9, 3), "unit": "GFLOP/s",
               "ms_per_step": round(ems, 3), "h2d_bytes_per_step": es * m * n, "d2h_bytes_per_step": es * m * n,
               "api": "tqr_factor(pinned host A): H2D + layout convert and R-out + D2H pipelined with the "
                      "factorization inside the call (per column tile; per row chunk of TS domains for a "
                      "single tile column)"}
        del Ah

    # ---- least squares throughput (NEXT-3): Q^T B (update kernel) + tile back substitution on a
    # device-resident B of --solve columns; B restored from a pristine copy between calls (untimed)
    solve = None
    if args.solve > 0:
        nr = args.solve
        gen_b = torch.Generator(device="cuda").manual_seed(seed + 1)
        B0 = torch.randn((nr, m), dtype=tdt, device="cuda", generator=gen_b).t()
        Bw = torch.empty((nr, m), dtype=tdt, device="cuda").t()
        plan.load(A0)
        plan.factor_tiles()
        Bw.copy_(B0)
        plan.solve_ls(Bw)
        torch.cuda.synchronize()
        st = 0.0
        for _ in range(K):
            Bw.copy_(B0)
            torch.cuda.synchronize()
            s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s0.record(stream)
            plan.solve_ls(Bw)
            s1.record(stream)
            torch.cuda.synchronize()
            st += s0.elapsed_time(s1)
        sms = st / K
        sfl = (4.0 * m * n - 1.0 * n * n) * nr      # Q^T B (4mn - 2n^2) + back substitution (n^2) per RHS
        solve = {"nrhs": nr, "ms": round(sms, 3), "gflops": round(sfl / (sms * 1e-3) / 1e9, 3),
                 "flops": "(4mn - n^2) nrhs: Householder Q^T B (4mn - 2n^2) + tile back substitution (n^2)"}
        del B0, Bw

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        import oracle
        v, dt, desc = oracle_sample(args.config)
        cpu = {"value": round(v, 3), "unit": "GFLOP/s", "cores": oracle.num_threads(), "kind": "oracle",
               "sample": desc}
        # the oracle on one thread as well (a narrower sample: ~1-3 s of host work)
        mm, nn = CONFIGS[args.config][0], CONFIGS[args.config][1]
        ns1 = int(min(256, nn, max(32, (2e10 / mm) ** 0.5)))      # <= ~2e10 flops of 1-thread work
        v1, dt1, desc1 = oracle_sample(args.config, nthreads=1, ncols=ns1)
        cpu["single_thread"] = {"value": round(v1, 3), "unit": "GFLOP/s", "cores": 1, "sample": desc1}

    if rank == 0:
        # achieved = algorithmic flops of all bulk-update launches / their device-busy time
        # (union of the launches' CUDA-event intervals on the 4 update streams; the launches of
        # one step overlap, so a per-launch average duration would not be a kernel duration)
        achieved = (uflops / (ums * 1e-3) / 1e12) if ucount else None
        prof = load_profile_summary(args.config + ("_f32" if f32 else ""))
        if ucount and ums >= pms:
            # dominant kernel: the bulk trailing update
            roofline = {"bound": "alu" if f32 else "tensor",
                        "kernel": "update_kernel32<%d,32,%d> (UNMQR+TSMQR chain, FFMA)" % (nb, ib) if f32 else
                        ("update_kernel16<%d,%d> (UNMQR+TSMQR chain, 16 warps, DMMA.8x8x4)" % (nb, ib)
                         if nb >= 256 and os.environ.get("TQR_W16", "1") != "0" else
                         "update_kernel<%d,32,%d> (UNMQR+TSMQR chain, DMMA.8x8x4)" % (nb, ib)),
                        "achieved": round(achieved, 3), "peak": peak, "unit": "TFLOP/s",
                        "frac": round(achieved / peak, 4),
                        "traffic": prof.get("dram_bytes_per_launch"), "traffic_note": prof.get("note"),
                        "peak_source": peak_src, "launches_per_step": ucount // K,
                        "busy_ms_per_step": round(ums / K, 3), "share_of_step": round(ums / K / ms, 3)}
        else:
            # dominant kernel: the panel step (C4: one column -> the whole factorisation is panel
            # work: TS-domain kernel + TT merge chain in tree mode; C1/C2: the flat panel wavefront)
            pach = pflops / max(pms, 1e-9) / 1e9
            roofline = {"bound": "alu" if f32 else "tensor",
                        "kernel": ("panel step (domain_kernel<%d,%d> + merge panel_kernel, DMMA.8x8x4)" % (nb, ib))
                        if pflags & tqr.PLAN_TREE else
                        ("panel_kernel<%d,%d> (GEQRT + flat TSQRT wavefront, factor_block + DMMA applies)" % (nb, ib)),
                        "achieved": round(pach, 3), "peak": peak, "unit": "TFLOP/s", "frac": round(pach / peak, 4),
                        "traffic": prof.get("dram_bytes_per_launch"), "traffic_note": prof.get("note"),
                        "peak_source": peak_src, "launches_per_step": pcount // K,
                        "busy_ms_per_step": round(pms / K, 3), "share_of_step": round(pms / K / ms, 3)}
            if pach / peak < 0.1:
                roofline["note"] = ("the panel chain (GEQRT + TSQRT wavefront, one ib block after another) is "
                                    "latency-bound here (SURVEY 8(d): no roofline claim for C1/C2): the step is "
                                    "the critical path of the flat TS panels, not a throughput limit")
        line = {
            "metric": METRIC,
            "value": round(value, 3), "unit": "GFLOP/s", "n_gpus": n_gpus, "steps": K, "warmup": W,
            "ms_per_step": round(ms, 3), "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": args.dtype, "data": "synthetic",
            ("pct_fp32_ffma_peak" if f32 else "pct_fp64_peak"): round(100.0 * value / 1e3 / (peak * n_gpus), 2),
            "config": {"workload": args.config, "m": m, "n": n, "nb": nb, "ib": ib, "seed": seed,
                       "input": "torch.randn N(0,1) %s on device (seeded)" % args.dtype, "guide": guide,
                       "parallelism": ("row-split x%d (per-rank TS trees + %s gather of the R factors, "
                                       "stage-2 merge on rank 0)" % (world, "IPC" if pflags & tqr.PLAN_IPC else "NCCL"))
                                      if pflags & tqr.PLAN_ROW_SPLIT else
                                      ("col-%s x%d%s" % (gmode, world, (", %s panel transport" %
                                                                        ("CUDA-IPC" if pflags & tqr.PLAN_IPC else "NCCL"))
                                                         if world > 1 else "")),
                       "ranks": world, "ranks_share_gpus": shared, "lookahead": not args.no_lookahead,
                       "tree": args.tree, "tree_group": args.tree_group,
                       "l2": "inputs larger than L2 (%.1f GiB >> 126 MB)" % (es * m * n / 2 ** 30)
                       if es * m * n > L2_BYTES else "input fits L2 (no flush)"},
            "roofline": roofline,
            "panel": {"launches": pcount, "avg_ms": round(pms / max(pcount, 1), 3),
                      "tflops": round(pflops / max(pms, 1e-9) / 1e9, 3) if pcount else None},
            "clocks": clk.summary(),
            "gpu_launches": launches,
            "e2e": e2e,
            "cpu_baseline": cpu,
        }
        if solve is not None:
            line["solve"] = solve
        print(json.dumps(line), flush=True)
    plan.close()
    if dist is not None:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
