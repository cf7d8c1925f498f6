"""Phase timing of apply_block (probe build with -DTQR_PHASE_PROF): clock64 deltas of warp 0."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import torch
import paper_conf_icpp_kimp13_b200 as tqr
from paper_conf_icpp_kimp13_b200 import build
cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
lib_path = os.path.join(build.OBJ, "libtqr_phaseprof.so")
tqr.LIB_PATH = lib_path
L = tqr.lib()
L.tqr_probe_phases.argtypes = [ctypes.POINTER(ctypes.c_ulonglong), ctypes.c_int]
from bench import CONFIGS
m, n, nb, ib, seed = CONFIGS[cfg]
g = torch.Generator(device="cuda").manual_seed(seed)
A = torch.randn((n, m), dtype=torch.float64, device="cuda", generator=g).t()
R = torch.empty((n, m), dtype=torch.float64, device="cuda").t()
buf = (ctypes.c_ulonglong * 36)()
with tqr.Plan(m, n, nb, ib) as p:
    p.load(A); p.factor_tiles(); p.store_r(R)
    L.tqr_probe_phases(buf, 1)
    p.load(A); p.factor_tiles(); p.store_r(R)
    torch.cuda.synchronize()
    L.tqr_probe_phases(buf, 0)
names = ["T cp.async+top ld", "GEMM1 half A", "GEMM1 half B", "stage1 st+sync", "RMW+sync", "wait V half A",
         "T-DMMA+sync", "top store", "GEMM2 half A", "GEMM2 half B", "-", "wait V half B"]
tot = sum(buf[i] for i in range(12))
for i, nm in enumerate(names):
    print("%-20s %6.2f%%" % (nm, 100.0 * buf[i] / tot))

pt = sum(buf[16 + i] for i in range(4))
if pt:
    print("panel last-leader chain:", ", ".join("%s %.1f%%" % (nm, 100.0 * buf[16 + i] / pt) for i, nm in
          enumerate(["flag waits", "applies", "gather+factor", "publish"])), "total Mcycles %.1f" % (pt / 1e6))
dt = sum(buf[20 + i] for i in range(3))
if dt:
    print("domain kernel (last CTA):", ", ".join("%s %.1f%%" % (nm, 100.0 * buf[20 + i] / dt) for i, nm in
          enumerate(["applies", "factor", "store+image+T"])), "total Mcycles %.1f" % (dt / 1e6))
ft = sum(buf[24 + i] for i in range(3))
if ft:
    print("factor_block (last CTA): columns %.1f Mcyc, Gram %.1f Mcyc, dlarft recurrence %.1f Mcyc" %
          tuple(buf[24 + i] / 1e6 for i in range(3)))
ct = sum(buf[28 + i] for i in range(6))
if ct:
    print("factor_block column step (last CTA):", ", ".join("%s %.1f%%" % (nm, 100.0 * buf[28 + i] / ct) for i, nm in
          enumerate(["shuffle+scale", "dots+record", "barrier", "sums+sqrt/div", "w_j", "update+store"])),
          "total Mcycles %.1f" % (ct / 1e6))
