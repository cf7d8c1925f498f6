"""Driver of tests/test_gpu_sanitizer.py: small factorizations + apply/solve over every kernel family
(flat, logical owners, lookahead, streamed I/O, tree + merge, tall streamed, row split) run under
compute-sanitizer; prints "ok <m n nb ib>" per case and "ok extra" at the end."""
import sys, os
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import paper_conf_icpp_kimp13_b200 as tqr
import synthetic
for (m, n, nb, ib) in [(256, 256, 64, 16), (512, 256, 128, 32), (1024, 1024, 512, 32)]:
    A = synthetic.gaussian(m, n, 3)
    Ad = torch.from_numpy(np.ascontiguousarray(A.T)).cuda().t()
    with tqr.Plan(m, n, nb, ib) as p:
        p.factor(Ad)
        B = torch.from_numpy(np.ascontiguousarray(synthetic.gaussian(m, 3, 4).T)).cuda().t()
        p.apply_qt(B, "T"); p.apply_qt(B, "N")
    with tqr.Plan(m, n, nb, ib, ndev=2, logical_devices=True) as p:
        Ad = torch.from_numpy(np.ascontiguousarray(A.T)).cuda().t()
        p.factor(Ad)
    print("ok", m, n, nb, ib, flush=True)
# round-1 additions: tile back substitution, streamed host I/O, tree jobs + two-level merge,
# streamed tall factor, row split
m, n, nb, ib = 512, 256, 128, 32
A = synthetic.gaussian(m, n, 5)
with tqr.Plan(m, n, nb, ib) as p:
    Ah = torch.from_numpy(np.ascontiguousarray(A.T)).pin_memory().t()
    p.factor(Ah)
    B = torch.from_numpy(np.ascontiguousarray(synthetic.gaussian(m, 40, 6).T)).cuda().t()
    p.solve_ls(B)
A = synthetic.gaussian(2048, 128, 7)
with tqr.Plan(2048, 128, 64, 16, tree_domain=1, tree_group=4) as p:
    Ad = torch.from_numpy(np.ascontiguousarray(A.T)).cuda().t()
    p.factor(Ad)
    B = torch.from_numpy(np.ascontiguousarray(synthetic.gaussian(2048, 3, 8).T)).cuda().t()
    p.apply_qt(B, "T"); p.apply_qt(B, "N")
os.environ["TQR_TREE_ONE_CTA"] = "1"
A = synthetic.gaussian(2048, 64, 9)
with tqr.Plan(2048, 64, 64, 16) as p:
    Ah = torch.from_numpy(np.ascontiguousarray(A.T)).pin_memory().t()
    p.factor(Ah)
with tqr.Plan(2048, 64, 64, 16, ndev=2, logical_devices=True, row_split=1) as p:
    Ad = torch.from_numpy(np.ascontiguousarray(A.T)).cuda().t()
    p.factor(Ad)
print("ok extra", flush=True)
