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
