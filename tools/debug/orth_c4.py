import sys, os
sys.path.insert(0, os.getcwd())
import torch, numpy as np
import paper_conf_icpp_kimp13_b200 as tqr
for (m, n, nb, ib) in [(1048576, 512, 512, 32), (262144, 512, 512, 32), (65536, 512, 512, 32), (1048576, 512, 512, 16), (262144, 512, 256, 32)]:
    gen = torch.Generator(device="cuda").manual_seed(104)
    Ad = torch.randn((n, m), dtype=torch.float64, device="cuda", generator=gen).t()
    Rd = torch.empty((n, m), dtype=torch.float64, device="cuda").t()
    with tqr.Plan(m, n, nb, ib) as plan:
        plan.load(Ad); plan.factor_tiles(); plan.store_r(Rd)
        E = torch.zeros((n, m), dtype=torch.float64, device="cuda").t()
        E[:n, :n] = torch.eye(n, dtype=torch.float64, device="cuda")
        plan.apply_qt(E, "N")
        I = torch.eye(n, dtype=torch.float64, device="cuda")
        orth = float((E.t() @ E - I).norm())
        res = float((Ad - E @ torch.triu(Rd[:n])).norm() / Ad.norm())
    Q2, R2 = torch.linalg.qr(Ad)
    orth2 = float((Q2.t() @ Q2 - I).norm())
    print(m, n, nb, ib, "tqr orth %.3e res %.3e | cusolver orth %.3e" % (orth, res, orth2), flush=True)
    del Ad, Rd, E, Q2, R2; torch.cuda.empty_cache()
