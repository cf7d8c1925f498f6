import sys, os
sys.path.insert(0, os.getcwd())
import torch
import paper_conf_icpp_kimp13_b200 as tqr
for n in [2048, 4096, 8192, 16384, 32768]:
    m, nb, ib = n, 512, 32
    gen = torch.Generator(device="cuda").manual_seed(1)
    Ad = torch.randn((n, m), dtype=torch.float64, device="cuda", generator=gen).t()
    Rd = torch.empty((n, m), dtype=torch.float64, device="cuda").t()
    with tqr.Plan(m, n, nb, ib) as plan:
        plan.load(Ad); plan.factor_tiles(); plan.store_r(Rd)
        for nr in [3, 40]:
            X = torch.randn((n, nr), dtype=torch.float64, device="cuda", generator=gen)
            RX = torch.zeros((nr, m), dtype=torch.float64, device="cuda").t()
            RX[:n] = torch.triu(Rd[:n]) @ X
            plan.apply_qt(RX, "N")
            res = float((Ad @ X - RX).norm() / (Ad.norm() * X.norm()))
            B = Ad @ X
            B2 = B.t().contiguous().t()
            plan.apply_qt(B2, "T")
            resT = float((B2[:n] - torch.triu(Rd[:n]) @ X).norm() / (Ad.norm() * X.norm()))
            print(n, nr, "resN %.3e resT %.3e" % (res, resT), flush=True)
    del Ad, Rd; torch.cuda.empty_cache()
