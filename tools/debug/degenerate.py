import sys, os
sys.path.insert(0, os.getcwd()); sys.path.insert(0, os.path.join(os.getcwd(), "tests"))
import numpy as np, torch
import oracle, synthetic
import paper_conf_icpp_kimp13_b200 as tqr
from conftest import sign_normalise_R
def run(A, nb=64, ib=16):
    m, n = A.shape
    p = tqr.Plan(m, n, nb, ib)
    Ad = torch.from_numpy(np.ascontiguousarray(A.T)).cuda().t()
    p.factor(Ad)
    Rg = np.triu(Ad.cpu().numpy()[:n]); Ro = oracle.qr(A).R
    a, b = sign_normalise_R(Rg), sign_normalise_R(Ro)
    cn = np.linalg.norm(b, axis=0); cn[cn == 0] = 1
    e = np.abs(a - b) / cn
    bad = np.argwhere(e > 1e-10)
    return e.max(), bad[:5].tolist()
base = synthetic.gaussian(256, 128, 85)
for name in ["zero5", "col70", "dup100", "all"]:
    A = base.copy()
    if name in ("zero5", "all"): A[:, 5] = 0
    if name in ("col70", "all"): A[70:, 70] = 0
    if name in ("dup100", "all"): A[:, 100] = A[:, 3]
    print(name, run(A))
A = base.copy(); A[:, 5] = 0
print("zero5 nb128", run(A, 128, 32))
print("diag R", np.diag(oracle.qr(A).R)[:8])
