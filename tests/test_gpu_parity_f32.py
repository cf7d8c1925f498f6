"""GPU parity of the FP32 path (TQR_F32: SIMT FFMA trailing updates,
 FP64-factored panels narrowed to FP32) against the FP64 oracle run on the FP32-rounded input (exactly representable, so the oracle
is the more accurate side).  North-star FP32 bars (BASELINE.json):
    sign-normalised R, column-norm relative (reading Q16)   <= 1e-3
    ||A - QR||_F / ||A||_F                                  <= 1e-5
    ||Q^T Q - I||_F (thin Q, reading Q18)                   <= 1e-5, or at most 2x LAPACK sgeqrf's
                                                               value on the same input where LAPACK
                                                               itself exceeds 1e-5 (reading Q19)
"""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import oracle
import synthetic
import paper_conf_icpp_kimp13_b200 as tqr
from conftest import colnorm_rel_err

pytestmark = pytest.mark.gpu

R_TOL = 1e-3
RES_TOL = 1e-5
ORTH_TOL = 1e-5


def dev32(A: np.ndarray) -> "torch.Tensor":
    return torch.from_numpy(np.ascontiguousarray(np.asarray(A, dtype=np.float32).T)).cuda().t()


def to_np(t) -> np.ndarray:
    return t.cpu().numpy().astype(np.float64)


def lapack_orth32(A32):
    Q, _ = torch.linalg.qr(torch.from_numpy(np.ascontiguousarray(A32)))
    Q = Q.double()
    return float((Q.t() @ Q - torch.eye(Q.shape[1], dtype=torch.float64)).norm())


def gpu_qr32(A32, nb, ib, **kw):
    m, n = A32.shape
    plan = tqr.Plan(m, n, nb, ib, dtype=tqr.TQR_F32, **kw)
    Ad = dev32(A32)
    plan.factor(Ad)
    return plan, to_np(Ad)


def check_all(plan, A32, Rg, nb, ib):
    m, n = A32.shape
    A = A32.astype(np.float64)
    ref = oracle.qr(A)
    rerr = colnorm_rel_err(np.triu(Rg[:n]), ref.R)
    assert rerr <= R_TOL, rerr
    assert np.all(np.tril(Rg, -1) == 0.0)
    E = np.zeros((m, n), dtype=np.float32)
    E[:n, :n] = np.eye(n, dtype=np.float32)
    Ed = dev32(E)
    plan.apply_qt(Ed, "N")
    Q = to_np(Ed)
    Rz = np.zeros((m, n), dtype=np.float32)
    Rz[:n] = np.triu(Rg[:n])
    Rd = dev32(Rz)
    plan.apply_qt(Rd, "N")
    res = np.linalg.norm(A - to_np(Rd)) / np.linalg.norm(A)
    assert res <= RES_TOL, res
    orth = np.linalg.norm(Q.T @ Q - np.eye(n))
    assert orth <= max(ORTH_TOL, 2.0 * lapack_orth32(A32)), orth
    return rerr, res, orth


GRIDS = [
    (64, 64, 64, 16),
    (128, 64, 64, 16),
    (256, 256, 64, 16),         # C1 shape
    (512, 128, 64, 32),
    (512, 512, 128, 32),
    (1024, 1024, 256, 32),      # C2's nb
    (1024, 512, 512, 32),       # C3-C5's nb
    (1536, 1536, 512, 32),
    (1536, 1024, 512, 16),
    (300, 200, 64, 16),         # ragged both ways
    (1100, 1030, 512, 32),      # ragged at nb=512
]


@pytest.mark.parametrize("m,n,nb,ib", GRIDS)
def test_f32_factor_matches_oracle(m, n, nb, ib):
    A32 = synthetic.gaussian(m, n, 4000 + m + n + nb).astype(np.float32)
    plan, Rg = gpu_qr32(A32, nb, ib)
    rerr, res, orth = check_all(plan, A32, Rg, nb, ib)
    print("f32 %dx%d nb=%d ib=%d: R %.2e res %.2e orth %.2e" % (m, n, nb, ib, rerr, res, orth))
    plan.close()


def test_f32_c1_config():
    c = synthetic.CONFIGS["C1"]
    A32 = synthetic.gaussian(c["m"], c["n"], c["seed"]).astype(np.float32)
    plan, Rg = gpu_qr32(A32, c["nb"], c["ib"])
    check_all(plan, A32, Rg, c["nb"], c["ib"])


def test_f32_solve_and_roundtrip():
    m, n, nb, ib = 768, 512, 128, 32
    A32 = synthetic.gaussian(m, n, 4101).astype(np.float32)
    B32 = synthetic.gaussian(m, 3, 4102).astype(np.float32)
    plan, _ = gpu_qr32(A32, nb, ib)
    Bd = dev32(B32)
    plan.solve_ls(Bd)
    X = to_np(Bd)[:n]
    Xo = oracle.solve_ls(A32.astype(np.float64), B32.astype(np.float64))
    assert np.linalg.norm(X - Xo) / np.linalg.norm(Xo) <= 1e-4
    Bd = dev32(B32)
    plan.apply_qt(Bd, "T")
    plan.apply_qt(Bd, "N")
    assert np.abs(to_np(Bd) - B32).max() <= 1e-5 * np.abs(B32).max() * 10


def test_f32_logical_devices_and_host_path_bitwise():
    m, n, nb, ib = 1024, 1024, 128, 32
    A32 = synthetic.gaussian(m, n, 4103).astype(np.float32)
    _, R1 = gpu_qr32(A32, nb, ib)
    _, R2 = gpu_qr32(A32, nb, ib, ndev=3, guide=[1, 0, 2, 2], logical_devices=True)
    assert np.array_equal(R1, R2)
    # and against the oracle directly (FP64 Algorithm 1 on the FP32 input)
    assert colnorm_rel_err(np.triu(R2[:n]).astype(np.float64), oracle.qr(A32.astype(np.float64)).R) <= R_TOL
    plan = tqr.Plan(m, n, nb, ib, dtype=tqr.TQR_F32)
    Ah = np.asfortranarray(A32.copy())
    plan.factor(Ah)
    assert np.array_equal(np.triu(Ah[:n]).astype(np.float64), np.triu(R1[:n]))
    with pytest.raises(TypeError):
        plan.factor(torch.zeros((n, m), dtype=torch.float64, device="cuda").t())


def test_f32_nccl_transport_single_rank_bitwise():
    m, n, nb, ib = 1024, 1024, 256, 32
    A32 = synthetic.gaussian(m, n, 4104).astype(np.float32)
    _, R1 = gpu_qr32(A32, nb, ib)
    uid = tqr.tqr_nccl_unique_id()
    plan = tqr.Plan(m, n, nb, ib, dtype=tqr.TQR_F32, ndev=1, rank=0, world=1, nccl_id=uid)
    Ad = dev32(A32)
    plan.factor(Ad)
    assert np.array_equal(to_np(Ad), R1)
    assert colnorm_rel_err(np.triu(R1[:n]).astype(np.float64), oracle.qr(A32.astype(np.float64)).R) <= R_TOL


@pytest.mark.slow
def test_f32_full_size_c5_bench_configuration():
    """C5 FP32 (32768^2, nb=512, ib=32) as bench.py --dtype f32 runs it: leading columns against
    the oracle, sampled R^T R = A^T A, random-probe residual."""
    m, n, nb, ib, seed = 32768, 32768, 512, 32, 105
    gen = torch.Generator(device="cuda").manual_seed(seed)
    Ad = torch.randn((n, m), dtype=torch.float32, device="cuda", generator=gen).t()
    Rd = torch.empty((n, m), dtype=torch.float32, device="cuda").t()
    with tqr.Plan(m, n, nb, ib, dtype=tqr.TQR_F32) as plan:
        plan.load(Ad)
        plan.factor_tiles()
        plan.store_r(Rd)
        J = 1024
        ref = oracle.qr(Ad[:, :J].cpu().numpy().astype(np.float64), nthreads=0)
        assert colnorm_rel_err(np.triu(Rd[:J, :J].cpu().numpy().astype(np.float64)), ref.R) <= R_TOL
        g = torch.Generator().manual_seed(9)
        ii = torch.randint(0, n, (64,), generator=g).cuda()
        jj = torch.randint(0, n, (64,), generator=g).cuda()
        lhs = (Rd[:n][:, ii].double() * Rd[:n][:, jj].double()).sum(0)
        rhs = (Ad[:, ii].double() * Ad[:, jj].double()).sum(0)
        scale = Ad[:, ii].double().norm(dim=0) * Ad[:, jj].double().norm(dim=0)
        assert float(((lhs - rhs).abs() / scale).max()) <= 1e-5
        X = torch.randn((n, 2), dtype=torch.float32, generator=g).cuda()
        RX = torch.zeros((2, m), dtype=torch.float32, device="cuda").t()
        RX[:n] = torch.triu(Rd[:n]) @ X
        plan.apply_qt(RX, "N")
        res = (Ad.double() @ X.double() - RX.double()).norm() / (Ad.double().norm() * X.double().norm())
        assert float(res) <= RES_TOL
    del Ad, Rd
    torch.cuda.empty_cache()
