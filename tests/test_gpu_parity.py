"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the same seeded
inputs.  Tolerances are BASELINE.json's north-star bars:
    sign-normalised R, column-norm relative (reading Q16)   <= 1e-10
    ||A - QR||_F / ||A||_F                                  <= 1e-13
    ||Q^T Q - I||_F (thin Q, reading Q18)                   <= 1e-13 at these sizes
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

R_TOL = 1e-10
RES_TOL = 1e-13
ORTH_TOL = 1e-13


def dev_colmajor(A: np.ndarray) -> "torch.Tensor":
    """numpy (m, n) -> CUDA float64 tensor with column-major strides (1, m)."""
    return torch.from_numpy(np.ascontiguousarray(A.T)).cuda().t()


def to_np(t) -> np.ndarray:
    return t.cpu().numpy()


def gpu_qr(A, nb, ib, **kw):
    m, n = A.shape
    plan = tqr.Plan(m, n, nb, ib, **kw)
    Ad = dev_colmajor(A)
    plan.factor(Ad)
    return plan, to_np(Ad)


def thin_q_and_residual(plan, A, Rfull):
    m, n = A.shape
    E = np.zeros((m, n))
    E[:n, :n] = np.eye(n)
    Ed = dev_colmajor(E)
    plan.apply_qt(Ed, "N")
    Q = to_np(Ed)
    Rz = np.zeros((m, n))
    Rz[:n] = np.triu(Rfull[:n])
    Rd = dev_colmajor(Rz)
    plan.apply_qt(Rd, "N")
    QR = to_np(Rd)
    return Q, np.linalg.norm(A - QR) / np.linalg.norm(A)


GRIDS = [
    # (m, n, nb, ib)  -- tile grids p x q
    (64, 64, 64, 16),       # 1x1: GEQRT only
    (128, 64, 64, 16),      # 2x1: GEQRT + TSQRT
    (64 * 3, 64 * 3, 64, 16),   # 3x3: Fig. 2 walk-through
    (256, 256, 64, 16),     # C1 shape (4x4)
    (512, 128, 64, 16),     # tall 8x2
    (256, 256, 128, 32),
    (512, 512, 256, 32),    # 2x2 at C2's nb
    (1024, 512, 512, 32),   # 2x1 at C3-C5's nb
    (1024, 1024, 512, 32),  # 2x2 at nb=512
    (512, 512, 128, 16),
]


@pytest.mark.parametrize("m,n,nb,ib", GRIDS)
def test_factor_matches_oracle(m, n, nb, ib):
    A = synthetic.gaussian(m, n, 1000 + m + n + nb)
    plan, Rg = gpu_qr(A, nb, ib)
    ref = oracle.qr(A)
    err = colnorm_rel_err(np.triu(Rg[:n]), ref.R)
    assert err <= R_TOL, err
    # strictly lower part of A is zeroed (tqr.h contract)
    assert np.all(np.tril(Rg, -1) == 0.0)
    Q, res = thin_q_and_residual(plan, A, Rg)
    assert res <= RES_TOL, res
    orth = np.linalg.norm(Q.T @ Q - np.eye(n))
    assert orth <= ORTH_TOL * max(1.0, np.sqrt(n / 256.0)), orth
    plan.close()


def test_c1_config_full_parity():
    c = synthetic.CONFIGS["C1"]
    A = synthetic.gaussian(c["m"], c["n"], c["seed"])
    plan, Rg = gpu_qr(A, c["nb"], c["ib"])
    ref = oracle.qr(A)
    assert colnorm_rel_err(np.triu(Rg), ref.R) <= R_TOL
    Q, res = thin_q_and_residual(plan, A, Rg)
    assert res <= RES_TOL
    assert np.linalg.norm(Q.T @ Q - np.eye(c["n"])) <= ORTH_TOL
    # thin Q is unique up to column signs: compare with the oracle's
    Qo = ref.thin_q()
    d = np.sign(np.diag(Rg)) * np.sign(np.diag(ref.R))
    np.testing.assert_allclose(Q * d[None, :], Qo, atol=1e-12)


def test_apply_qt_top_rows_equal_R_and_roundtrip():
    m, n, nb, ib = 512, 256, 64, 16
    A = synthetic.gaussian(m, n, 77)
    plan, Rg = gpu_qr(A, nb, ib)
    Ad = dev_colmajor(A)
    plan.apply_qt(Ad, "T")
    QtA = to_np(Ad)
    np.testing.assert_allclose(np.triu(QtA[:n]), np.triu(Rg[:n]), atol=1e-12 * np.abs(Rg).max())
    assert np.linalg.norm(np.tril(QtA, -1)) <= 1e-12 * np.linalg.norm(A)
    B = synthetic.gaussian(m, 5, 78)
    Bd = dev_colmajor(B)
    plan.apply_qt(Bd, "T")
    plan.apply_qt(Bd, "N")
    np.testing.assert_allclose(to_np(Bd), B, atol=1e-12)


def test_solve_ls_matches_oracle():
    m, n, nb, ib = 512, 256, 64, 16
    A = synthetic.gaussian(m, n, 79)
    B = synthetic.gaussian(m, 3, 80)
    plan, _ = gpu_qr(A, nb, ib)
    Bd = dev_colmajor(B)
    plan.solve_ls(Bd)
    X = to_np(Bd)[:n]
    Xo = oracle.solve_ls(A, B)
    np.testing.assert_allclose(X, Xo, rtol=1e-9, atol=1e-11)


def test_host_pointer_and_pinned_paths_match_device():
    m, n, nb, ib = 384, 256, 64, 16
    A = synthetic.gaussian(m, n, 81)
    _, Rd = gpu_qr(A, nb, ib)
    plan = tqr.Plan(m, n, nb, ib)
    Ah = np.asfortranarray(A.copy())
    plan.factor(Ah)                     # pageable host
    assert np.array_equal(np.triu(Ah[:n]), np.triu(Rd[:n]))
    Ap = torch.from_numpy(np.ascontiguousarray(A.T)).pin_memory().t()
    plan.factor(Ap)                     # pinned host
    assert np.array_equal(np.triu(Ap.numpy()[:n]), np.triu(Rd[:n]))


@pytest.mark.parametrize("ndev,guide", [(2, None), (2, [1, 0]), (3, [1, 0, 1, 0, 1, 2]), (4, [0, 0, 1, 3, 2])])
def test_logical_devices_partition_bitwise(ndev, guide):
    """Guide-array partitions (Eq. 12) on logical devices: identical R to the 1-owner run."""
    m, n, nb, ib = 512, 512, 64, 16
    A = synthetic.gaussian(m, n, 82)
    _, R1 = gpu_qr(A, nb, ib)
    plan, Rp = gpu_qr(A, nb, ib, ndev=ndev, guide=guide, logical_devices=True)
    assert np.array_equal(np.triu(Rp[:n]), np.triu(R1[:n]))
    g = guide if guide is not None else list(range(ndev))
    assert [plan.owner(j) for j in range(n // nb)] == [g[j % len(g)] for j in range(n // nb)]


def test_lookahead_off_bitwise_identical():
    m, n, nb, ib = 512, 512, 128, 32
    A = synthetic.gaussian(m, n, 83)
    _, R1 = gpu_qr(A, nb, ib)
    _, R2 = gpu_qr(A, nb, ib, lookahead=False)
    assert np.array_equal(R1, R2)


def test_repeat_factor_deterministic():
    m, n, nb, ib = 512, 512, 128, 32
    A = synthetic.gaussian(m, n, 84)
    plan = tqr.Plan(m, n, nb, ib)
    outs = []
    for _ in range(3):
        Ad = dev_colmajor(A)
        plan.factor(Ad)
        outs.append(to_np(Ad))
    assert np.array_equal(outs[0], outs[1]) and np.array_equal(outs[1], outs[2])


def test_zero_and_degenerate_columns():
    """Zero column (tau = 0, reading Q3), a column already zero below row 70, and a repeated
    column.  Where R_ii = 0 the rows i.. of R are not unique (q_i is any unit vector orthogonal
    to q_0..q_{i-1}), so those rows are checked through R^T R = A^T A only."""
    m, n, nb, ib = 256, 128, 64, 16
    base = synthetic.gaussian(m, n, 85)
    # (a) zero column 5: R(:, 5) = 0; rows 0..4 unique
    A = base.copy()
    A[:, 5] = 0.0
    plan, Rg = gpu_qr(A, nb, ib)
    R = np.triu(Rg[:n])
    assert np.all(np.isfinite(R)) and np.all(R[:, 5] == 0.0)
    assert np.linalg.norm(R.T @ R - A.T @ A) <= 1e-12 * np.linalg.norm(A) ** 2
    assert colnorm_rel_err(R[:5], oracle.qr(A).R[:5]) <= R_TOL
    # (b) column 70 zero below row 70 before any reflection: full-rank, unique
    A = base.copy()
    A[70:, 70] = 0.0
    _, Rg = gpu_qr(A, nb, ib)
    assert colnorm_rel_err(np.triu(Rg[:n]), oracle.qr(A).R) <= R_TOL
    # (c) column 100 repeats column 3: rows < 100 unique, R_100,100 ~ 0
    A = base.copy()
    A[:, 100] = A[:, 3]
    _, Rg = gpu_qr(A, nb, ib)
    R = np.triu(Rg[:n])
    assert np.linalg.norm(R.T @ R - A.T @ A) <= 1e-12 * np.linalg.norm(A) ** 2
    assert colnorm_rel_err(R[:100], oracle.qr(A).R[:100]) <= R_TOL
    assert abs(R[100, 100]) <= 1e-12 * np.linalg.norm(A[:, 3])


def test_integer_and_ill_conditioned_inputs():
    m, n, nb, ib = 256, 256, 64, 16
    A = synthetic.integer_matrix(m, n, 86)
    _, Rg = gpu_qr(A, nb, ib)
    assert colnorm_rel_err(np.triu(Rg), oracle.qr(A).R) <= R_TOL
    A = synthetic.ill_conditioned(m, n, 87, cond=1e10)
    plan, Rg = gpu_qr(A, nb, ib)
    _, res = thin_q_and_residual(plan, A, Rg)
    assert res <= RES_TOL


def test_errors_and_states():
    with pytest.raises(tqr.TqrError) as e:
        tqr.Plan(100, 64, 64, 16)           # m not a multiple of nb
    assert e.value.status == 7
    with pytest.raises(tqr.TqrError) as e:
        tqr.Plan(64, 128, 64, 16)           # m < n
    assert e.value.status == 1
    with pytest.raises(tqr.TqrError) as e:
        tqr.Plan(128, 128, 64, 16, ndev=2, guide=[0, 2])
    assert e.value.status == 1
    plan = tqr.Plan(128, 128, 64, 16)
    B = dev_colmajor(np.ones((128, 2)))
    with pytest.raises(tqr.TqrError) as e:
        plan.apply_qt(B)
    assert e.value.status == 5
    A = np.zeros((128, 128), order="F")
    A[:, :] = np.eye(128)
    A[5, 5] = 0.0
    plan.factor(dev_colmajor(A))
    with pytest.raises(tqr.TqrError) as e:
        plan.solve_ls(dev_colmajor(np.ones((128, 1))))
    assert e.value.status == 6


def test_full_size_c2_sampled_parity():
    """C2 (4096^2, nb=256, ib=32) in the bench launch configuration: R checked against the
    oracle in full (the oracle finishes C2 in tens of seconds on the host) and the residual /
    orthogonality properties that hold at any size."""
    c = synthetic.CONFIGS["C2"]
    m, n = c["m"], c["n"]
    A = synthetic.gaussian(m, n, c["seed"])
    plan, Rg = gpu_qr(A, c["nb"], c["ib"])
    ref = oracle.qr(A, nthreads=0)
    assert colnorm_rel_err(np.triu(Rg), ref.R) <= R_TOL
    # random-probe residual ||A x - Q (R x)|| for a few x
    X = synthetic.gaussian(n, 4, 88)
    RX = np.zeros((m, 4))
    RX[:n] = np.triu(Rg) @ X
    RXd = dev_colmajor(RX)
    plan.apply_qt(RXd, "N")
    res = np.linalg.norm(A @ X - to_np(RXd)) / (np.linalg.norm(A) * np.linalg.norm(X))
    assert res <= RES_TOL
