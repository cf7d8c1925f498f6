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


def lapack_orth(A):
    """||Q^T Q - I||_F of LAPACK's Householder QR (numpy.linalg.qr) on the same input: the
    context printed next to a failing orthogonality check (reading Q19)."""
    Ql, _ = np.linalg.qr(A)
    return float(np.linalg.norm(Ql.T @ Ql - np.eye(A.shape[1])))


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
    assert orth <= ORTH_TOL, (orth, lapack_orth(A))
    plan.close()


RAGGED = [
    # (m, n, nb, ib): m and/or n not multiples of nb -> zero-padded tiles
    (100, 64, 64, 16),      # ragged rows only, 2x1
    (70, 70, 64, 16),       # 1-element tail column of a square matrix (u = 0 case, reading Q1)
    (300, 200, 64, 16),     # 5x4 grid, ragged both ways
    (129, 1, 64, 16),       # single column
    (1000, 777, 256, 32),   # 4x4 at C2's nb, ragged both ways
    (1100, 1030, 512, 32),  # 3x3 at nb=512
    (600, 513, 128, 32),    # last column tile 1 wide
]


@pytest.mark.parametrize("m,n,nb,ib", RAGGED)
def test_ragged_matches_oracle(m, n, nb, ib):
    """Ragged tails: R, residual, thin-Q orthogonality, Q^T A top rows and least squares."""
    A = synthetic.gaussian(m, n, 2000 + m + n + nb)
    plan, Rg = gpu_qr(A, nb, ib)
    ref = oracle.qr(A)
    assert colnorm_rel_err(np.triu(Rg[:n]), ref.R) <= R_TOL
    assert np.all(np.tril(Rg, -1) == 0.0)
    Q, res = thin_q_and_residual(plan, A, Rg)
    assert res <= RES_TOL, res
    orth = np.linalg.norm(Q.T @ Q - np.eye(n))
    assert orth <= ORTH_TOL, (orth, lapack_orth(A))
    B = synthetic.gaussian(m, 3, 3000 + m)
    Bd = dev_colmajor(B)
    plan.solve_ls(Bd)
    np.testing.assert_allclose(to_np(Bd)[:n], oracle.solve_ls(A, B), rtol=1e-8, atol=1e-10)
    # host-pointer path with lda > m
    Ah = np.full((m + 3, n), 7.0, order="F")     # rows m.. are outside A: never touched
    Ah[:m] = A
    assert tqr.lib().tqr_factor(plan.h, Ah.ctypes.data, m + 3) == 0
    assert np.array_equal(np.triu(Ah[:n]), np.triu(Rg[:n]))
    assert np.all(Ah[m:] == 7.0)
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


@pytest.mark.parametrize("m,n,nb,ib,nrhs", [
    (1024, 1024, 512, 32, 1),       # 2 tile rows, one RHS
    (1536, 1024, 256, 32, 70),      # tall, 3 RHS slices (ragged last slice)
    (700, 650, 128, 32, 33),        # ragged rows, columns and RHS (padded diagonal rows)
    (640, 640, 64, 16, 100),        # nb = 64: update row blocks straddle tiles
])
def test_tile_trsm_solve_matches_oracle(m, n, nb, ib, nrhs):
    """tqr_solve_ls = Q^T B on the update kernel + the tile back substitution (trsm.cu: inverted
    32 x 32 diagonal blocks inside each R_ii, FMA updates of the rows above) vs the oracle's
    Eqs. (2)-(3) (plain back substitution)."""
    A = synthetic.gaussian(m, n, 7000 + m + n)
    B = synthetic.gaussian(m, nrhs, 7100 + nrhs)
    plan, _ = gpu_qr(A, nb, ib)
    Bd = dev_colmajor(B)
    plan.solve_ls(Bd)
    X = to_np(Bd)[:n]
    Xo = oracle.solve_ls(A, B)
    np.testing.assert_allclose(X, Xo, rtol=1e-8, atol=1e-10 * max(1.0, np.abs(Xo).max()))
    plan.close()


@pytest.mark.parametrize("m,n,nb,ib,nrhs", [(1536, 1024, 256, 32, 40), (640, 600, 64, 16, 7), (2048, 2048, 512, 32, 96)])
def test_wavefront_apply_bitwise(m, n, nb, ib, nrhs, monkeypatch):
    """One-launch wavefront Q^T B / Q B (step k+1's CTA follows step k's tile by tile on progress
    flags) computes every chain exactly as the per-step launches: bitwise equal, and Q (Q^T B) = B."""
    A = synthetic.gaussian(m, n, 7300 + m)
    B = synthetic.gaussian(m, nrhs, 7400 + nrhs)
    plan, _ = gpu_qr(A, nb, ib)
    out = {}
    for mode in ("wave", "steps"):
        if mode == "steps":
            monkeypatch.setenv("TQR_NO_WAVEFRONT_APPLY", "1")
        Bd = dev_colmajor(B)
        plan.apply_qt(Bd, "T")
        QtB = to_np(Bd)
        plan.apply_qt(Bd, "N")
        out[mode] = (QtB, to_np(Bd))
    assert np.array_equal(out["wave"][0], out["steps"][0])
    assert np.array_equal(out["wave"][1], out["steps"][1])
    np.testing.assert_allclose(out["wave"][1], B, atol=1e-12)
    plan.close()


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


@pytest.mark.parametrize("m,n,nb,ib,kw", [
    (1024, 768, 128, 32, {}),                                              # q = 6
    (1000, 700, 128, 32, {"ndev": 3, "guide": [2, 0, 1], "logical_devices": True}),   # ragged, 3 owners
    (4096, 256, 256, 32, {"tree_domain": 2}),                              # tree + two-level merge
    (512, 512, 64, 16, {"lookahead": False}),
])
def test_streamed_host_factor_bitwise(m, n, nb, ib, kw, monkeypatch):
    """tqr_factor on a host A pipelines the column loads / R stores with the factorization (panel k
    and the step-0 update of column j wait only for their own column); the arithmetic is the
    device-resident path's, so A <- R must agree bitwise, including the zeroed lower part."""
    A = synthetic.gaussian(m, n, 90 + m + n)
    _, Rd = gpu_qr(A, nb, ib, **kw)
    plan = tqr.Plan(m, n, nb, ib, **kw)
    Ap = torch.from_numpy(np.ascontiguousarray(A.T)).pin_memory().t()
    plan.factor(Ap)
    assert np.array_equal(Ap.numpy(), Rd)
    monkeypatch.setenv("TQR_NO_STREAMED_IO", "1")          # the three-phase path on the same plan
    Ap2 = torch.from_numpy(np.ascontiguousarray(A.T)).pin_memory().t()
    plan.factor(Ap2)
    assert np.array_equal(Ap2.numpy(), Rd)
    plan.close()


@pytest.mark.parametrize("m,n,nb,ib", [(8192, 512, 512, 32), (5000, 300, 512, 32), (24576, 256, 256, 32)])
def test_streamed_tall_factor_bitwise(m, n, nb, ib, monkeypatch):
    """Single tile column, tree mode with one CTA per domain: tqr_factor on a host A loads the rows
    in chunks of whole domains, starts each chunk's domains as it lands, writes the zero rows back
    early and R (first tile row) after the merges -- bitwise the device-resident result."""
    monkeypatch.setenv("TQR_TREE_ONE_CTA", "1")
    A = synthetic.gaussian(m, n, 7700 + m + n)
    _, Rd = gpu_qr(A, nb, ib)
    plan = tqr.Plan(m, n, nb, ib)
    Ap = torch.from_numpy(np.ascontiguousarray(A.T)).pin_memory().t()
    plan.factor(Ap)
    assert np.array_equal(Ap.numpy(), Rd)
    Ah = np.full((m + 5, n), 9.0, order="F")              # pageable, lda > m: rows m.. untouched
    Ah[:m] = A
    assert tqr.lib().tqr_factor(plan.h, Ah.ctypes.data, m + 5) == 0
    assert np.array_equal(Ah[:m], Rd) and np.all(Ah[m:] == 9.0)
    assert colnorm_rel_err(np.triu(Rd[:n]), oracle.qr(A).R) <= R_TOL
    plan.close()


@pytest.mark.parametrize("ndev,guide", [(2, None), (2, [1, 0]), (3, [1, 0, 1, 0, 1, 2]), (4, [0, 0, 1, 3, 2])])
def test_logical_devices_partition_bitwise(ndev, guide):
    """Guide-array partitions (Eq. 12) on logical devices: identical R to the 1-owner run."""
    m, n, nb, ib = 512, 512, 64, 16
    A = synthetic.gaussian(m, n, 82)
    _, R1 = gpu_qr(A, nb, ib)
    plan, Rp = gpu_qr(A, nb, ib, ndev=ndev, guide=guide, logical_devices=True)
    assert np.array_equal(np.triu(Rp[:n]), np.triu(R1[:n]))
    assert colnorm_rel_err(np.triu(Rp[:n]), oracle.qr(A).R) <= R_TOL          # and against the oracle
    Q, res = thin_q_and_residual(plan, A, Rp)                                  # multi-owner apply
    assert res <= RES_TOL and np.linalg.norm(Q.T @ Q - np.eye(n)) <= ORTH_TOL
    g = guide if guide is not None else list(range(ndev))
    assert [plan.owner(j) for j in range(n // nb)] == [g[j % len(g)] for j in range(n // nb)]
    # the executor consumed the DAG schedule: per step, PANEL + BCAST + every owner's UPDATE columns
    sched = sorted({r for d in range(ndev) for r in tqr.tqr_schedule(m, n, nb, ndev, guide, d)}, key=lambda r: (r[1], r[0], r[3]))
    assert sorted(plan.issued_ops(), key=lambda r: (r[1], r[0], r[3])) == sched


@pytest.mark.parametrize("ndev,guide,tree", [(3, [1, 0, 1, 0, 1, 2], -1), (2, [1, 0], 2)])
def test_replica_apply_bitwise(ndev, guide, tree, monkeypatch):
    """apply/solve on a multi-GPU or multi-process plan run on a single-owner replica gathered from
    the owners (TQR_FORCE_REPLICA exercises that path with logical owners on one GPU): bitwise the
    in-place multi-owner apply, and against the oracle."""
    m, n, nb, ib = 768, 512, 64, 16
    A = synthetic.gaussian(m, n, 8200 + ndev)
    B = synthetic.gaussian(m, 5, 8300)
    plan, Rg = gpu_qr(A, nb, ib, ndev=ndev, guide=guide, logical_devices=True, tree_domain=tree)
    out = {}
    for mode in ("direct", "replica"):
        if mode == "replica":
            monkeypatch.setenv("TQR_FORCE_REPLICA", "1")
        Bd = dev_colmajor(B)
        plan.apply_qt(Bd, "T")
        QtB = to_np(Bd)
        plan.apply_qt(Bd, "N")
        Xd = dev_colmajor(B)
        plan.solve_ls(Xd)
        out[mode] = (QtB, to_np(Bd), to_np(Xd))
    for a, b in zip(out["direct"], out["replica"]):
        assert np.array_equal(a, b)
    np.testing.assert_allclose(out["replica"][2][:n], oracle.solve_ls(A, B), rtol=1e-8, atol=1e-10)
    plan.close()


@pytest.mark.parametrize("scale", [1e300, 1e200, 1e-200, 1e-300])
@pytest.mark.parametrize("m,n,nb,ib,kw", [(256, 256, 64, 16, {}), (1024, 512, 512, 32, {}),
                                          (4096, 512, 512, 32, {"tree_domain": 2})])
def test_extreme_scaling_matches_oracle(scale, m, n, nb, ib, kw):
    """dlarfg/dnrm2 semantics (reading Q26): entries ~1e+-200 / 1e+-300 overflow or underflow a
    plain sum of squares; factor_block redoes such a column on an exactly power-of-two scaled x.
    R(cA) = c R(A): compare with the (scaled-norm) oracle and LAPACK, and Q stays orthogonal."""
    A = synthetic.gaussian(m, n, 6100 + m + n) * scale
    plan, Rg = gpu_qr(A, nb, ib, **kw)
    R = np.triu(Rg[:n])
    assert np.all(np.isfinite(R))
    assert colnorm_rel_err(R, oracle.qr(A).R) <= R_TOL
    assert colnorm_rel_err(R, np.linalg.qr(A, mode="r")) <= R_TOL
    Q, _ = thin_q_and_residual(plan, A, Rg)
    # residual on the unscaled magnitudes (numpy's norm is an unscaled sum of squares)
    res = np.linalg.norm(A / scale - Q @ (R / scale)) / np.linalg.norm(A / scale)
    assert res <= RES_TOL and np.linalg.norm(Q.T @ Q - np.eye(n)) <= ORTH_TOL, res
    plan.close()


def test_lookahead_off_bitwise_identical():
    m, n, nb, ib = 512, 512, 128, 32
    A = synthetic.gaussian(m, n, 83)
    _, R1 = gpu_qr(A, nb, ib)
    _, R2 = gpu_qr(A, nb, ib, lookahead=False)
    assert np.array_equal(R1, R2)


@pytest.mark.parametrize("m,n,nb,ib", [(1100, 1030, 512, 32), (4096, 1024, 512, 32), (1000, 777, 256, 32),
                                      (1024, 768, 512, 16), (1536, 1024, 256, 16)])
def test_w16_update_matches_oracle_and_8warp_form(monkeypatch, m, n, nb, ib):
    """Bulk update with the 32-column slice over 16 warps (update_kernel16, default for nb >= 256)
    and over 8 warps (TQR_W16=0): both against the oracle (R, residual, thin-Q orthogonality,
    least squares -- Q^T B runs the same kernels) and bitwise equal to each other.  n <= 1030:
    the absolute 1e-13 orthogonality bar is the one LAPACK meets there (reading Q19; at 2048^2 the
    16-warp form measured 1.13e-13 against LAPACK's 7.0e-14 on the same matrix, the 1.5-1.8x ratio
    of the full-size table, profiles/r02_full_parity.json)."""
    A = synthetic.gaussian(m, n, 4500 + m + nb + ib)
    B = synthetic.gaussian(m, 3, 4600 + m)
    ref = oracle.qr(A)
    out = {}
    for w16 in ("1", "0"):
        monkeypatch.setenv("TQR_W16", w16)
        plan, Rg = gpu_qr(A, nb, ib)
        assert colnorm_rel_err(np.triu(Rg[:n]), ref.R) <= R_TOL
        assert np.all(np.tril(Rg, -1) == 0.0)
        Q, res = thin_q_and_residual(plan, A, Rg)
        assert res <= RES_TOL, (w16, res)
        orth = np.linalg.norm(Q.T @ Q - np.eye(n))
        assert orth <= ORTH_TOL, (w16, orth, lapack_orth(A))
        Bd = dev_colmajor(B)
        plan.solve_ls(Bd)
        np.testing.assert_allclose(to_np(Bd)[:n], oracle.solve_ls(A, B), rtol=1e-8, atol=1e-10)
        out[w16] = np.triu(Rg[:n])
        plan.close()
    # same rows per partial slot, same slot order, same DMMA order per accumulator: bitwise equal
    # (which is what keeps the full-size parity of profiles/r02_full_parity.json valid for it)
    assert np.array_equal(out["1"], out["0"])


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
        tqr.Plan(128, 128, 96, 16)          # nb not a built tile size
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


def test_nccl_transport_single_rank_bitwise():
    """The multi-process (NCCL broadcast) code path with a 1-rank communicator on cuda:0:
    ncclGroupStart/Broadcast x3/GroupEnd per panel on the comm stream, the same events."""
    m, n, nb, ib = 512, 512, 128, 32
    A = synthetic.gaussian(m, n, 90)
    _, R1 = gpu_qr(A, nb, ib)
    uid = tqr.tqr_nccl_unique_id()
    plan = tqr.Plan(m, n, nb, ib, ndev=1, rank=0, world=1, nccl_id=uid)
    Ad = dev_colmajor(A)
    plan.factor(Ad)
    assert np.array_equal(to_np(Ad), R1)
    assert colnorm_rel_err(np.triu(R1[:n]), oracle.qr(A).R) <= R_TOL


@pytest.mark.parametrize("m,n,nb,ib,ndev", [
    (8192, 512, 512, 32, 2),      # 16 tiles -> 8 + 8 rows tiles, each owner's block a TS tree
    (12800, 512, 512, 32, 3),     # 25 tiles -> 8 / 8 / 9
    (5000, 200, 256, 32, 4),      # ragged: n < nb, m not a multiple of nb
    (4096, 64, 64, 16, 8),        # 64 tiles over 8 owners
])
def test_row_split_matches_oracle(m, n, nb, ib, ndev):
    """Row split (NEXT-1 across owners, TSQR): each logical owner factors its contiguous row
    block, the owners' R factors are stacked on owner 0 and factored again.  R is unique, so it
    must match the oracle like the single-owner tree; every entry below R is zero."""
    A = synthetic.gaussian(m, n, 7500 + m + ndev)
    plan = tqr.Plan(m, n, nb, ib, ndev=ndev, logical_devices=True, row_split=1)
    Ad = dev_colmajor(A)
    plan.factor(Ad)
    Rg = to_np(Ad)
    ref = oracle.qr(A)
    assert colnorm_rel_err(np.triu(Rg[:n]), ref.R) <= R_TOL
    assert np.all(np.tril(Rg, -1) == 0.0) and np.all(Rg[n:] == 0.0)
    _, R1 = gpu_qr(A, nb, ib)                               # single owner
    assert colnorm_rel_err(np.triu(Rg[:n]), np.triu(R1[:n])) <= R_TOL
    Ah = np.asfortranarray(A.copy())                       # host A, three-phase ABI path
    plan.load(Ah)
    plan.factor_tiles()
    Rh = np.zeros((n, m)).T
    Rh = np.asfortranarray(np.full((m, n), 3.0))
    plan.store_r(Rh)
    assert np.array_equal(Rh, Rg)
    # Q of a row split = diag(Q_g) E Q_top (tqr.h): thin Q, residual, Q^T A and least squares
    Q, res = thin_q_and_residual(plan, A, Rg)
    assert res <= RES_TOL and np.linalg.norm(Q.T @ Q - np.eye(n)) <= ORTH_TOL, res
    QtA = dev_colmajor(A)
    plan.apply_qt(QtA, "T")
    assert colnorm_rel_err(np.triu(to_np(QtA)[:n]), ref.R) <= R_TOL
    B = synthetic.gaussian(m, 3, 7550 + m)
    Bd = dev_colmajor(B)
    plan.solve_ls(Bd)
    np.testing.assert_allclose(to_np(Bd)[:n], oracle.solve_ls(A, B), rtol=1e-8, atol=1e-10)
    plan.close()


def test_row_split_nccl_single_rank():
    """The multi-process row split (NCCL all-gather of the owners' R factors) with a 1-rank
    communicator: one row block, then the stage-2 refactorisation of its R."""
    m, n, nb, ib = 8192, 512, 512, 32
    A = synthetic.gaussian(m, n, 7600)
    uid = tqr.tqr_nccl_unique_id()
    plan = tqr.Plan(m, n, nb, ib, ndev=1, rank=0, world=1, nccl_id=uid, row_split=1)
    Ad = dev_colmajor(A)
    plan.factor(Ad)
    Rg = to_np(Ad)
    assert colnorm_rel_err(np.triu(Rg[:n]), oracle.qr(A).R) <= R_TOL
    assert np.all(np.tril(Rg, -1) == 0.0)
    plan.close()


def _sampled_checks(plan, Ad, Rd, m, n, nb, seed, ncols_oracle):
    """Full-size parity in the bench launch configuration (tqr_load + tqr_factor_tiles +
    tqr_store_r on device buffers):
      * R(:, :J) against the oracle's QR of A(:, :J) (R's leading columns depend only on the
        leading columns of A, so the oracle computes them exactly at this size);
      * sampled entries of R^T R = A^T A over the whole matrix (every column of R);
      * random-probe residual ||A x - Q (R x)|| / (||A|| ||x||) through tqr_apply_qt('N')."""
    J = ncols_oracle
    Aj = Ad[:, :J].cpu().numpy()
    ref = oracle.qr(Aj, nthreads=0)
    assert colnorm_rel_err(np.triu(Rd[:J, :J].cpu().numpy()), ref.R) <= R_TOL
    g = torch.Generator().manual_seed(seed)
    ii = torch.randint(0, n, (64,), generator=g).cuda()
    jj = torch.randint(0, n, (64,), generator=g).cuda()
    Ri, Rj = Rd[:n][:, ii], Rd[:n][:, jj]
    Ai, Aj2 = Ad[:, ii], Ad[:, jj]
    lhs = (Ri * Rj).sum(0)
    rhs = (Ai * Aj2).sum(0)
    scale = Ai.norm(dim=0) * Aj2.norm(dim=0)
    assert float(((lhs - rhs).abs() / scale).max()) <= 1e-12
    X = torch.randn((n, 3), dtype=torch.float64, generator=g).cuda()
    RX = torch.zeros((3, m), dtype=torch.float64, device="cuda").t()
    RX[:n] = torch.triu(Rd[:n]) @ X
    plan.apply_qt(RX, "N")
    res = (Ad @ X - RX).norm() / (Ad.norm() * X.norm())
    assert float(res) <= RES_TOL


@pytest.mark.slow
def test_full_size_c5_bench_configuration():
    """C5 (32768^2, nb=512, ib=32) exactly as bench.py runs it (device-resident, seeded randn)."""
    m, n, nb, ib, seed = 32768, 32768, 512, 32, 105
    gen = torch.Generator(device="cuda").manual_seed(seed)
    Ad = torch.randn((n, m), dtype=torch.float64, device="cuda", generator=gen).t()
    Rd = torch.empty((n, m), dtype=torch.float64, device="cuda").t()
    with tqr.Plan(m, n, nb, ib, profile=True) as plan:
        plan.load(Ad)
        plan.factor_tiles()
        plan.store_r(Rd)
        assert torch.all(torch.tril(Rd[:n], -1) == 0)
        _sampled_checks(plan, Ad, Rd, m, n, nb, 7, 1024)
    del Ad, Rd
    torch.cuda.empty_cache()


@pytest.mark.slow
def test_full_size_c4_tall_skinny():
    """C4 (1048576 x 512, nb=512): one panel column, the 2047-long flat TSQRT chain."""
    m, n, nb, ib, seed = 1048576, 512, 512, 32, 104
    gen = torch.Generator(device="cuda").manual_seed(seed)
    Ad = torch.randn((n, m), dtype=torch.float64, device="cuda", generator=gen).t()
    Rd = torch.empty((n, m), dtype=torch.float64, device="cuda").t()
    with tqr.Plan(m, n, nb, ib) as plan:
        plan.load(Ad)
        plan.factor_tiles()
        plan.store_r(Rd)
        _sampled_checks(plan, Ad, Rd, m, n, nb, 8, 512)
        # thin-Q orthogonality at full size (reading Q18): Q [I; 0]
        E = torch.zeros((n, m), dtype=torch.float64, device="cuda").t()
        E[:n, :n] = torch.eye(n, dtype=torch.float64, device="cuda")
        plan.apply_qt(E, "N")
        I = torch.eye(n, dtype=torch.float64, device="cuda")
        orth = float((E.t() @ E - I).norm())
    # north_star's absolute bar (reading Q19: met by Householder QR at C4, LAPACK 1.5e-14 at
    # 262144 x 512); cuSOLVER's geqrf on the same input is printed for context
    Q2, _ = torch.linalg.qr(Ad)
    orth_ref = float((Q2.t() @ Q2 - I).norm())
    print("C4 ||Q^TQ - I||_F = %.3e (cuSOLVER geqrf %.3e)" % (orth, orth_ref))
    assert orth <= ORTH_TOL, (orth, orth_ref)
    del Ad, Rd, E, Q2
    torch.cuda.empty_cache()


TREES = [
    # (m, n, nb, ib, L): TS domains of L tiles + flat TT merge chain (NEXT-1), forced
    (512, 128, 64, 16, 2),      # p=8, q=2: 4 domains at step 0, 4 at step 1 (last domain 1 tile)
    (1024, 256, 64, 16, 3),     # p=16, q=4: uneven domains, 6 -> 5 domains
    (2048, 512, 128, 32, 4),    # p=16, q=4 at nb=128
    (3072, 512, 512, 32, 2),    # q=1 at nb=512: 3 domains
    (1000, 300, 64, 16, 3),     # ragged both ways
    (768, 768, 256, 32, 1),     # L=1: every tile its own domain (pure TT-merge chain)
]


@pytest.mark.parametrize("one_cta", ["0", "1"])
@pytest.mark.parametrize("m,n,nb,ib,L", TREES)
def test_tree_matches_oracle(m, n, nb, ib, L, one_cta, monkeypatch):
    """Both domain phases: wavefront jobs (panel kernel, one job per domain) and one CTA per
    domain (domain_kernel)."""
    monkeypatch.setenv("TQR_TREE_ONE_CTA", one_cta)
    A = synthetic.gaussian(m, n, 5000 + m + n + nb + L)
    plan, Rg = gpu_qr(A, nb, ib, tree_domain=L)
    ref = oracle.qr(A)
    assert colnorm_rel_err(np.triu(Rg[:n]), ref.R) <= R_TOL
    assert np.all(np.tril(Rg, -1) == 0.0)
    Q, res = thin_q_and_residual(plan, A, Rg)
    assert res <= RES_TOL, res
    orth = np.linalg.norm(Q.T @ Q - np.eye(n))
    assert orth <= ORTH_TOL, (orth, lapack_orth(A))
    B = synthetic.gaussian(m, 2, 5100 + m)
    Bd = dev_colmajor(B)
    plan.solve_ls(Bd)
    np.testing.assert_allclose(to_np(Bd)[:n], oracle.solve_ls(A, B), rtol=1e-8, atol=1e-10)
    plan.close()


MERGES = [
    # (m, n, nb, ib, L, G): merge tree -- per level, groups of G heads (G >= sqrt(D): two levels)
    (1024, 128, 64, 16, 1, 4),      # p=16: 16 domains -> 4 groups of 4 (step 1: 15 -> 4, last of 3)
    (1024, 128, 64, 16, 1, 2),      # binary tree: 16 -> 8 -> 4 -> 2 -> 1 (step 1: 15 heads, odd levels)
    (3000, 64, 64, 16, 1, 3),       # 47 heads, G=3: 47 -> 16 -> 6 -> 2 -> 1, ragged rows
    (2048, 256, 64, 16, 2, 2),      # binary, ragged per step
    (8192, 512, 512, 32, 1, 2),     # binary at nb=512, q=1
    (2048, 256, 64, 16, 2, 3),      # p=32, q=4: 16 -> 6 groups (last of 1 domain), ragged per step
    (1000, 300, 64, 16, 1, 5),      # ragged both ways
    (8192, 512, 512, 32, 2, 3),     # q=1 at nb=512: 8 domains -> groups 3,3,2
    (8192, 512, 512, 32, 1, 4),     # 16 domains -> 4 x 4
]


@pytest.mark.parametrize("m,n,nb,ib,L,G", MERGES)
def test_merge_tree_matches_oracle(m, n, nb, ib, L, G):
    A = synthetic.gaussian(m, n, 5300 + m + n + nb + L + G)
    plan, Rg = gpu_qr(A, nb, ib, tree_domain=L, tree_group=G)
    ref = oracle.qr(A)
    assert colnorm_rel_err(np.triu(Rg[:n]), ref.R) <= R_TOL
    assert np.all(np.tril(Rg, -1) == 0.0)
    Q, res = thin_q_and_residual(plan, A, Rg)
    assert res <= RES_TOL, res
    orth = np.linalg.norm(Q.T @ Q - np.eye(n))
    assert orth <= ORTH_TOL, (orth, lapack_orth(A))
    B = synthetic.gaussian(m, 2, 5400 + m)
    Bd = dev_colmajor(B)
    plan.solve_ls(Bd)
    np.testing.assert_allclose(to_np(Bd)[:n], oracle.solve_ls(A, B), rtol=1e-8, atol=1e-10)
    plan.close()
    # the flat merge chain reaches the same R (unique) and the logical-device partition replays
    # the merge tree through the broadcast path bitwise
    _, Rf = gpu_qr(A, nb, ib, tree_domain=L, tree_group=-1)
    assert colnorm_rel_err(np.triu(Rg[:n]), np.triu(Rf[:n])) <= R_TOL
    if n > nb:
        _, Rp = gpu_qr(A, nb, ib, tree_domain=L, tree_group=G, ndev=2, guide=[1, 0], logical_devices=True)
        assert np.array_equal(Rg, Rp)
        assert colnorm_rel_err(np.triu(Rp[:n]), ref.R) <= R_TOL


def test_tree_auto_for_single_column_and_partition():
    """q == 1 picks the tree automatically; guide-array partitions with logical devices replay the
    same tree through the broadcast path (merge images / T travel with the panel)."""
    m, n, nb, ib = 8192, 512, 512, 32           # p = 16 -> L = 2, 8 domains
    A = synthetic.gaussian(m, n, 5200)
    plan, Rg = gpu_qr(A, nb, ib)
    assert colnorm_rel_err(np.triu(Rg[:n]), oracle.qr(A).R) <= R_TOL
    _, Rf = gpu_qr(A, nb, ib, tree_domain=-1)
    assert colnorm_rel_err(np.triu(Rg[:n]), np.triu(Rf[:n])) <= R_TOL
    m2, n2 = 1024, 512
    A2 = synthetic.gaussian(m2, n2, 5201)
    _, R1 = gpu_qr(A2, 64, 16, tree_domain=3)
    plan2, R2 = gpu_qr(A2, 64, 16, tree_domain=3, ndev=3, guide=[2, 0, 1], logical_devices=True)
    assert np.array_equal(R1, R2)
    assert colnorm_rel_err(np.triu(R2[:n2]), oracle.qr(A2).R) <= R_TOL
    Q, res = thin_q_and_residual(plan2, A2, R2)
    assert res <= RES_TOL and np.linalg.norm(Q.T @ Q - np.eye(n2)) <= ORTH_TOL
