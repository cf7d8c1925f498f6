"""Pins for the CPU oracle (no GPU).  Each test ties oracle/ to something other than itself:
closed forms, a textbook exact case, 50-digit brute force, invariants, special cases, and
LAPACK.  A plausible slip (dropped term, wrong sign, transposed operand, wrong row range)
fails at least one of them."""
import json
import os

import numpy as np
import pytest

import oracle
import synthetic
from conftest import colnorm_rel_err, sign_normalise_R

EPS = np.finfo(np.float64).eps


def _load(golden_dir, name):
    with open(os.path.join(golden_dir, name)) as f:
        return json.load(f)


def test_closed_form_2x2(golden_dir):
    g = _load(golden_dir, "qr_2x2_closed_form.json")
    f = oracle.qr(np.array(g["A"], dtype=float))
    np.testing.assert_allclose(sign_normalise_R(f.R), np.array(g["R"]), rtol=0, atol=1e-14)


def test_textbook_3x3_R_and_Q(golden_dir):
    g = _load(golden_dir, "qr_3x3_textbook.json")
    A = np.array(g["A"], dtype=float)
    f = oracle.qr(A)
    d = np.where(np.diag(f.R) < 0, -1.0, 1.0)
    np.testing.assert_allclose(f.R * d[:, None], np.array(g["R"], float), rtol=0, atol=1e-12)
    Q = f.thin_q() * d[None, :]
    np.testing.assert_allclose(Q, np.array(g["Q_num"], float) / g["Q_den"], rtol=0, atol=1e-15)


def _mp_gram_schmidt_R(A, dps=50):
    """Classical Gram-Schmidt in 50-digit arithmetic: the exact (R_ii > 0) R to >> 16 digits."""
    import mpmath as mp

    mp.mp.dps = dps
    m, n = A.shape
    cols = [[mp.mpf(float(A[i, j])) for i in range(m)] for j in range(n)]
    Q = []
    R = [[mp.mpf(0)] * n for _ in range(n)]
    for j in range(n):
        v = list(cols[j])
        for i, q in enumerate(Q):
            rij = mp.fsum(q[r] * cols[j][r] for r in range(m))
            R[i][j] = rij
            v = [v[r] - rij * q[r] for r in range(m)]
        nrm = mp.sqrt(mp.fsum(x * x for x in v))
        R[j][j] = nrm
        Q.append([x / nrm for x in v])
    return np.array([[float(R[i][j]) for j in range(n)] for i in range(n)])


@pytest.mark.parametrize("m,n,seed", [(1, 1, 1), (2, 2, 2), (5, 3, 3), (8, 8, 4), (7, 1, 5), (6, 6, 6)])
def test_mpmath_gram_schmidt(m, n, seed):
    A = synthetic.gaussian(m, n, seed)
    R_exact = _mp_gram_schmidt_R(A)
    f = oracle.qr(A)
    assert colnorm_rel_err(f.R, R_exact) < 50 * EPS


@pytest.mark.parametrize("m,n", [(64, 64), (200, 120), (257, 255)])
def test_invariants_RtR_det(m, n):
    A = synthetic.gaussian(m, n, m * 7 + n)
    f = oracle.qr(A)
    R = f.R
    # R^T R = A^T A
    lhs, rhs = R.T @ R, A.T @ A
    assert np.linalg.norm(lhs - rhs) <= 100 * n * EPS * np.linalg.norm(A) ** 2
    # strictly upper triangular R returned; Q^T A has a (numerically) zero lower part
    QtA = f.apply_q(A, "T")
    assert np.linalg.norm(np.tril(QtA, -1)) <= 100 * np.sqrt(m) * EPS * np.linalg.norm(A)
    np.testing.assert_allclose(np.triu(QtA[:n]), R, rtol=0, atol=100 * EPS * np.linalg.norm(A))
    if m == n:
        sign, logdet = np.linalg.slogdet(A)
        assert abs(np.sum(np.log(np.abs(np.diag(R)))) - logdet) < 1e-10 * n


def test_orthogonal_input_gives_diag_pm1():
    Q0, _ = np.linalg.qr(synthetic.gaussian(50, 50, 9))
    f = oracle.qr(Q0)
    np.testing.assert_allclose(np.abs(f.R), np.eye(50), atol=1e-13)


def test_triangular_and_diagonal_inputs():
    U = np.triu(synthetic.gaussian(40, 40, 10)) + 5 * np.eye(40)
    f = oracle.qr(U)
    np.testing.assert_allclose(sign_normalise_R(f.R), sign_normalise_R(U), rtol=0, atol=1e-13 * np.abs(U).max())
    D = np.diag(np.arange(-5.0, 5.0) + 0.5)
    f = oracle.qr(D)
    np.testing.assert_allclose(f.R, np.diag(np.abs(np.diag(D))) * np.sign(np.diag(f.R))[:, None], atol=1e-15)
    np.testing.assert_allclose(np.abs(np.diag(f.R)), np.abs(np.diag(D)), atol=1e-15)


def test_zero_column_reading_Q3():
    A = synthetic.gaussian(10, 6, 11)
    A[:, 2] = 0.0
    A[3:, 4] = 0.0
    f = oracle.qr(A)
    assert np.all(np.isfinite(f.R))
    assert np.all(f.V[:, 2] == 0.0)          # Q_2 = I
    lhs, rhs = f.R.T @ f.R, A.T @ A
    np.testing.assert_allclose(lhs, rhs, atol=1e-12)


@pytest.mark.parametrize("m,n", [(256, 256), (1024, 300)])
def test_lapack_agreement(m, n):
    A = synthetic.gaussian(m, n, 12)
    f = oracle.qr(A)
    R_lapack = np.linalg.qr(A, mode="r")
    assert colnorm_rel_err(f.R, R_lapack) < 1e-13


@pytest.mark.parametrize("scale", [1e300, 1e200, 1e-200, 1e-300])
def test_extreme_scaling_matches_lapack(scale):
    """Reading Q26: ||a_k|| (Alg. 1 lines 6 and 8) is the Euclidean norm, computed without
    overflow or underflow.  sqrt(sum x^2) is inf for entries ~1e200 and 0 for ~1e-200 (tau = 0,
    nothing eliminated); LAPACK's dlarfg/dnrm2 scale.  R(cA) = c R(A) for a power-of-ten c, so
    the oracle's R of the scaled matrix must match LAPACK's and c x the unscaled oracle R."""
    A = synthetic.gaussian(96, 64, 22)
    As = A * scale
    f = oracle.qr(As)
    assert np.all(np.isfinite(f.R))
    R_lapack = np.linalg.qr(As, mode="r")
    assert colnorm_rel_err(f.R, R_lapack) < 1e-13
    assert colnorm_rel_err(f.R / scale, oracle.qr(A).R) < 1e-13
    Q = f.thin_q()
    assert np.linalg.norm(Q.T @ Q - np.eye(64)) < 1e-13


def test_scaled_norm_bitwise_in_normal_range():
    """Power-of-two scaling is exact: in the normal range the scaled norm is bitwise the plain
    sqrt(sum x^2) of Alg. 1 (the closed forms above pin the same arithmetic)."""
    A = synthetic.gaussian(50, 1, 23) * 3.0
    f = oracle.qr(A)
    s = 0.0
    for x in A[:, 0]:                        # ascending rows, as Alg. 1's sum is taken
        s += float(x) * float(x)
    assert abs(f.R[0, 0]) == np.sqrt(s)


def test_thin_q_orthogonal_and_reconstructs():
    A = synthetic.gaussian(300, 120, 13)
    f = oracle.qr(A)
    Q = f.thin_q()
    assert np.linalg.norm(Q.T @ Q - np.eye(120)) < 1e-13
    assert np.linalg.norm(A - Q @ f.R) / np.linalg.norm(A) < 1e-14
    Qn, Rn = np.linalg.qr(A)
    d = np.sign(np.diag(f.R)) * np.sign(np.diag(Rn))
    np.testing.assert_allclose(Q * d[None, :], Qn, atol=1e-12)


def test_apply_q_roundtrip_and_transpose():
    A = synthetic.gaussian(120, 80, 14)
    f = oracle.qr(A)
    B = synthetic.gaussian(120, 7, 15)
    np.testing.assert_allclose(f.apply_q(f.apply_q(B, "T"), "N"), B, atol=1e-13)
    # <Q^T x, y> = <x, Q y>
    x, y = synthetic.gaussian(120, 1, 16)[:, 0], synthetic.gaussian(120, 1, 17)[:, 0]
    assert abs(f.apply_q(x, "T") @ y - x @ f.apply_q(y, "N")) < 1e-12


def test_solve_ls_matches_lstsq():
    A = synthetic.gaussian(200, 60, 18)
    b = synthetic.gaussian(200, 3, 19)
    x = oracle.solve_ls(A, b)
    x_ref = np.linalg.lstsq(A, b, rcond=None)[0]
    np.testing.assert_allclose(x, x_ref, rtol=1e-11, atol=1e-12)


def test_thread_count_bitwise_identical():
    A = synthetic.gaussian(300, 200, 20)
    r1 = oracle.qr(A, nthreads=1).R
    r4 = oracle.qr(A, nthreads=4).R
    assert np.array_equal(r1, r4)


def test_qr_columns_prefix_matches_full():
    A = synthetic.gaussian(90, 40, 21)
    part = oracle.qr_columns(A, 10)
    full = oracle.qr(A)
    np.testing.assert_allclose(np.triu(part[:10, :]), np.triu(np.hstack([full.R[:10], ]))[:10, :], atol=1e-12)


# ---- Algorithm 4 / Eq. 12 -------------------------------------------------------------

def test_guide_array_paper_example(golden_dir):
    g = _load(golden_dir, "guide_array_example.json")
    ratio = oracle.guide.get_ratio(g["rates"])
    assert ratio == g["ratio"]
    assert oracle.guide.generate_array(ratio) == g["guide_array"]


def test_guide_array_properties():
    rng = np.random.default_rng(0)
    for _ in range(200):
        p = int(rng.integers(1, 9))
        ratio = [int(x) for x in rng.integers(0, 6, size=p)]
        if sum(ratio) == 0:
            continue
        ga = oracle.guide.generate_array(ratio)
        assert len(ga) == sum(ratio)
        for d in range(p):
            assert ga.count(d) == ratio[d]
        # the device with the largest ratio appears first
        assert ga[0] == int(np.argmax(ratio))


def test_distribution_eq12():
    ga = [1, 0, 1, 0, 1, 2]
    assert [oracle.guide.distribute(i, ga) for i in range(13)] == [1, 0, 1, 0, 1, 2, 1, 0, 1, 0, 1, 2, 1]
    assert oracle.guide.generate_array([1, 1, 1, 1]) == [0, 1, 2, 3]


# ---- synthetic generator ----------------------------------------------------------------

def test_synthetic_counter_based_and_gaussian():
    A = synthetic.gaussian(300, 200, 7)
    rows = np.array([0, 5, 299, 17]); cols = np.array([0, 199, 3, 100])
    np.testing.assert_array_equal(synthetic.gaussian_entries(300, rows, cols, 7), A[rows, cols])
    assert abs(A.mean()) < 0.01 and abs(A.std() - 1) < 0.01
    assert not np.array_equal(A, synthetic.gaussian(300, 200, 8))
