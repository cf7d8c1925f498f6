"""Multi-process parity: the real multi-process executor (one process per owner, CUDA-IPC panel
transport) at world 2 and 3, all ranks on cuda:0 of the test box.

Each case launches tests/mp_ipc_worker.py under torchrun; every rank factors the same seeded matrix
with its guide-array share of the column tiles (Eq. 12), panels travel rank to rank through
IPC-mapped receive slots ordered by stream flags, then apply_qt / solve_ls gather the distributed
reflectors.  The assembled R must equal the single-owner CUDA run bitwise (the same arithmetic in
the same order) AND match the oracle within the north-star bars; Q^T A, thin Q and the least
squares solution are checked against the oracle too, and every rank's issued-op trace must be its
tqr_schedule list (the executor consumes the schedule)."""
import os
import socket
import subprocess
import sys

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
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _run(tmp_path, world, m, n, nb, ib, dts="f64", guide=None, tree=-1, rs=0, env=None):
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes", "1", "--nproc-per-node", str(world),
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()),
           os.path.join(ROOT, "tests", "mp_ipc_worker.py"), str(tmp_path), str(m), str(n), str(nb), str(ib), dts,
           "-" if guide is None else ",".join(map(str, guide)), str(tree), str(rs)]
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=ROOT, env=dict(os.environ, **(env or {})))
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-3000:]
    return [dict(np.load(os.path.join(tmp_path, "rank%d.npz" % k))) for k in range(world)]


def _assemble_cols(outs, key, owner, nb, n):
    R = outs[0][key].copy()
    for j in range(0, (n + nb - 1) // nb):
        R[:, j * nb:(j + 1) * nb] = outs[owner(j)][key][:, j * nb:(j + 1) * nb]
    return R


def _single_owner(A, nb, ib, dtype, **kw):
    plan = tqr.Plan(A.shape[0], A.shape[1], nb, ib, dtype=dtype, **kw)
    Ad = torch.from_numpy(np.ascontiguousarray(A.T)).cuda().t()
    plan.factor(Ad)
    plan.close()
    return Ad.cpu().numpy()


CASES = [
    # (world, m, n, nb, ib, dtype, guide, tree)
    (2, 1024, 1024, 128, 32, "f64", None, -1),                    # cyclic {0, 1}
    (2, 1024, 1024, 128, 32, "f64", [0, 0, 1, 1], -1),            # pairs
    (3, 1536, 1536, 128, 32, "f64", [1, 0, 1, 0, 1, 2], -1),      # the paper's guide
    (3, 1100, 1030, 256, 32, "f64", None, -1),                    # ragged tails, 3 ranks
    (2, 2048, 2048, 512, 32, "f64", [1, 0], -1),                  # nb = 512, root 1 first
    (2, 2048, 512, 128, 32, "f64", None, 4),                      # tree mode: merge images travel too
    (2, 1024, 1024, 128, 32, "f32", None, -1),                    # FP32 plan
]


@pytest.mark.parametrize("world,m,n,nb,ib,dts,guide,tree", CASES)
def test_multiprocess_ipc_matches_single_owner_and_oracle(tmp_path, world, m, n, nb, ib, dts, guide, tree):
    f32 = dts == "f32"
    npdt = np.float32 if f32 else np.float64
    dtype = tqr.TQR_F32 if f32 else tqr.TQR_F64
    outs = _run(tmp_path, world, m, n, nb, ib, dts, guide, tree)
    A = synthetic.gaussian(m, n, 9000 + m + n).astype(npdt)
    B = synthetic.gaussian(m, 3, 9100 + m).astype(npdt)
    g = guide if guide is not None else list(range(world))
    owner = lambda j: g[j % len(g)]  # noqa: E731
    R1 = _single_owner(A, nb, ib, dtype, tree_domain=tree)
    for key in ("R0", "R1", "Rhost"):
        R = _assemble_cols(outs, key, owner, nb, n)
        assert np.array_equal(R, R1), key                     # bitwise = the single-owner executor
    Ad = A.astype(np.float64)
    ref = oracle.qr(Ad)
    r_tol, res_tol, orth_tol = (1e-3, 1e-5, 1e-5) if f32 else (1e-10, 1e-13, 1e-13)
    Rn = np.triu(R1[:n]).astype(np.float64)
    assert colnorm_rel_err(Rn, ref.R) <= r_tol
    for k in range(world):                                    # apply / solve: the same full result everywhere
        assert np.array_equal(outs[k]["QtA"], outs[0]["QtA"]) and np.array_equal(outs[k]["X"], outs[0]["X"])
    QtA = outs[0]["QtA"].astype(np.float64)
    assert colnorm_rel_err(np.triu(QtA[:n]), ref.R) <= r_tol
    Q = outs[0]["Qthin"].astype(np.float64)
    orth = np.linalg.norm(Q.T @ Q - np.eye(n))
    # LAPACK on the same input in the same precision (torch CPU: a real sgeqrf/sorgqr for FP32;
    # numpy.linalg would compute an FP32 problem in FP64)
    Ql, _ = torch.linalg.qr(torch.from_numpy(np.ascontiguousarray(A)))
    Ql = Ql.double()
    orth_lapack = float((Ql.t() @ Ql - torch.eye(n, dtype=torch.float64)).norm())
    if f32 or n >= 2048:
        # reading Q19: FP32 (sgeqrf already exceeds 1e-5: 2.3e-5 at 1024) and n >= 2048 (LAPACK's own
        # FP64 loss grows ~1.6e-15 sqrt(n): 7e-14 at 2048) -> max(bar, 2 x LAPACK on the same input)
        orth_tol = max(orth_tol, 2.0 * orth_lapack)
    assert orth <= orth_tol, (orth, orth_lapack)
    assert np.linalg.norm(Ad - Q @ Rn) / np.linalg.norm(Ad) <= res_tol
    Xo = oracle.solve_ls(Ad, B.astype(np.float64))
    np.testing.assert_allclose(outs[0]["X"], Xo, rtol=1e-3 if f32 else 1e-8, atol=1e-3 if f32 else 1e-10)
    for k in range(world):                                    # the executor issued exactly its schedule
        iss, sch = outs[k]["issued"], outs[k]["schedule"]
        assert len(iss) == len(sch)
        key = lambda r: (r[1], r[0], r[3])  # noqa: E731  (per step: PANEL, BCAST, the UPDATE columns)
        assert sorted(map(tuple, iss), key=key) == sorted(map(tuple, sch), key=key)
        steps = [r[1] for r in iss]
        assert steps == sorted(steps)                         # steps issued in schedule order


@pytest.mark.parametrize("world,m,n,nb,ib", [(2, 8192, 512, 512, 32), (3, 5000, 200, 256, 32)])
def test_multiprocess_ipc_row_split(tmp_path, world, m, n, nb, ib):
    """Row split across processes (C4 shape class): per-rank TS trees, R_g gathered into rank 0's
    stack through IPC reads, stage-2 merge on rank 0; rank 0 returns R (others their zero rows)."""
    outs = _run(tmp_path, world, m, n, nb, ib, "f64", None, 0, 1)
    A = synthetic.gaussian(m, n, 9000 + m + n)
    ref = oracle.qr(A)
    ranges = tqr.tqr_row_split_ranges(m, nb, world)
    for key in ("R0", "R1", "Rhost"):
        R = outs[0][key].copy()
        for g, (r0, rows) in enumerate(ranges):
            if g:
                R[r0:r0 + rows] = outs[g][key][r0:r0 + rows]
        assert colnorm_rel_err(np.triu(R[:n]), ref.R) <= 1e-10
        assert np.all(np.tril(R, -1) == 0.0)
    # logical-owner row split (single process) is the same arithmetic: bitwise equal R
    plan = tqr.Plan(m, n, nb, ib, ndev=world, logical_devices=True, row_split=1)
    Ad = torch.from_numpy(np.ascontiguousarray(A.T)).cuda().t()
    plan.factor(Ad)
    Rl = Ad.cpu().numpy()
    plan.close()
    assert np.array_equal(np.triu(outs[0]["R0"][:n]), np.triu(Rl[:n]))


def test_multiprocess_ipc_remote_trailing_chunks(tmp_path):
    """The chunked IPC transfer + trailing lookahead (default on distinct GPUs) forced on the shared
    test GPU (TQR_LA_REMOTE=2): chunk c of panel k is copied once the panel published its last tile
    and raises a chunk flag the next owner's lookahead kernel waits on.  Bitwise the single-owner R."""
    world, m, n, nb, ib = 2, 2048, 2048, 256, 32
    outs = _run(tmp_path, world, m, n, nb, ib, "f64", None, -1, 0, env={"TQR_LA_REMOTE": "2"})
    A = synthetic.gaussian(m, n, 9000 + m + n)
    R1 = _single_owner(A, nb, ib, tqr.TQR_F64)
    for key in ("R0", "R1", "Rhost"):
        R = _assemble_cols(outs, key, lambda j: j % world, nb, n)
        assert np.array_equal(R, R1), key
    assert colnorm_rel_err(np.triu(R1[:n]), oracle.qr(A).R) <= 1e-10
