"""Multi-process (world_size 2 and 3) CPU test of the distributed path's host logic over gloo.

Each rank asks the C library for its schedule (`tqr_schedule`: Fig. 3 DAG partitioned by the
guide array, Eq. 12), owns only its column tiles, executes PANEL / BCAST / UPDATE records in
that order with LAPACK tile kernels (scipy dgeqrt/dtpqrt/dgemqrt/dtpmqrt -- test
infrastructure standing in for the CUDA kernels), and exchanges panels with
torch.distributed.broadcast exactly where the schedule says.  A mismatched schedule deadlocks
or mis-sizes a collective; a wrong owner, payload or ordering changes R.  R is gathered and
checked against the CPU oracle (reading Q16, 1e-10)."""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, guide, m, n, nb, ib, seed, port, out_dir):
    import sys
    sys.path.insert(0, ROOT)
    import scipy.linalg.lapack as lap
    import synthetic
    import paper_conf_icpp_kimp13_b200 as tqr

    dist.init_process_group("gloo", init_method="tcp://127.0.0.1:%d" % port, rank=rank, world_size=world)
    p, q = m // nb, n // nb
    A = synthetic.gaussian(m, n, seed)
    ops = tqr.tqr_schedule(m, n, nb, world, guide, rank)
    own = [j for j in range(q) if guide[j % len(guide)] == rank]
    tiles = {(i, j): np.asfortranarray(A[i * nb:(i + 1) * nb, j * nb:(j + 1) * nb].copy())
             for j in own for i in range(p)}
    Tf = {}
    panels = {}
    bytes_seen = []
    for op, k, _i, j, root in ops:
        if op == tqr.OP_PANEL:
            assert root == rank and k in own
            a, t, info = lap.dgeqrt(ib, tiles[(k, k)])
            assert info == 0
            tiles[(k, k)], Tf[(k, k)] = a, t
            for i in range(k + 1, p):
                r, b, t, info = lap.dtpqrt(0, ib, np.triu(tiles[(k, k)]), tiles[(i, k)])
                assert info == 0
                tiles[(k, k)] = np.where(np.triu(np.ones((nb, nb), bool)), r, tiles[(k, k)])
                tiles[(i, k)], Tf[(i, k)] = b, t
        elif op == tqr.OP_BCAST:
            # payload, as the executor sends it: the reflector images of tiles k..p-1
            # of column k, their T factors, and the explicit unit-lower V of the diagonal tile
            # (Vexp: the UNMQR operand; the diagonal tile itself holds R above its diagonal)
            size = (p - k) * nb * nb + (p - k) * ib * nb + nb * nb
            buf = torch.zeros(size, dtype=torch.float64)
            if root == rank:
                vexp = np.tril(tiles[(k, k)], -1) + np.eye(nb)
                parts = [tiles[(i, k)].ravel(order="F") for i in range(k, p)] + \
                        [Tf[(i, k)].ravel(order="F") for i in range(k, p)] + [vexp.ravel(order="F")]
                buf.copy_(torch.from_numpy(np.concatenate(parts)))
            dist.broadcast(buf, src=root)
            bytes_seen.append(8 * size)
            v = buf.numpy()
            Vt = [v[(i - k) * nb * nb:(i - k + 1) * nb * nb].reshape((nb, nb), order="F") for i in range(k, p)]
            off = (p - k) * nb * nb
            Tt = [v[off + (i - k) * ib * nb: off + (i - k + 1) * ib * nb].reshape((ib, nb), order="F")
                  for i in range(k, p)]
            off += (p - k) * ib * nb
            Vexp = v[off:off + nb * nb].reshape((nb, nb), order="F")
            assert np.all(np.triu(Vexp, 1) == 0) and np.all(np.diag(Vexp) == 1.0)
            panels[k] = (Vt, Tt, Vexp)
        elif op == tqr.OP_UPDATE:
            assert guide[j % len(guide)] == rank and j > k
            Vt, Tt, Vexp = panels[k]
            c, info = lap.dgemqrt(np.asfortranarray(Vexp), Tt[0], tiles[(k, j)], side="L", trans="T")
            assert info == 0
            tiles[(k, j)] = c
            for i in range(k + 1, p):
                a_, b_, info = lap.dtpmqrt(0, Vt[i - k], Tt[i - k], tiles[(k, j)], tiles[(i, j)], side="L", trans="T")
                assert info == 0
                tiles[(k, j)], tiles[(i, j)] = a_, b_
    # gather R column tiles at rank 0
    mine = {j: np.vstack([tiles[(i, j)] for i in range(p)])[:n] for j in own}
    gathered = [None] * world
    dist.all_gather_object(gathered, mine)
    if rank == 0:
        R = np.zeros((n, n))
        for d in gathered:
            for j, colblk in d.items():
                R[:, j * nb:(j + 1) * nb] = colblk
        np.save(os.path.join(out_dir, "R.npy"), np.triu(R))
        np.save(os.path.join(out_dir, "bytes.npy"), np.array(bytes_seen))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,guide", [(2, [0, 1]), (2, [1, 0, 0]), (3, [1, 0, 1, 0, 1, 2])])
def test_distributed_schedule_and_broadcast(tmp_path, world, guide):
    import oracle
    import synthetic
    from conftest import colnorm_rel_err
    from paper_conf_icpp_kimp13_b200 import build
    build.build()
    m, n, nb, ib, seed = 384, 384, 64, 16, 4242
    mp.spawn(_worker, args=(world, guide, m, n, nb, ib, seed, _free_port(), str(tmp_path)), nprocs=world, join=True)
    R = np.load(tmp_path / "R.npy")
    ref = oracle.qr(synthetic.gaussian(m, n, seed)).R
    assert colnorm_rel_err(R, ref) <= 1e-10
    p = m // nb
    assert list(np.load(tmp_path / "bytes.npy")) == [8 * ((m - k * nb) * nb + (p - k) * ib * nb + nb * nb)
                                                     for k in range(n // nb)]


def _rowsplit_worker(rank, world, m, n, nb, ib, seed, port, out_dir):
    """Row split (tqr_options.row_split) protocol with LAPACK tile kernels standing in for the
    CUDA ones: rank g takes its rows from tqr_row_split_ranges, factors them as a flat TS chain
    (dgeqrt + dtpqrt), the owners' nb x n triangular factors are all-gathered (the NCCL
    all-gather of the library), and rank 0 factors the stacked triu(R_g)."""
    import sys
    sys.path.insert(0, ROOT)
    import scipy.linalg.lapack as lap
    import synthetic
    import paper_conf_icpp_kimp13_b200 as tqr

    dist.init_process_group("gloo", init_method="tcp://127.0.0.1:%d" % port, rank=rank, world_size=world)
    A = synthetic.gaussian(m, n, seed)
    ranges = tqr.tqr_row_split_ranges(m, nb, world)
    r0, rows = ranges[rank]
    blk = np.zeros((-(-rows // nb) * nb, n))
    blk[:rows] = A[r0:r0 + rows]
    a, t, info = lap.dgeqrt(ib, np.asfortranarray(blk[:nb]))
    assert info == 0
    top = np.triu(a)
    for i in range(1, blk.shape[0] // nb):
        r, b, t, info = lap.dtpqrt(0, ib, top, np.asfortranarray(blk[i * nb:(i + 1) * nb]))
        assert info == 0
        top = np.triu(r)
    send = torch.from_numpy(np.ascontiguousarray(top[:nb, :n]))
    recv = [torch.zeros_like(send) for _ in range(world)]
    dist.all_gather(recv, send)
    if rank == 0:
        stk = np.vstack([x.numpy() for x in recv])             # ndev*nb x n, triu blocks
        a, t, info = lap.dgeqrt(ib, np.asfortranarray(stk[:nb]))
        top = np.triu(a)
        for g in range(1, world):
            r, b, t, info = lap.dtpqrt(0, ib, top, np.asfortranarray(stk[g * nb:(g + 1) * nb]))
            top = np.triu(r)
        np.save(os.path.join(out_dir, "R.npy"), top[:n, :n])
        np.save(os.path.join(out_dir, "ranges.npy"), np.array(ranges))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,m", [(2, 1024), (3, 1000)])
def test_row_split_protocol(tmp_path, world, m):
    import oracle
    import synthetic
    from conftest import colnorm_rel_err
    from paper_conf_icpp_kimp13_b200 import build
    build.build()
    n, nb, ib, seed = 64, 64, 16, 4343
    mp.spawn(_rowsplit_worker, args=(world, m, n, nb, ib, seed, _free_port(), str(tmp_path)), nprocs=world, join=True)
    R = np.load(tmp_path / "R.npy")
    ref = oracle.qr(synthetic.gaussian(m, n, seed)).R
    assert colnorm_rel_err(R, ref) <= 1e-10
    ranges = np.load(tmp_path / "ranges.npy")
    assert ranges[0][0] == 0 and sum(r for _, r in ranges) == m                 # contiguous cover
    assert all(ranges[g][0] + ranges[g][1] == ranges[g + 1][0] for g in range(world - 1))
    assert all(r0 % nb == 0 and r >= n for r0, r in ranges)
