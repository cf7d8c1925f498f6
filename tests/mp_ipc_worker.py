"""One rank of a multi-process tiled QR (launched by tests/test_gpu_multiproc.py via torchrun).

Every rank runs the REAL multi-process executor of libtqr.so (tqr_create_ex with rank / world, the
CUDA-IPC panel transport, tqr_ipc_handle / tqr_ipc_connect) on cuda:0 -- several ranks share the one
GPU of the test box, each in its own process and CUDA context, exactly as one rank per GPU would
run on a multi-GPU node except that the peer copies stay in one HBM.  torch.distributed (gloo) is
used only to exchange the IPC export blobs and for the host barrier.

    torchrun --nproc-per-node W tests/mp_ipc_worker.py OUT_DIR m n nb ib dtype guide tree row_split
      dtype: f64 | f32; guide: comma list or "-"; tree: tree_domain; row_split: 0 | 1

Writes OUT_DIR/rank<r>.npz: R (A <- R of tqr_factor on a device A), QtA (apply_qt 'T' on A),
Qthin (apply_qt 'N' on [I; 0]), X (solve_ls of B), issued (tqr_issued_ops), schedule (tqr_schedule).
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import synthetic  # noqa: E402
import paper_conf_icpp_kimp13_b200 as tqr  # noqa: E402


def main():
    out, m, n, nb, ib, dts, guide, tree, rs = sys.argv[1:10]
    m, n, nb, ib, tree, rs = int(m), int(n), int(nb), int(ib), int(tree), int(rs)
    guide = None if guide == "-" else [int(x) for x in guide.split(",")]
    rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
    torch.cuda.set_device(0)
    dist.init_process_group("gloo")
    f32 = dts == "f32"
    npdt = np.float32 if f32 else np.float64
    A = synthetic.gaussian(m, n, 9000 + m + n).astype(npdt)
    B = synthetic.gaussian(m, 3, 9100 + m).astype(npdt)

    def dev(X):
        return torch.from_numpy(np.ascontiguousarray(X.T)).cuda().t()

    plan = tqr.Plan(m, n, nb, ib, dtype=tqr.TQR_F32 if f32 else tqr.TQR_F64, ndev=world, guide=guide,
                    rank=rank, world=world, transport="ipc", tree_domain=tree, row_split=1 if rs else -1)
    plan.connect()
    res = {}
    for it in range(2):                      # twice: the flags must re-arm across factorizations
        Ad = dev(A)
        plan.factor(Ad)
        res["R%d" % it] = Ad.cpu().numpy()
    Ah = np.asfortranarray(A.copy())         # host A: the streamed path of tqr_factor
    plan.factor(Ah)
    res["Rhost"] = Ah
    if not rs:
        res["issued"] = np.array(plan.issued_ops(), dtype=np.int32).reshape(-1, 5)
        res["schedule"] = np.array(tqr.tqr_schedule(m, n, nb, world, guide, rank), dtype=np.int32).reshape(-1, 5)
    if rs:                                   # Q stays distributed across processes (row split)
        torch.cuda.synchronize()
        dist.barrier()
        plan.close()
        np.savez(os.path.join(out, "rank%d.npz" % rank), **res)
        dist.barrier()
        dist.destroy_process_group()
        return
    QtA = dev(A)
    plan.apply_qt(QtA, "T")
    res["QtA"] = QtA.cpu().numpy()
    E = np.zeros((m, n), dtype=npdt)
    E[:n, :n] = np.eye(n, dtype=npdt)
    Ed = dev(E)
    plan.apply_qt(Ed, "N")
    res["Qthin"] = Ed.cpu().numpy()
    Bd = dev(B)
    plan.solve_ls(Bd)
    res["X"] = Bd.cpu().numpy()[:n]
    torch.cuda.synchronize()
    dist.barrier()
    plan.close()
    np.savez(os.path.join(out, "rank%d.npz" % rank), **res)
    dist.barrier()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
