"""paper_conf_icpp_kimp13_b200 -- B200-native tiled Householder QR (Kim & Park, ICPP'13).

Thin ctypes binding over the C ABI in ``include/tqr.h`` (libtqr.so, built in-tree for
sm_100a by ``build.py``).  Same names as the ABI: ``tqr_create``, ``tqr_factor``,
``tqr_apply_qt``, ``tqr_solve_ls``, ``tqr_destroy`` (+ the phase / helper calls), plus a
small ``Plan`` convenience class.  Argument marshalling only: every step of the
factorisation runs in the CUDA kernels of ``csrc/``.  There is no CPU fallback: if the
library cannot be loaded, every call raises.

Arrays: torch tensors (CUDA or CPU) or numpy arrays, column-major (stride(0) == 1 for torch,
Fortran order for numpy), dtype float64 (TQR_F64 plans) or float32 (TQR_F32 plans).  The leading
dimension is taken from the array.
"""
from __future__ import annotations

import ctypes
import os

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("TQR_LIB") or os.path.join(_PKG, "libtqr.so")   # TQR_LIB: probe builds only

TQR_F64, TQR_F32 = 0, 1
STATUS = {0: "TQR_OK", 1: "TQR_ERR_ARG", 2: "TQR_ERR_ALLOC", 3: "TQR_ERR_CUDA", 4: "TQR_ERR_NCCL",
          5: "TQR_ERR_STATE", 6: "TQR_ERR_SINGULAR", 7: "TQR_ERR_UNSUPPORTED"}
OP_PANEL, OP_BCAST, OP_UPDATE = 0, 1, 2
TRANSPORT = {"auto": 0, "nccl": 1, "ipc": 2}


class TqrError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__("%s: %s" % (STATUS.get(status, status), msg))
        self.status = status


class Options(ctypes.Structure):
    _fields_ = [("logical_devices", ctypes.c_int32), ("rank", ctypes.c_int32), ("world", ctypes.c_int32),
                ("nccl_id", ctypes.c_void_p), ("no_lookahead", ctypes.c_int32), ("profile", ctypes.c_int32),
                ("tree_domain", ctypes.c_int32), ("tree_group", ctypes.c_int32),
                ("row_split", ctypes.c_int32), ("transport", ctypes.c_int32)]


class TileTimes(ctypes.Structure):
    _fields_ = [("t_T", ctypes.c_double), ("t_E", ctypes.c_double), ("t_UT", ctypes.c_double),
                ("t_UE", ctypes.c_double)]


_lib = None


def lib():
    """Load libtqr.so (raises if it was not built: no fallback path exists)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError("libtqr.so not built: run `python -m paper_conf_icpp_kimp13_b200.build`")
        L = ctypes.CDLL(LIB_PATH)
        i64, i32, vp, P = ctypes.c_int64, ctypes.c_int32, ctypes.c_void_p, ctypes.POINTER
        L.tqr_create.argtypes = [i64, i64, i32, i32, i32, i32, P(i32), i32, P(vp)]
        L.tqr_create_ex.argtypes = [i64, i64, i32, i32, i32, i32, P(i32), i32, P(Options), P(vp)]
        L.tqr_factor.argtypes = [vp, vp, i64]
        L.tqr_load.argtypes = [vp, vp, i64]
        L.tqr_factor_tiles.argtypes = [vp]
        L.tqr_store_r.argtypes = [vp, vp, i64]
        L.tqr_apply_qt.argtypes = [vp, ctypes.c_char, vp, i64, i64]
        L.tqr_solve_ls.argtypes = [vp, vp, i64, i64]
        L.tqr_destroy.argtypes = [vp]
        L.tqr_status_string.argtypes = [i32]
        L.tqr_status_string.restype = ctypes.c_char_p
        L.tqr_last_error.argtypes = [vp]
        L.tqr_last_error.restype = ctypes.c_char_p
        L.tqr_nccl_unique_id.argtypes = [vp]
        L.tqr_owner.argtypes = [vp, i64]
        L.tqr_owner.restype = i32
        L.tqr_schedule.argtypes = [i64, i64, i32, i32, P(i32), i32, i32, P(i32), i64, P(i64)]
        L.tqr_generate_guide.argtypes = [P(i32), i32, P(i32), i32, P(i32)]
        L.tqr_select_main.argtypes = [i32, P(TileTimes), P(i32)]
        L.tqr_row_split_ranges.argtypes = [i64, i32, i32, P(i64), P(i64)]
        L.tqr_select_ndev.argtypes = [i32, i32, i32, i32, i32, P(TileTimes), P(ctypes.c_double), i32, P(i32),
                                      P(ctypes.c_double), P(i32)]
        L.tqr_kernel_stats.argtypes = [vp, i32, P(i64), P(ctypes.c_double), P(ctypes.c_double), i32]
        L.tqr_launch_count.argtypes = [vp]
        L.tqr_launch_count.restype = i64
        L.tqr_ipc_handle.argtypes = [vp, vp, i64, P(i64)]
        L.tqr_ipc_connect.argtypes = [vp, vp, i64]
        L.tqr_issued_ops.argtypes = [vp, P(i32), i64, P(i64)]
        L.tqr_plan_flags.argtypes = [vp]
        L.tqr_plan_flags.restype = i32
        for f in ("tqr_create", "tqr_create_ex", "tqr_factor", "tqr_load", "tqr_factor_tiles", "tqr_store_r",
                  "tqr_apply_qt", "tqr_solve_ls", "tqr_destroy", "tqr_nccl_unique_id", "tqr_schedule",
                  "tqr_generate_guide", "tqr_kernel_stats", "tqr_select_main", "tqr_select_ndev", "tqr_row_split_ranges",
                  "tqr_ipc_handle", "tqr_ipc_connect", "tqr_issued_ops"):
            getattr(L, f).restype = i32
        _lib = L
    return _lib


EXPORTED = ["tqr_create", "tqr_create_ex", "tqr_factor", "tqr_load", "tqr_factor_tiles", "tqr_store_r",
            "tqr_apply_qt", "tqr_solve_ls", "tqr_destroy", "tqr_status_string", "tqr_last_error",
            "tqr_nccl_unique_id", "tqr_owner", "tqr_schedule", "tqr_generate_guide", "tqr_kernel_stats",
            "tqr_launch_count", "tqr_select_main", "tqr_select_ndev", "tqr_row_split_ranges",
            "tqr_ipc_handle", "tqr_ipc_connect", "tqr_issued_ops", "tqr_plan_flags"]
PLAN_ROW_SPLIT, PLAN_TREE, PLAN_MULTIPROC, PLAN_IPC, PLAN_NCCL, PLAN_F32 = 1, 2, 4, 8, 16, 32


def _check(st: int, h=None):
    if st != 0:
        raise TqrError(st, lib().tqr_last_error(h).decode(errors="replace"))


def _i32_array(vals):
    if vals is None:
        return None, 0
    arr = (ctypes.c_int32 * len(vals))(*[int(v) for v in vals])
    return arr, len(vals)


_PLAN_DTYPE = {}   # plan handle value -> TQR_F64 / TQR_F32 (argument checking only)
_PLAN_SHAPE = {}   # plan handle value -> (m, n) (argument checking only)


def _check_shape(x, need_rows, need_cols):
    """The library reads / writes need_rows x need_cols elements through the pointer: refuse arrays
    that are smaller (would be an out-of-bounds host or device access)."""
    shp = tuple(x.shape)
    rows = shp[0] if len(shp) >= 1 else 0
    cols = shp[1] if len(shp) >= 2 else 1
    if rows < need_rows or cols < need_cols:
        raise ValueError("array of shape %s is smaller than the plan's %d x %d" % (shp, need_rows, need_cols))


def _ptr_ld(x, rows: int, h=None, need_cols=None):
    """(pointer, leading dimension) of a column-major 2-D torch tensor or numpy array whose element
    type matches the plan's dtype (and, for a known plan, at least m rows and need_cols columns)."""
    want = _PLAN_DTYPE.get(getattr(h, "value", None), None)
    shape = _PLAN_SHAPE.get(getattr(h, "value", None), None)
    if shape is not None:
        _check_shape(x, shape[0], shape[1] if need_cols is None else need_cols)
    try:
        import torch
        if isinstance(x, torch.Tensor):
            tt = {torch.float64: TQR_F64, torch.float32: TQR_F32}.get(x.dtype)
            if tt is None or (want is not None and tt != want):
                raise TypeError("tensor dtype %s does not match the plan (float64 for TQR_F64, float32 for TQR_F32)"
                                % x.dtype)
            if x.dim() == 1:
                return x.data_ptr(), max(rows, x.shape[0])
            if x.stride(0) != 1:
                raise ValueError("tensor must be column-major (stride(0) == 1); use t().contiguous().t()")
            return x.data_ptr(), max(x.stride(1), rows) if x.shape[1] > 1 else max(rows, x.shape[0])
    except ImportError:  # pragma: no cover
        pass
    import numpy as np
    if isinstance(x, np.ndarray):
        tt = {np.dtype(np.float64): TQR_F64, np.dtype(np.float32): TQR_F32}.get(x.dtype)
        if tt is None or (want is not None and tt != want):
            raise TypeError("array dtype %s does not match the plan" % x.dtype)
        if x.ndim == 1:
            return x.ctypes.data, max(rows, x.shape[0])
        if not x.flags.f_contiguous:
            raise ValueError("numpy array must be Fortran (column-major) ordered")
        return x.ctypes.data, x.shape[0]
    raise TypeError("expected a torch tensor or numpy array")


# ------------------------------------------------------------------ ABI-named functions
def tqr_create(m, n, nb, ib, dtype=TQR_F64, ndev=1, guide=None, logical_devices=False, rank=0, world=1,
               nccl_id=None, lookahead=True, profile=False, tree_domain=0, tree_group=0, row_split=0,
               transport="auto"):
    g, glen = _i32_array(guide)
    opt = Options(int(bool(logical_devices)), int(rank), int(world), None, int(not lookahead), int(bool(profile)),
                  int(tree_domain), int(tree_group), int(row_split), int(TRANSPORT[transport]))
    idbuf = None
    if nccl_id is not None:
        idbuf = ctypes.create_string_buffer(bytes(nccl_id), 128)
        opt.nccl_id = ctypes.cast(idbuf, ctypes.c_void_p)
    h = ctypes.c_void_p()
    st = lib().tqr_create_ex(int(m), int(n), int(nb), int(ib), int(dtype), int(ndev), g, glen, ctypes.byref(opt),
                             ctypes.byref(h))
    _check(st, None)
    _PLAN_DTYPE[h.value] = int(dtype)
    _PLAN_SHAPE[h.value] = (int(m), int(n))
    return h


def tqr_factor(h, A):
    ptr, ld = _ptr_ld(A, 0, h)
    _check(lib().tqr_factor(h, ptr, ld), h)


def tqr_load(h, A):
    ptr, ld = _ptr_ld(A, 0, h)
    _check(lib().tqr_load(h, ptr, ld), h)


def tqr_factor_tiles(h):
    _check(lib().tqr_factor_tiles(h), h)


def tqr_store_r(h, A):
    ptr, ld = _ptr_ld(A, 0, h)
    _check(lib().tqr_store_r(h, ptr, ld), h)


def tqr_apply_qt(h, B, trans="T"):
    nrhs = 1 if len(B.shape) == 1 else B.shape[1]
    ptr, ld = _ptr_ld(B, B.shape[0], h, need_cols=nrhs)
    _check(lib().tqr_apply_qt(h, trans.encode()[:1], ptr, ld, nrhs), h)


def tqr_solve_ls(h, B):
    nrhs = 1 if len(B.shape) == 1 else B.shape[1]
    ptr, ld = _ptr_ld(B, B.shape[0], h, need_cols=nrhs)
    _check(lib().tqr_solve_ls(h, ptr, ld, nrhs), h)


def tqr_destroy(h):
    if h:
        _PLAN_DTYPE.pop(h.value, None)
        _PLAN_SHAPE.pop(h.value, None)
        lib().tqr_destroy(h)


def tqr_nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(lib().tqr_nccl_unique_id(buf), None)
    return buf.raw


def tqr_ipc_handle(h) -> bytes:
    """This rank's CUDA-IPC export blob (IPC transport, multi-process)."""
    ln = ctypes.c_int64()
    _check(lib().tqr_ipc_handle(h, None, 0, ctypes.byref(ln)), h)
    buf = ctypes.create_string_buffer(ln.value)
    _check(lib().tqr_ipc_handle(h, buf, ln.value, ctypes.byref(ln)), h)
    return buf.raw


def tqr_ipc_connect(h, blobs):
    """Open every rank's export (blobs: list of bytes in rank order)."""
    allb = b"".join(bytes(b) for b in blobs)
    buf = ctypes.create_string_buffer(allb, len(allb))
    _check(lib().tqr_ipc_connect(h, buf, len(allb)), h)


def tqr_issued_ops(h):
    cnt = ctypes.c_int64()
    _check(lib().tqr_issued_ops(h, None, 0, ctypes.byref(cnt)), h)
    buf = (ctypes.c_int32 * max(1, 5 * cnt.value))()
    _check(lib().tqr_issued_ops(h, buf, cnt.value, ctypes.byref(cnt)), h)
    return [tuple(buf[5 * i: 5 * i + 5]) for i in range(cnt.value)]


def tqr_owner(h, j):
    return int(lib().tqr_owner(h, int(j)))


def tqr_schedule(m, n, nb, ndev, guide, rank):
    g, glen = _i32_array(guide)
    cnt = ctypes.c_int64()
    _check(lib().tqr_schedule(m, n, nb, ndev, g, glen, rank, None, 0, ctypes.byref(cnt)), None)
    buf = (ctypes.c_int32 * (5 * cnt.value))()
    _check(lib().tqr_schedule(m, n, nb, ndev, g, glen, rank, buf, cnt.value, ctypes.byref(cnt)), None)
    return [tuple(buf[5 * i: 5 * i + 5]) for i in range(cnt.value)]


def _times(times):
    arr = (TileTimes * len(times))()
    for i, t in enumerate(times):
        arr[i] = TileTimes(*[float(x) for x in t])
    return arr


def tqr_row_split_ranges(m, nb, ndev):
    """Row blocks of a row-split plan: [(r0, rows)] per owner."""
    r0 = (ctypes.c_int64 * ndev)()
    rows = (ctypes.c_int64 * ndev)()
    _check(lib().tqr_row_split_ranges(m, nb, ndev, r0, rows), None)
    return list(zip(r0, rows))


def tqr_select_main(times):
    """Algorithm 2: times = [(t_T, t_E, t_UT, t_UE), ...] per device -> main device id."""
    out = ctypes.c_int32()
    _check(lib().tqr_select_main(len(times), _times(times), ctypes.byref(out)), None)
    return out.value


def tqr_select_ndev(M, N, T, elem_size, times, speed, main_dev):
    """Algorithm 3 + Eqs. (10)-(11): -> (order, [T(p) for p = 1..ndev], p_best)."""
    nd = len(times)
    sp = (ctypes.c_double * (nd * nd))(*[float(speed[x][y]) if x != y else 0.0 for x in range(nd) for y in range(nd)])
    order = (ctypes.c_int32 * nd)()
    tp = (ctypes.c_double * nd)()
    pb = ctypes.c_int32()
    _check(lib().tqr_select_ndev(M, N, T, elem_size, nd, _times(times), sp, main_dev, order, tp, ctypes.byref(pb)),
           None)
    return list(order), list(tp), pb.value


def tqr_generate_guide(rates):
    r, nd = _i32_array(rates)
    ln = ctypes.c_int32()
    _check(lib().tqr_generate_guide(r, nd, None, 0, ctypes.byref(ln)), None)
    out = (ctypes.c_int32 * ln.value)()
    _check(lib().tqr_generate_guide(r, nd, out, ln.value, ctypes.byref(ln)), None)
    return list(out)


def tqr_kernel_stats(h, which, reset=False):
    c, ms, fl = ctypes.c_int64(), ctypes.c_double(), ctypes.c_double()
    _check(lib().tqr_kernel_stats(h, int(which), ctypes.byref(c), ctypes.byref(ms), ctypes.byref(fl), int(reset)), h)
    return c.value, ms.value, fl.value


def tqr_launch_count(h):
    return int(lib().tqr_launch_count(h))


class Plan:
    """RAII wrapper: ``with Plan(m, n, nb, ib) as p: p.factor(A)``."""

    def __init__(self, m, n, nb, ib, dtype=TQR_F64, ndev=1, guide=None, **kw):
        self.m, self.n, self.nb, self.ib = m, n, nb, ib
        self.h = tqr_create(m, n, nb, ib, dtype, ndev, guide, **kw)

    def factor(self, A):
        tqr_factor(self.h, A)

    def load(self, A):
        tqr_load(self.h, A)

    def factor_tiles(self):
        tqr_factor_tiles(self.h)

    def store_r(self, A):
        tqr_store_r(self.h, A)

    def apply_qt(self, B, trans="T"):
        tqr_apply_qt(self.h, B, trans)

    def solve_ls(self, B):
        tqr_solve_ls(self.h, B)

    def owner(self, j):
        return tqr_owner(self.h, j)

    def ipc_handle(self):
        return tqr_ipc_handle(self.h)

    def ipc_connect(self, blobs):
        tqr_ipc_connect(self.h, blobs)

    def connect(self, group=None):
        """IPC transport: exchange the export blobs over torch.distributed (all_gather_object on
        `group`) and connect.  Host-side handshake only; no data moves."""
        import torch.distributed as dist
        blobs = [None] * dist.get_world_size(group)
        dist.all_gather_object(blobs, self.ipc_handle(), group=group)
        self.ipc_connect(blobs)

    def issued_ops(self):
        return tqr_issued_ops(self.h)

    def flags(self):
        """TQR_PLAN_* bit mask (row split, tree, multi-process, transport, FP32)."""
        return int(lib().tqr_plan_flags(self.h))

    def kernel_stats(self, which, reset=False):
        return tqr_kernel_stats(self.h, which, reset)

    def launch_count(self):
        return tqr_launch_count(self.h)

    def close(self):
        if self.h:
            tqr_destroy(self.h)
            self.h = None

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def flops(m: int, n: int) -> float:
    """Algorithmic flop count of Householder QR, 2mn^2 - 2n^3/3 (BASELINE.json metric)."""
    return 2.0 * m * n * n - 2.0 * n ** 3 / 3.0
