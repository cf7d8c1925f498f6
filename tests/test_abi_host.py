"""CPU-only checks of the C-ABI library: it loads, exports every symbol include/tqr.h
declares, and its pure host logic (guide array, schedule, argument validation) is right.
No compute calls are made here (no GPU in this container)."""
import ctypes
import os
import re

import numpy as np
import pytest

import oracle
import paper_conf_icpp_kimp13_b200 as tqr

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    from paper_conf_icpp_kimp13_b200 import build
    build.build()
    return tqr.lib()


def header_symbols():
    src = open(os.path.join(ROOT, "include", "tqr.h")).read()
    decl = r"^(?:tqr_status|const char\*|int32_t|int64_t)\s+(tqr_[a-z0-9_]+)\s*\("
    return sorted(set(re.findall(decl, src, flags=re.M)))


def test_header_symbols_exported(L):
    syms = header_symbols()
    assert "tqr_create" in syms and "tqr_solve_ls" in syms
    for s in syms:
        assert hasattr(L, s), s
    assert sorted(syms) == sorted(tqr.EXPORTED)


def test_status_strings(L):
    for code in range(8):
        assert L.tqr_status_string(code).decode().startswith(tqr.STATUS[code])


def test_generate_guide_matches_oracle_and_paper(L):
    assert tqr.tqr_generate_guide([8, 12, 4]) == [1, 0, 1, 0, 1, 2]
    rng = np.random.default_rng(1)
    for _ in range(100):
        rates = [int(x) for x in rng.integers(1, 9, size=int(rng.integers(1, 9)))]
        assert tqr.tqr_generate_guide(rates) == oracle.guide.generate_array(oracle.guide.get_ratio(rates))


def _expected_schedule(q, guide, rank):
    own = [oracle.guide.distribute(j, guide) for j in range(q)]
    out = []
    for k in range(q):
        if own[k] == rank:
            out.append((0, k, k, k, own[k]))
        out.append((1, k, k, k, own[k]))
        out += [(2, k, k, j, own[k]) for j in range(k + 1, q) if own[j] == rank]
    return out


@pytest.mark.parametrize("guide,ndev", [([0, 1], 2), ([1, 0, 1, 0, 1, 2], 3), ([0], 1), ([3, 2, 1, 0], 4)])
def test_schedule_covers_dag(L, guide, ndev):
    m, n, nb = 1024, 768, 64
    q = n // nb
    per_rank = [tqr.tqr_schedule(m, n, nb, ndev, guide, r) for r in range(ndev)]
    for r in range(ndev):
        assert per_rank[r] == _expected_schedule(q, guide, r)
    # union: every panel once, every update (k, j>k) exactly once, on the owner of j (Eq. 12)
    panels = [op for ops in per_rank for op in ops if op[0] == 0]
    assert sorted(op[1] for op in panels) == list(range(q))
    ups = sorted((op[1], op[3]) for ops in per_rank for op in ops if op[0] == 2)
    assert ups == [(k, j) for k in range(q) for j in range(k + 1, q)]
    # Table I (TS reading, Q6): per step k, 1 GEQRT, p-k-1 TSQRT, q-k-1 UNMQR, (p-k-1)(q-k-1) TSMQR
    p = m // nb
    for k in range(q):
        n_up = sum(1 for (kk, j) in ups if kk == k)
        assert n_up == q - k - 1
        assert (p - k - 1) * n_up == (p - k - 1) * (q - k - 1)


def test_schedule_ragged_sizes(L):
    """m, n not multiples of nb: zero-padded to whole tiles, q = ceil(n / nb) column tiles."""
    for (m, n, nb) in [(100, 64, 64), (300, 200, 64), (1000, 777, 256), (65, 65, 64)]:
        q = -(-n // nb)
        assert tqr.tqr_schedule(m, n, nb, 1, None, 0) == _expected_schedule(q, [0], 0)


def test_schedule_rejects_bad_args(L):
    with pytest.raises(tqr.TqrError):
        tqr.tqr_schedule(64, 100, 64, 1, None, 0)      # m < n
    with pytest.raises(tqr.TqrError):
        tqr.tqr_schedule(128, 128, 64, 2, [0, 5], 0)


def test_create_without_gpu_fails_cleanly(L):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    with pytest.raises(tqr.TqrError) as e:
        tqr.Plan(128, 128, 64, 16)
    assert e.value.status == 3
    # argument errors are reported before any CUDA call
    with pytest.raises(tqr.TqrError) as e:
        tqr.Plan(64, 128, 64, 16)
    assert e.value.status == 1
    assert L.tqr_destroy(None) == 0


# ---------------------------------------------------------------- Alg. 2 / Alg. 3 + Eqs. 10-11
from oracle import device_select as ds   # noqa: E402


def test_select_main_pins(L):
    """Alg. 2: among the devices that finish T before every other UE and E before
    every other UT, the SLOWEST updater is the main device (the faster ones should update)."""
    times = [(1, 1, 2, 2),     # speed 1/4, candidate
             (1, 1, 1, 1),     # speed 1/2, candidate
             (5, 5, 1, 1)]     # T = 5 > other UEs: not a candidate
    assert tqr.tqr_select_main(times) == 0 == ds.main_selection(times)
    # no candidate at all -> the fastest updater
    times2 = [(9, 9, 3, 3), (9, 9, 1, 2), (9, 9, 2, 2)]
    assert tqr.tqr_select_main(times2) == 1 == ds.main_selection(times2)
    assert tqr.tqr_select_main([(1, 2, 3, 4)]) == 0


def test_select_ndev_closed_form(L):
    """Eq. 10 by hand: 4 identical devices, M = N = 8, (T, E, UT, UE) = (1, 2, 1, 2) s, free links.
    p = 1: M(T+E) + 7 columns x M x (UT+UE) = 24 + 168 = 192.  p = 2 (guide {0,1}): main gets
    columns 2,4,6 -> 24 + 72 = 96, device 1 gets 1,3,5,7 -> 96.  p = 4: main columns 4 -> 24 + 24 =
    48, device 1 columns 1,5 -> 48.  Eq. 11 with 1 GB/s links, 8-byte elements, T = 1 adds
    3 M (p - 1) 8 B / 1e9 + (M - 1) 8 B / 1e9 for p > 1."""
    times = [(1.0, 2.0, 1.0, 2.0)] * 4
    free = [[1e300] * 4 for _ in range(4)]
    order, Tp, pb = tqr.tqr_select_ndev(8, 8, 1, 8, times, free, 0)
    assert order == [0, 1, 2, 3]
    np.testing.assert_allclose(Tp, [192.0, 96.0, 72.0, 48.0], rtol=1e-12)
    assert pb == 4
    slow = [[1e9] * 4 for _ in range(4)]
    _, Tp2, _ = tqr.tqr_select_ndev(8, 8, 1, 8, times, slow, 0)
    comm = [0.0] + [3 * 8 * (p - 1) * 8 / 1e9 + 7 * 8 / 1e9 for p in (2, 3, 4)]
    np.testing.assert_allclose(Tp2, np.array([192.0, 96.0, 72.0, 48.0]) + comm, rtol=1e-12)
    # links slow enough that one device wins
    crawl = [[1.0] * 4 for _ in range(4)]
    assert tqr.tqr_select_ndev(8, 8, 1, 8, times, crawl, 0)[2] == 1


@pytest.mark.parametrize("seed", range(12))
def test_select_matches_oracle(L, seed):
    """Randomised heterogeneous devices: the library's Alg. 2/3 equal the step-by-step oracle."""
    rng = np.random.default_rng(seed)
    nd = int(rng.integers(1, 9))
    times = [tuple(float(x) for x in rng.uniform(1e-4, 5e-3, 4)) for _ in range(nd)]
    speed = rng.uniform(2e10, 9e11, (nd, nd)).tolist()
    M, N, T = int(rng.integers(1, 70)), int(rng.integers(1, 70)), int(rng.choice([64, 256, 512]))
    main = tqr.tqr_select_main(times)
    assert main == ds.main_selection(times)
    order, Tp, pb = tqr.tqr_select_ndev(M, N, T, 8, times, speed, main)
    lo, Tpo, pbo = ds.num_dev_selection(M, N, T, 8, times, speed, main)
    assert order == lo and pb == pbo
    np.testing.assert_allclose(Tp, Tpo, rtol=1e-12)


def test_guide_and_selection_bounded_on_extreme_rates(L):
    """a guide longer than the cap (2^20 entries) is TQR_ERR_ARG, not an overflowed
    length or a huge allocation; the device-count model clamps wildly mismatched rates."""
    with pytest.raises(tqr.TqrError) as e:
        tqr.tqr_generate_guide([2 ** 30, 1])
    assert e.value.status == 1
    assert len(tqr.tqr_generate_guide([2 ** 19, 2 ** 19 + 2])) == 2 ** 18 + 2 ** 18 + 1
    times = [(1e-3, 1e-3, 1e-12, 1e-12), (1e-3, 1e-3, 1e3, 1e3)]     # update speeds 1e15 apart
    order, tp, pb = tqr.tqr_select_ndev(4, 4, 64, 8, times, [[0, 1e9], [1e9, 0]], 0)
    assert pb in (1, 2) and len(tp) == 2 and all(x > 0 for x in tp)


def test_plan_queries_without_gpu(L):
    """The plan-query entry points are NULL-safe (no GPU needed)."""
    assert L.tqr_plan_flags(None) == 0
    assert L.tqr_owner(None, 0) == -1
    cnt = ctypes.c_int64()
    assert L.tqr_issued_ops(None, None, 0, ctypes.byref(cnt)) == 1
    assert L.tqr_ipc_handle(None, None, 0, ctypes.byref(cnt)) == 1
