"""oracle.device_select -- TEST INFRASTRUCTURE ONLY.

Main computing device selection (Algorithm 2) and the number-of-devices selection (Algorithm 3
with the cost model of Eqs. 10-11) of Kim & Park (ICPP'13), written out step by step in the
paper's order and notation.  Only tests/ import this.

Readings (Q22-Q25; the paper gives no worked example for these, so the model is
"parity unpinned" against the paper -- it is pinned by hand-computed closed forms in the tests):

* Q22 Alg. 2: ``can_finish_T_before_UE(i)``: time_i(T) <= time_j(UE) for every other device j;
  ``can_finish_E_before_UT(i)``: time_i(E) <= time_j(UT) for every other device j.  Among the
  candidates the one with the minimum update speed (speed = 1 / (time(UT) + time(UE))) is the
  main device, lowest ID on ties; no candidate -> the fastest updater (lowest ID on ties).
* Q23 Eq. 10, first iteration of an M x N tile grid: #tile_m = M (T and E of the first column on
  the main device, the paper's per-tile accounting of Table I); #tile(i) = M x the number of the
  trailing columns j = 1..N-1 with distribute(j) = i (Eq. 12 over the guide array of Alg. 4
  built for the first p devices of the list); each update tile costs time_i(UT) + time_i(UE).
* Q24 Eq. 11: sum over i = 1..p of 3 M T^2 size / speed(m, i) (reading Q15: speed(m, i); the
  printed speed(m, p) / speed(c, p) are the same quantity with c = m), plus
  (M - 1) T^2 size / speed(j, m) with j = distribute(1), the device of the next column;
  speed(x, x) = infinity (no transfer).
* Q25 Alg. 4 inside Alg. 3: the integer ratio of the p devices' update rates is
  round(speed_i / min speed) (>= 1), then divided by the GCD (GET_RATIO, reading Q14).
"""
from __future__ import annotations

from typing import List, Sequence, Tuple

from .guide import distribute, generate_array, get_ratio


def update_speed(t) -> float:
    """Tiles updated per second: 1 / (time(UT) + time(UE))."""
    return 1.0 / (t[2] + t[3])


def main_selection(times: Sequence[Tuple[float, float, float, float]]) -> int:
    """Algorithm 2.  times[i] = (time_i(T), time_i(E), time_i(UT), time_i(UE))."""
    num_dev = len(times)
    cand = []
    for i in range(num_dev):                                               # line 2
        others = [j for j in range(num_dev) if j != i]
        can_t = all(times[i][0] <= times[j][3] for j in others)            # line 3: T before UE
        can_e = all(times[i][1] <= times[j][2] for j in others)            # line 4: E before UT
        if can_t and can_e:
            cand.append(i)                                                 # line 5
    if not cand:
        best = 0
        for i in range(1, num_dev):
            if update_speed(times[i]) > update_speed(times[best]):
                best = i
        return best
    main = cand[0]                                                         # line 10: minimum speed
    for i in cand[1:]:
        if update_speed(times[i]) < update_speed(times[main]):
            main = i
    return main


def ordered_list(times, main: int) -> List[int]:
    """Alg. 3 lines 2-6: devices by descending update speed (stable), main moved to the head."""
    lst = sorted(range(len(times)), key=lambda i: -update_speed(times[i]))
    lst.remove(main)
    return [main] + lst


def guide_for(times, devs: Sequence[int]) -> List[int]:
    """Alg. 4 over the devices `devs` (positions 0..p-1 of the list); reading Q25."""
    sp = [update_speed(times[d]) for d in devs]
    lo = min(sp)
    rates = [max(1, int(round(s / lo))) for s in sp]
    return generate_array(get_ratio(rates))


def calc_top(M: int, N: int, times, devs: Sequence[int]) -> float:
    """Eq. (10) / CALC_Top: first-iteration operation time on p = len(devs) devices."""
    g = guide_for(times, devs)
    ntile = [0] * len(devs)
    for j in range(1, N):                         # trailing columns of the first iteration
        ntile[distribute(j, g)] += M
    vals = []
    for pos, d in enumerate(devs):
        upd = ntile[pos] * (times[d][2] + times[d][3])
        if pos == 0:                              # the main computing device: T + E as well
            vals.append(M * (times[d][0] + times[d][1]) + upd)
        else:
            vals.append(upd)
    return max(vals)


def calc_tcomm(M: int, N: int, T: int, size: int, times, devs: Sequence[int], speed) -> float:
    """Eq. (11) / CALC_Tcomm.  speed[x][y] = bytes/s from x to y."""
    m = devs[0]
    inv = lambda x, y: 0.0 if x == y else 1.0 / speed[x][y]
    t = 0.0
    for d in devs:                                # sum over i = 1..p (reading Q24)
        t += 3.0 * M * T * T * size * inv(m, d)
    if N > 1:
        j = devs[distribute(1, guide_for(times, devs))]
        t += (M - 1) * T * T * size * inv(j, m)
    return t


def num_dev_selection(M: int, N: int, T: int, size: int, times, speed, main: int):
    """Algorithm 3: returns (ordered list, [T(p) for p = 1..N_dev], p_min)."""
    lst = ordered_list(times, main)
    Tp = []
    pmin, tmin = 0, float("inf")                  # T(0) <- inf, pmin <- 0
    for p in range(1, len(lst) + 1):
        devs = lst[:p]
        t = calc_top(M, N, times, devs) + calc_tcomm(M, N, T, size, times, devs, speed)
        Tp.append(t)
        if t < tmin:
            pmin, tmin = p, t
    return lst, Tp, pmin
