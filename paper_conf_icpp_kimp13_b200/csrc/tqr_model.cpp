// tqr_model.cpp -- the paper's device selection (NEXT-2 / NEXT-4): main computing
// device selection (Algorithm 2) and the number-of-devices selection (Algorithm 3,
// P:L957-995) with the first-iteration cost model of Eqs. (10)-(11), fed with
// measured per-tile operation times and link speeds (tools/device_select.py measures them on
// B200).  Host-only code; readings Q22-Q25 in DESIGN.md sec. 2.
#include "../../include/tqr.h"

#include <algorithm>
#include <cmath>
#include <limits>
#include <vector>

namespace {

double upd_speed(const tqr_tile_times& t) { return 1.0 / (t.t_UT + t.t_UE); }

bool valid(int32_t ndev, const tqr_tile_times* t) {
    if (ndev < 1 || !t) return false;
    for (int i = 0; i < ndev; ++i)
        if (!(t[i].t_T >= 0 && t[i].t_E >= 0 && t[i].t_UT >= 0 && t[i].t_UE >= 0 && t[i].t_UT + t[i].t_UE > 0))
            return false;
    return true;
}

// Alg. 4 guide array over the devices at list positions 0..p-1 (reading Q25)
std::vector<int32_t> guide_for(const tqr_tile_times* t, const std::vector<int>& devs) {
    double lo = std::numeric_limits<double>::infinity();
    for (int d : devs) lo = std::min(lo, upd_speed(t[d]));
    std::vector<int32_t> rates(devs.size());
    // ratios clamped to [1, 4096] before the rounding cast (no int overflow for wildly mismatched rates)
    for (size_t i = 0; i < devs.size(); ++i)
        rates[i] = (int32_t)std::lround(std::min(4096.0, std::max(1.0, upd_speed(t[devs[i]]) / lo)));
    int32_t len = 0;
    if (tqr_generate_guide(rates.data(), (int32_t)rates.size(), nullptr, 0, &len) != TQR_OK) return {};
    std::vector<int32_t> g(len);
    tqr_generate_guide(rates.data(), (int32_t)rates.size(), g.data(), len, &len);
    return g;
}

}  // namespace

extern "C" {

tqr_status tqr_select_main(int32_t ndev, const tqr_tile_times* t, int32_t* main_dev) {
    if (!valid(ndev, t) || !main_dev) return TQR_ERR_ARG;
    int best = -1;
    for (int i = 0; i < ndev; ++i) {
        bool can_t = true, can_e = true;   // T before every other UE, E before every other UT
        for (int j = 0; j < ndev; ++j) {
            if (j == i) continue;
            if (t[i].t_T > t[j].t_UE) can_t = false;
            if (t[i].t_E > t[j].t_UT) can_e = false;
        }
        if (can_t && can_e && (best < 0 || upd_speed(t[i]) < upd_speed(t[best]))) best = i;
    }
    if (best < 0) {   // no candidate: the fastest updater
        best = 0;
        for (int i = 1; i < ndev; ++i)
            if (upd_speed(t[i]) > upd_speed(t[best])) best = i;
    }
    *main_dev = best;
    return TQR_OK;
}

tqr_status tqr_select_ndev(int32_t M, int32_t N, int32_t T, int32_t elem_size, int32_t ndev,
                           const tqr_tile_times* t, const double* speed, int32_t main_dev, int32_t* order,
                           double* Tp, int32_t* pbest) {
    if (M < 1 || N < 1 || T < 1 || elem_size < 1 || !valid(ndev, t) || !speed || main_dev < 0 ||
        main_dev >= ndev || !pbest)
        return TQR_ERR_ARG;
    for (int x = 0; x < ndev; ++x)
        for (int y = 0; y < ndev; ++y)
            if (x != y && !(speed[x * ndev + y] > 0)) return TQR_ERR_ARG;
    // Alg. 3 lines 2-6: descending update speed (stable by ID), main device at the head
    std::vector<int> lst(ndev);
    for (int i = 0; i < ndev; ++i) lst[i] = i;
    std::stable_sort(lst.begin(), lst.end(), [&](int a, int b) { return upd_speed(t[a]) > upd_speed(t[b]); });
    lst.erase(std::find(lst.begin(), lst.end(), (int)main_dev));
    lst.insert(lst.begin(), (int)main_dev);
    if (order) std::copy(lst.begin(), lst.end(), order);
    auto inv = [&](int x, int y) { return x == y ? 0.0 : 1.0 / speed[x * ndev + y]; };
    const double tile_bytes = (double)T * T * elem_size;
    double tmin = std::numeric_limits<double>::infinity();
    int pmin = 0;
    for (int p = 1; p <= ndev; ++p) {
        std::vector<int> devs(lst.begin(), lst.begin() + p);
        const std::vector<int32_t> g = guide_for(t, devs);
        if (g.empty()) return TQR_ERR_ARG;
        // Eq. 10: trailing columns j = 1..N-1 by Eq. 12, M update tiles each
        std::vector<double> ntile(p, 0.0);
        for (int j = 1; j < N; ++j) ntile[g[j % g.size()]] += M;
        double top = 0.0;
        for (int pos = 0; pos < p; ++pos) {
            const tqr_tile_times& d = t[devs[pos]];
            double v = ntile[pos] * (d.t_UT + d.t_UE);
            if (pos == 0) v += (double)M * (d.t_T + d.t_E);
            top = std::max(top, v);
        }
        // Eq. 11: 3 M T^2 to every participant, (M-1) T^2 from the next column's device to main
        const int m = devs[0];
        double tc = 0.0;
        for (int d : devs) tc += 3.0 * M * tile_bytes * inv(m, d);
        if (N > 1) tc += (M - 1) * tile_bytes * inv(devs[g[1 % g.size()]], m);
        const double tp = top + tc;
        if (Tp) Tp[p - 1] = tp;
        if (tp < tmin) { tmin = tp; pmin = p; }
    }
    *pbest = pmin;
    return TQR_OK;
}

}  // extern "C"
