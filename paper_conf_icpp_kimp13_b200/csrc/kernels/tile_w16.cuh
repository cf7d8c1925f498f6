// tile_w16.cuh -- bulk trailing update with 16 warps per CTA (4 per scheduler).
//
// Same block-reflector apply as apply_block (tile_ops.cuh, Eq. 9 per ib block: GEMM1 W = X1 +
// V_s^T X, reduction + T multiply, GEMM2 X -= V_s W'), same NB x 32 column slice per CTA, but the
// slice is split over 16 warps: warp (rg, cg) = (wq % 8, wq / 8) holds rows rg*RW.. of the 16
// columns cg*16.. (X: 32 doubles per thread instead of 64), so the CTA fits 512 threads at <= 128
// registers and every SM sub-partition has four warps to issue DMMAs from instead of two.  The two
// warps of a row group share its staged V rows (one cp.async.bulk per half, issued by the cg = 0
// warp; a 64-thread named barrier (id 1 + rg) before each refill), the partials of the two column
// groups go to separate 8-slot sets, and the reduction / T multiply is spread over all 512 threads.
// Measured (one B200, 3 alternating runs each): C5 1602-1608 ms vs 1628-1631 ms with the 8-warp
// kernel, C3 226.2-226.4 vs 228.2-230.4 ms.  Keeping the reduction local to each column group
// (named 256-thread barriers) measured slower (C5 1618 ms): the row-group pair syncs of the shared
// V staging re-align the groups every block anyway.
#pragma once
#include "tile_ops.cuh"

namespace tqr {

constexpr int kThreads16 = 512;
constexpr int kWarps16 = 16;

template <int NB, int IB>
struct Smem16 {
    using G = Geom<NB, 32, IB>;              // RW = NB/8 rows per row group, HC, LDR, LDW, LDT2
    uint64_t mbar[8][2];                     // [row group][half]
    double Vst[8][2][G::HC][G::RW];          // [row group][half], layout of vst_off
    double red[2 * 8 * 16 * G::LDR];         // [cg][rg][col 0..15][ib] partial slots; the 4 pad doubles
                                             // of each slot column hold -W' (GEMM2 operand), wsm_off
    double Wsm[32 * G::LDW];                 // W (reduce-scatter)
    double Traw[IB * G::LDT2];               // T(r', r) at r*LDT2 + r'
    double topsm[32 * G::LDW];               // X1 rows (r, c) at c*LDW + r
};

template <int NB, int IB>
struct Slice16 {
    using G = Geom<NB, 32, IB>;
    static constexpr int NF = G::NF;         // 8-row fragments of the row group
    double acc[2][NF][2];                    // (row rg*RW + nf*8 + 2t + e, col cg*16 + mf*8 + g)
    __device__ __forceinline__ int r0() const { return (warp_id() & 7) * G::RW + 2 * (lane_id() & 3); }
    __device__ __forceinline__ int c0() const { return (warp_id() >> 3) * 16 + (lane_id() >> 2); }
    __device__ __forceinline__ void load(const double* P, int64_t ld) {
#pragma unroll
        for (int mf = 0; mf < 2; ++mf)
#pragma unroll
            for (int nf = 0; nf < NF; ++nf) {
                const double2 v = ld2(P + (int64_t)(c0() + mf * 8) * ld + r0() + nf * 8);
                acc[mf][nf][0] = v.x;
                acc[mf][nf][1] = v.y;
            }
    }
    __device__ __forceinline__ void load_cg(const double* P, int64_t ld) {
#pragma unroll
        for (int mf = 0; mf < 2; ++mf)
#pragma unroll
            for (int nf = 0; nf < NF; ++nf) {
                const double2 v = ld2_cg(P + (int64_t)(c0() + mf * 8) * ld + r0() + nf * 8);
                acc[mf][nf][0] = v.x;
                acc[mf][nf][1] = v.y;
            }
    }
    __device__ __forceinline__ void store(double* P, int64_t ld) const {
#pragma unroll
        for (int mf = 0; mf < 2; ++mf)
#pragma unroll
            for (int nf = 0; nf < NF; ++nf)
                st2(P + (int64_t)(c0() + mf * 8) * ld + r0() + nf * 8, acc[mf][nf][0], acc[mf][nf][1]);
    }
};

// -W'(col, r) in the padding of the partial slots (ib 32..35 of slot (col / 16, r / 4), column
// col % 16): no partial store ever writes there, so the next block's GEMM1 stores cannot race with
// a slower warp's GEMM2 reads, and the T multiply can write it without a barrier after its reads
// of Wsm.  Lanes (g, t) of an A-fragment load hit banks (4g + t) mod 16: two wavefronts.
template <int LDR>
__device__ __forceinline__ int wsm_off(int col, int r) {
    return ((col >> 4) * 8 + (r >> 2)) * (16 * LDR) + (col & 15) * LDR + (LDR - 4) + (r & 3);
}

__device__ __forceinline__ void pair_sync(int rg) {   // the two warps of row group rg
    asm volatile("bar.sync %0, 64;" ::"r"(1 + rg) : "memory");
}

// half h of block image `blk` for row group rg (issued by the cg = 0 warp once both warps of the
// group finished reading the buffer: the caller pair_syncs first)
template <int NB, int IB>
__device__ __forceinline__ void stage16(Smem16<NB, IB>& sm, const double* blk, int h) {
    using G = Geom<NB, 32, IB>;
    const int wq = warp_id(), rg = wq & 7;
    if (wq < 8 && lane_id() == 0) {
        fence_proxy_async_shared();
        bulk_g2s(&sm.Vst[rg][h][0][0], blk + (rg * 2 + h) * (G::HC * G::RW), G::HC * G::RW * 8, &sm.mbar[rg][h]);
    }
}

// One ib block, Q^T (TRANS) form only.  Entry: half A of Vs in flight (or staged); Exit: half A of
// `next` in flight.
template <int NB, int IB, bool KM>
__device__ __forceinline__ void apply_block16(Slice16<NB, IB>& X, Smem16<NB, IB>& sm, const double* __restrict__ Vs,
                                              const double* __restrict__ Ts, double* top, int64_t ldtop, int kmin,
                                              const double* next, unsigned& vph) {
    using G = Geom<NB, 32, IB>;
    constexpr int NF = G::NF, JC = G::JC, HC = G::HC;
    const int lane = lane_id(), g = lane >> 2, t = lane & 3, wq = warp_id(), tid = threadIdx.x;
    const int rg = wq & 7, cg = wq >> 3, tg = tid & 255;
    const int rbase = rg * G::RW;

    // ---- (0) half B of V (both warps of the row group are done with the previous block's half B),
    //      T block and X1 rows (each column group loads its X1 columns)
    pair_sync(rg);
    stage16(sm, Vs, 1);
    for (int id = tid; id < IB * IB / 2; id += kThreads16) {
        const int c = id / (IB / 2), r2 = id % (IB / 2);
        cp_async16<false>(&sm.Traw[c * G::LDT2 + 2 * r2], Ts + c * IB + 2 * r2);
    }
    if (top)
        for (int id = tg; id < 16 * IB / 2; id += 256) {
            const int c = cg * 16 + id / (IB / 2), r2 = id % (IB / 2);
            cp_async16<true>(&sm.topsm[c * G::LDW + 2 * r2], top + (int64_t)c * ldtop + 2 * r2);
        }
    cp_async_commit();

    // ---- (1) GEMM1: partial W^T(col, ib) over the group's rows -> slot (cg, rg)
    double* slot = sm.red + (cg * 8 + rg) * (16 * G::LDR);
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        mbar_wait(&sm.mbar[rg][h], (vph >> h) & 1u);
        vph ^= 1u << h;
        const double* vh = &sm.Vst[rg][h][0][0];
        double c1[2][JC][2];
#pragma unroll
        for (int mf = 0; mf < 2; ++mf)
#pragma unroll
            for (int j = 0; j < JC; ++j) c1[mf][j][0] = c1[mf][j][1] = 0.0;
#pragma unroll
        for (int nf = 0; nf < NF; ++nf) {
            if (KM && rbase + nf * 8 + 8 <= kmin) continue;
            double2 b[JC];
#pragma unroll
            for (int j = 0; j < JC; ++j)
                b[j] = *reinterpret_cast<const double2*>(vh + vst_off<NB, 32, IB>(nf * 8 + 2 * t, j * 8 + g));
#pragma unroll
            for (int mf = 0; mf < 2; ++mf)
#pragma unroll
                for (int j = 0; j < JC; ++j) dmma(c1[mf][j][0], c1[mf][j][1], X.acc[mf][nf][0], b[j].x);
#pragma unroll
            for (int mf = 0; mf < 2; ++mf)
#pragma unroll
                for (int j = 0; j < JC; ++j) dmma(c1[mf][j][0], c1[mf][j][1], X.acc[mf][nf][1], b[j].y);
        }
#pragma unroll
        for (int mf = 0; mf < 2; ++mf)
#pragma unroll
            for (int j = 0; j < JC; ++j)
                st2(slot + (mf * 8 + g) * G::LDR + h * HC + j * 8 + 2 * t, c1[mf][j][0], c1[mf][j][1]);
    }
    cp_async_wait<0>();
    __syncthreads();
    // ---- (2) reduce-scatter: W(col, ib) = X1 + sum of the column group's 8 slots -> Wsm
    for (int idx = tg; idx < 16 * IB / 2; idx += 256) {
        const int cl = idx / (IB / 2), ib = 2 * (idx % (IB / 2));
        const int c = cg, col = cg * 16 + cl;
        double2 sv = top ? ld2(&sm.topsm[col * G::LDW + ib]) : make_double2(0.0, 0.0);
#pragma unroll
        for (int r = 0; r < 8; ++r) {
            const double2 pv = ld2(&sm.red[(c * 8 + r) * (16 * G::LDR) + cl * G::LDR + ib]);
            sv.x += pv.x;
            sv.y += pv.y;
        }
        st2(&sm.Wsm[col * G::LDW + ib], sv.x, sv.y);
    }
    __syncthreads();
    // ---- (3) T multiply W'^T = W^T T (T upper triangular), the group's 2*IB/8 fragments one per warp
    constexpr int NFRAG = 2 * (IB / 8);
    const int wl = wq & 7;
    const int fmf = cg * 2 + wl / (IB / 8), fjf = wl % (IB / 8);
    double w0 = 0.0, w1 = 0.0, v0 = 0.0, v1 = 0.0;
    if (wl < NFRAG) {
#pragma unroll
        for (int kk = 0; kk < IB; kk += 4) {
            if (kk >= fjf * 8 + 8) continue;   // warp-uniform: exact zeros of T
            const double av = sm.Wsm[(fmf * 8 + g) * G::LDW + kk + t];
            const double bv = sm.Traw[(fjf * 8 + g) * G::LDT2 + kk + t];
            if ((kk >> 2) & 1) dmma(v0, v1, av, bv);
            else               dmma(w0, w1, av, bv);
        }
    }
    if (wl < NFRAG) {
        const int col = fmf * 8 + g, r = fjf * 8 + 2 * t;
        const double a0 = w0 + v0, a1 = w1 + v1;
        st2(&sm.red[wsm_off<G::LDR>(col, r)], -a0, -a1);   // r even: r, r+1 in one 16-byte pair
        if (top) st2(top + (int64_t)col * ldtop + r, sm.topsm[col * G::LDW + r] - a0, sm.topsm[col * G::LDW + r + 1] - a1);
    }
    __syncthreads();
    // ---- (4) GEMM2: X^T(col, row) += (-W'^T)(col, ib) V^T(ib, row); half A of `next` after half A
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        if (h == 1 && next != nullptr) {
            pair_sync(rg);
            stage16(sm, next, 0);
        }
        const double* vh = &sm.Vst[rg][h][0][0];
#pragma unroll
        for (int kk = 0; kk < HC; kk += 4) {
            double a[2];
#pragma unroll
            for (int mf = 0; mf < 2; ++mf) a[mf] = sm.red[wsm_off<G::LDR>(cg * 16 + mf * 8 + g, h * HC + kk + t)];
#pragma unroll
            for (int nf = 0; nf < NF; ++nf) {
                if (KM && rbase + nf * 8 + 8 <= kmin) continue;
                const double b = vh[vst_off<NB, 32, IB>(nf * 8 + g, kk + t)];
#pragma unroll
                for (int mf = 0; mf < 2; ++mf) dmma(X.acc[mf][nf][0], X.acc[mf][nf][1], a[mf], b);
            }
        }
    }
}

}  // namespace tqr
