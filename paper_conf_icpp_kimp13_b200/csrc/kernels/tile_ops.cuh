// tile_ops.cuh -- register-resident block-reflector apply and ib-panel factorisation.
//
// The method's tile operations (Sec. II.B), with the PLASMA/LAPACK
// storage of reading Q8 (V in place, T as ib x nb per tile):
//   GEQRT  A_kk = Q_kk R_kk                         Eqs. (4)-(5)
//   UNMQR  A_kj <- Q_kk^T A_kj                      Eq. (6),  P:L268-274 (reading Q5: Q^T)
//   TSQRT  [R_kk; A_ik] = Q_ik [R_kk'; 0]           Eqs. (7)-(8)
//   TSMQR  [A_kj; A_ij] <- Q_ik^T [A_kj; A_ij]      Eq. (9),
// Every one of them is built from two primitives operating on a CTA-resident NB x W slice X
// (see common.cuh for the register layout):
//   apply_block : X <- (I - V_s T_s^T V_s^T) X for one ib-wide block s of reflectors, with an
//                 optional "top" row block X1 (the R / A_kj rows of a TS pair):
//                   W  = X1 + V_s^T X            (GEMM1, K = NB rows, DMMA)
//                   W  = T_s^T W                 (ib x ib triangular, SIMT in smem)
//                   X1 -= W ;  X -= V_s W       (GEMM2, K = ib, DMMA)
//   factor_block: Householder reflectors of ib consecutive columns (dlarfg convention,
//                 beta = -sgn(x0) ||x||, reading Q1/Q4), warp-shuffle + smem reductions,
//                 then the compact-WY T_s by the forward dlarft recurrence
//                 T(0:c, c) = -tau_c T(0:c, 0:c) (V(:, 0:c)^T v_c), Gram matrix on DMMA.
#pragma once
#include "common.cuh"

namespace tqr {

constexpr int kThreads = 256;
constexpr int kWarps = 8;

template <int NB, int W, int IB>
struct Geom {
    static constexpr int RW = NB / kWarps;   // rows per warp
    static constexpr int NF = RW / 8;        // 8-row fragments per warp
    static constexpr int MF = W / 8;         // 8-column fragments
    static constexpr int JF = IB / 8;        // 8-wide ib fragments
    static constexpr int JC = (JF < 2) ? JF : 2;  // ib fragments per GEMM1 pass (register budget)
    static constexpr int LDR = IB + 8;       // red[w][col][ib]   (== 8 mod 16: conflict-free v2 stores)
    static constexpr int LDW = IB + 4;       // Wsm[col][ib]      (== 4 mod 16: conflict-free A-frag loads)
    static constexpr int LDT = IB;           // Tsm[r'][r]
    static_assert(NB % 64 == 0 && W % 8 == 0 && IB % 8 == 0 && NB % IB == 0, "tile geometry");
    static_assert(IB % (8 * JC) == 0, "ib chunking");
};

// Shared-memory workspace of one CTA (apply + factor).  Placed in dynamic smem.
template <int NB, int W, int IB>
struct Smem {
    using G = Geom<NB, W, IB>;
    double red[kWarps * W * G::LDR];   // per-warp GEMM partials
    double Wsm[W * G::LDW];            // -T^T W  (A operand of GEMM2), element (ib, col) at col*LDW + ib
    double Tsm[IB * G::LDT];           // T block, element used as Tsm[r'*LDT + r]
    double Rsm[IB * IB];               // TSQRT diagonal R block (row c, col j) at c*IB + j
    double tau[IB];
    double wvec[IB];
    double red1[kWarps];
    double x0;
};

// ---------------------------------------------------------------- register slice I/O
template <int NB, int W, int IB>
struct Slice {
    using G = Geom<NB, W, IB>;
    double acc[G::MF][G::NF][2];

    // element (r, c) of the slice at P[c*ld + r]
    __device__ __forceinline__ void load(const double* P, int64_t ld) {
        const int g = lane_id() >> 2, t = lane_id() & 3, r0 = warp_id() * G::RW + 2 * t;
#pragma unroll
        for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
            for (int nf = 0; nf < G::NF; ++nf) {
                double2 v = ld2(P + (int64_t)(mf * 8 + g) * ld + r0 + nf * 8);
                acc[mf][nf][0] = v.x;
                acc[mf][nf][1] = v.y;
            }
    }
    __device__ __forceinline__ void load_cg(const double* P, int64_t ld) {
        const int g = lane_id() >> 2, t = lane_id() & 3, r0 = warp_id() * G::RW + 2 * t;
#pragma unroll
        for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
            for (int nf = 0; nf < G::NF; ++nf) {
                double2 v = ld2_cg(P + (int64_t)(mf * 8 + g) * ld + r0 + nf * 8);
                acc[mf][nf][0] = v.x;
                acc[mf][nf][1] = v.y;
            }
    }
    __device__ __forceinline__ void store(double* P, int64_t ld) const {
        const int g = lane_id() >> 2, t = lane_id() & 3, r0 = warp_id() * G::RW + 2 * t;
#pragma unroll
        for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
            for (int nf = 0; nf < G::NF; ++nf)
                st2(P + (int64_t)(mf * 8 + g) * ld + r0 + nf * 8, acc[mf][nf][0], acc[mf][nf][1]);
    }
};

// V loads: the panel kernel reads V published by sibling CTAs of the same grid -> L2 (.cg);
// the update kernel reads V that is immutable during the launch -> read-only path (.nc).
template <bool CG>
__device__ __forceinline__ double2 vld2(const double* p) {
    if constexpr (CG) return ld2_cg(p); else return __ldg(reinterpret_cast<const double2*>(p));
}
template <bool CG>
__device__ __forceinline__ double vld(const double* p) {
    if constexpr (CG) return ld_cg(p); else return __ldg(p);
}

// ---------------------------------------------------------------- apply one ib block
// X (registers, NB x W) <- H_s X where H_s = I - V_s T_s^T V_s^T (TRANS) or I - V_s T_s V_s^T.
//   Vs   : column s*IB of V (NB x IB, ld = ldv); rows < kmin are zero (their DMMAs skipped).
//   Ts   : T block s (IB x IB column-major, ld = IB) = T_tile + s*IB*IB.
//   top  : if non-null, the X1 rows (IB x W, element (r, c) at top[c*ldtop + r]).
// Latency hiding (8 warps/SM only, 254 registers): every global operand is loaded one step
// ahead of its use -- GEMM1's V fragments one row-fragment ahead, GEMM2's first fragments and
// the top rows / T block before the reduction barriers, GEMM2's next k-step during the current.
template <int NB, int W, int IB, bool TRANS, bool CG>
__device__ __forceinline__ void apply_block(Slice<NB, W, IB>& X, Smem<NB, W, IB>& sm,
                                            const double* __restrict__ Vs, int64_t ldv,
                                            const double* __restrict__ Ts,
                                            double* top, int64_t ldtop, int kmin) {
    using G = Geom<NB, W, IB>;
    constexpr int NR = (W * IB + kThreads - 1) / kThreads;     // reduce outputs per thread
    constexpr int NT = (IB * IB + kThreads - 1) / kThreads;    // T entries per thread
    const int lane = lane_id(), g = lane >> 2, t = lane & 3, wq = warp_id();
    const int rbase = wq * G::RW;
    const int tid = threadIdx.x;

    // ---- (0) early loads: top rows and T block (consumed after the first barrier)
    double topv[NR];
#pragma unroll
    for (int r = 0; r < NR; ++r) {
        const int idx = tid + r * kThreads;
        topv[r] = 0.0;
        if (top && idx < W * IB) topv[r] = top[(int64_t)(idx / IB) * ldtop + (idx % IB)];
    }
    double tv[NT];
#pragma unroll
    for (int r = 0; r < NT; ++r) {
        const int idx = tid + r * kThreads;
        tv[r] = 0.0;
        if (idx < IB * IB) {
            const int rp = idx / IB, rr = idx % IB;
            if constexpr (TRANS) { if (rp <= rr) tv[r] = vld<CG>(Ts + rr * IB + rp); }   // T(r', r): W' = T^T W
            else                 { if (rp >= rr) tv[r] = vld<CG>(Ts + rp * IB + rr); }   // T(r, r'): W' = T W
        }
    }

    // ---- (1) GEMM1: partial W^T(col, ib) = sum_{my rows} X(row, col) V(row, ib)
#pragma unroll
    for (int jc = 0; jc < G::JF; jc += G::JC) {
        double c1[G::MF][G::JC][2];
#pragma unroll
        for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
            for (int j = 0; j < G::JC; ++j) c1[mf][j][0] = c1[mf][j][1] = 0.0;
        const double* vb = Vs + (int64_t)(jc * 8 + g) * ldv + rbase + 2 * t;
        double2 bn[G::JC];
#pragma unroll
        for (int j = 0; j < G::JC; ++j) bn[j] = vld2<CG>(vb + (int64_t)j * 8 * ldv);
#pragma unroll
        for (int nf = 0; nf < G::NF; ++nf) {
            double2 b[G::JC];
#pragma unroll
            for (int j = 0; j < G::JC; ++j) b[j] = bn[j];
            if (nf + 1 < G::NF) {
#pragma unroll
                for (int j = 0; j < G::JC; ++j) bn[j] = vld2<CG>(vb + (int64_t)j * 8 * ldv + (nf + 1) * 8);
            }
            if (rbase + nf * 8 + 8 > kmin) {                 // rows < kmin of V are zero
#pragma unroll
                for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
                    for (int j = 0; j < G::JC; ++j) dmma(c1[mf][j][0], c1[mf][j][1], X.acc[mf][nf][0], b[j].x);
#pragma unroll
                for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
                    for (int j = 0; j < G::JC; ++j) dmma(c1[mf][j][0], c1[mf][j][1], X.acc[mf][nf][1], b[j].y);
            }
        }
        // c1[mf][j] = W^T[col mf*8+g][ib (jc+j)*8 + 2t + e]
        double* rw = sm.red + wq * (W * G::LDR);
#pragma unroll
        for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
            for (int j = 0; j < G::JC; ++j)
                st2(rw + (mf * 8 + g) * G::LDR + (jc + j) * 8 + 2 * t, c1[mf][j][0], c1[mf][j][1]);
    }
    // GEMM2's first V fragments, in flight across the reduction barriers
    const double* v2 = Vs + rbase + g + (int64_t)t * ldv;
    double bq[G::NF];
#pragma unroll
    for (int nf = 0; nf < G::NF; ++nf) bq[nf] = vld<CG>(v2 + nf * 8);
#pragma unroll
    for (int r = 0; r < NT; ++r) {
        const int idx = tid + r * kThreads;
        if (idx < IB * IB) sm.Tsm[(idx / IB) * G::LDT + (idx % IB)] = tv[r];
    }
    __syncthreads();
    // ---- (2) reduce the 8 warp partials (+ top) -> red[warp 0 slot]
#pragma unroll
    for (int r = 0; r < NR; ++r) {
        const int idx = tid + r * kThreads;
        if (idx < W * IB) {
            const int col = idx / IB, ib = idx % IB;
            double s = topv[r];
#pragma unroll
            for (int w = 0; w < kWarps; ++w) s += sm.red[w * (W * G::LDR) + col * G::LDR + ib];
            sm.red[col * G::LDR + ib] = s;   // slot 0 entry (col, ib) is read above by this thread only
        }
    }
    __syncthreads();
    // ---- (3) W' = op(T) W;  top -= W';  Wsm = -W'
#pragma unroll
    for (int r = 0; r < NR; ++r) {
        const int idx = tid + r * kThreads;
        if (idx < W * IB) {
            const int col = idx / IB, rr = idx % IB;
            const double* wc = sm.red + col * G::LDR;
            double s = 0.0;
#pragma unroll 8
            for (int rp = 0; rp < IB; ++rp) s += sm.Tsm[rp * G::LDT + rr] * wc[rp];
            if (top) top[(int64_t)col * ldtop + rr] -= s;
            sm.Wsm[col * G::LDW + rr] = -s;
        }
    }
    __syncthreads();
    // ---- (4) GEMM2: X^T(col, row) += (-W'^T)(col, ib) V^T(ib, row), next k-step prefetched
    double a[G::MF];
#pragma unroll
    for (int mf = 0; mf < G::MF; ++mf) a[mf] = sm.Wsm[(mf * 8 + g) * G::LDW + t];
#pragma unroll
    for (int kk = 0; kk < IB; kk += 4) {
        double ac[G::MF], bc[G::NF];
#pragma unroll
        for (int mf = 0; mf < G::MF; ++mf) ac[mf] = a[mf];
#pragma unroll
        for (int nf = 0; nf < G::NF; ++nf) bc[nf] = bq[nf];
        if (kk + 4 < IB) {
#pragma unroll
            for (int mf = 0; mf < G::MF; ++mf) a[mf] = sm.Wsm[(mf * 8 + g) * G::LDW + kk + 4 + t];
#pragma unroll
            for (int nf = 0; nf < G::NF; ++nf) bq[nf] = vld<CG>(v2 + (int64_t)(kk + 4) * ldv + nf * 8);
        }
#pragma unroll
        for (int nf = 0; nf < G::NF; ++nf) {
            if (rbase + nf * 8 + 8 <= kmin) continue;
#pragma unroll
            for (int mf = 0; mf < G::MF; ++mf) dmma(X.acc[mf][nf][0], X.acc[mf][nf][1], ac[mf], bc[nf]);
        }
    }
    // Next call writes red before its first __syncthreads; Wsm/Tsm are rewritten only after
    // that barrier, which every warp reaches after finishing this GEMM2.
}

// ---------------------------------------------------------------- factor ib columns
// X holds W = IB columns.  GEQRT mode (GE=true): column c's diagonal row is d = dbase + c,
// rows < d are R (kept), rows > d become v (unit v_d implied, stored beta at row d).
// TSQRT mode (GE=false): the top is sm.Rsm (IB x IB upper triangle, row c is R(dbase+c, :));
// all NB rows of X are the dense V2 part.  On exit: X = reflectors, sm.tau, sm.Tsm holds the
// IB x IB T factor as Tsm[i*LDT + c] = T(i, c) (upper triangle, zeros below).
template <int NB, int IB, bool GE>
__device__ __forceinline__ void factor_block(Slice<NB, IB, IB>& X, Smem<NB, IB, IB>& sm, int dbase) {
    using G = Geom<NB, IB, IB>;
    const int lane = lane_id(), g = lane >> 2, t = lane & 3, wq = warp_id();
    const int rbase = wq * G::RW + 2 * t;   // row of acc[.][nf][e] = rbase + nf*8 + e

#pragma unroll
    for (int mfc = 0; mfc < G::MF; ++mfc) {
#pragma unroll 1
        for (int gc = 0; gc < 8; ++gc) {
            const int c = mfc * 8 + gc;
            const int d = dbase + c;
            const bool mycol = (g == gc);
            // 1. ||x_below||^2
            double ss = 0.0;
            if (mycol) {
#pragma unroll
                for (int nf = 0; nf < G::NF; ++nf)
#pragma unroll
                    for (int e = 0; e < 2; ++e) {
                        const int r = rbase + nf * 8 + e;
                        const double x = X.acc[mfc][nf][e];
                        if (!GE || r > d) ss += x * x;
                        if (GE && r == d) sm.x0 = x;
                    }
            }
            ss += __shfl_xor_sync(0xffffffffu, ss, 1);
            ss += __shfl_xor_sync(0xffffffffu, ss, 2);
            if (lane == gc * 4) sm.red1[wq] = ss;
            __syncthreads();
            double xn2 = 0.0;
#pragma unroll
            for (int w = 0; w < kWarps; ++w) xn2 += sm.red1[w];
            const double x0 = GE ? sm.x0 : sm.Rsm[c * IB + c];
            double beta = x0, tau = 0.0, scale = 0.0;
            if (xn2 > 0.0) {
                const double nrm = sqrt(x0 * x0 + xn2);
                beta = (x0 < 0.0) ? nrm : -nrm;          // beta = -sgn(x0) ||x||, sgn(0)=+1
                tau = (beta - x0) / beta;
                scale = 1.0 / (x0 - beta);
            }
            // 2. v = x / (x0 - beta) below the diagonal; diagonal <- beta
            if (mycol) {
#pragma unroll
                for (int nf = 0; nf < G::NF; ++nf)
#pragma unroll
                    for (int e = 0; e < 2; ++e) {
                        const int r = rbase + nf * 8 + e;
                        if (!GE || r > d) X.acc[mfc][nf][e] *= scale;
                        else if (r == d) X.acc[mfc][nf][e] = beta;
                    }
            }
            if (threadIdx.x == 0) {
                sm.tau[c] = tau;
                if (!GE) sm.Rsm[c * IB + c] = beta;
            }
            // 3. v for my rows (from the lane holding column c, same t)
            double vv[G::NF][2];
#pragma unroll
            for (int nf = 0; nf < G::NF; ++nf)
#pragma unroll
                for (int e = 0; e < 2; ++e) {
                    const double x = __shfl_sync(0xffffffffu, X.acc[mfc][nf][e], gc * 4 + t);
                    const int r = rbase + nf * 8 + e;
                    vv[nf][e] = GE ? ((r > d) ? x : (r == d ? 1.0 : 0.0)) : x;
                }
            // 4. partial dots v^T X(:, j) for my columns j > c
            double pd[G::MF];
#pragma unroll
            for (int mf = 0; mf < G::MF; ++mf) {
                double s = 0.0;
                if (mf * 8 + g > c) {
#pragma unroll
                    for (int nf = 0; nf < G::NF; ++nf) s += vv[nf][0] * X.acc[mf][nf][0] + vv[nf][1] * X.acc[mf][nf][1];
                }
                s += __shfl_xor_sync(0xffffffffu, s, 1);
                s += __shfl_xor_sync(0xffffffffu, s, 2);
                pd[mf] = s;
            }
            if (t == 0) {
#pragma unroll
                for (int mf = 0; mf < G::MF; ++mf)
                    if (mf * 8 + g > c) sm.red[wq * IB + mf * 8 + g] = pd[mf];
            }
            __syncthreads();
            // 5. w_j = R(c, j) + sum_w partial ; R(c, j) -= tau w_j
            if (threadIdx.x > c && threadIdx.x < IB) {
                const int j = threadIdx.x;
                double s = GE ? 0.0 : sm.Rsm[c * IB + j];
#pragma unroll
                for (int w = 0; w < kWarps; ++w) s += sm.red[w * IB + j];
                sm.wvec[j] = s;
                if (!GE) sm.Rsm[c * IB + j] -= tau * s;
            }
            __syncthreads();
            // 6. X(:, j) -= tau v w_j
#pragma unroll
            for (int mf = 0; mf < G::MF; ++mf) {
                if (mf * 8 + g > c) {
                    const double tw = tau * sm.wvec[mf * 8 + g];
#pragma unroll
                    for (int nf = 0; nf < G::NF; ++nf) {
                        X.acc[mf][nf][0] -= tw * vv[nf][0];
                        X.acc[mf][nf][1] -= tw * vv[nf][1];
                    }
                }
            }
        }
    }

    // ---- T factor: Gram G = V^T V (strict upper part used), DMMA on register fragments
    {
        double gacc[G::MF][G::MF][2];
#pragma unroll
        for (int i = 0; i < G::MF; ++i)
#pragma unroll
            for (int j = 0; j < G::MF; ++j) gacc[i][j][0] = gacc[i][j][1] = 0.0;
#pragma unroll
        for (int nf = 0; nf < G::NF; ++nf)
#pragma unroll
            for (int e = 0; e < 2; ++e) {
                const int r = rbase + nf * 8 + e;
                double v[G::MF];
#pragma unroll
                for (int mf = 0; mf < G::MF; ++mf) {
                    const double x = X.acc[mf][nf][e];
                    const int dc = dbase + mf * 8 + g;
                    v[mf] = GE ? ((r > dc) ? x : (r == dc ? 1.0 : 0.0)) : x;
                }
#pragma unroll
                for (int i = 0; i < G::MF; ++i)
#pragma unroll
                    for (int j = 0; j < G::MF; ++j) dmma(gacc[i][j][0], gacc[i][j][1], v[i], v[j]);
            }
        // gacc[i][j] = G[c' = i*8+g][c = j*8 + 2t + e]
        double* rw = sm.red + wq * (IB * G::LDR);
#pragma unroll
        for (int i = 0; i < G::MF; ++i)
#pragma unroll
            for (int j = 0; j < G::MF; ++j)
                st2(rw + (i * 8 + g) * G::LDR + j * 8 + 2 * t, gacc[i][j][0], gacc[i][j][1]);
        __syncthreads();
        for (int idx = threadIdx.x; idx < IB * IB; idx += kThreads) {
            const int cp = idx / IB, c = idx % IB;
            double s = 0.0;
#pragma unroll
            for (int w = 0; w < kWarps; ++w) s += sm.red[w * (IB * G::LDR) + cp * G::LDR + c];
            sm.Wsm[cp * G::LDW + c] = s;   // Gram(c', c)
        }
        __syncthreads();
        // forward dlarft recurrence by warp 0: T(c,c) = tau_c; T(0:c, c) = -tau_c T(0:c,0:c) G(0:c, c)
        if (wq == 0) {
            for (int i = lane; i < IB * IB; i += 32) sm.Tsm[i] = 0.0;
            __syncwarp();
            for (int c = 0; c < IB; ++c) {
                const double tc = sm.tau[c];
                double s = 0.0;
                if (lane < c) {
                    for (int l = lane; l < c; ++l) s += sm.Tsm[lane * G::LDT + l] * sm.Wsm[l * G::LDW + c];
                }
                __syncwarp();
                if (lane < c) sm.Tsm[lane * G::LDT + c] = -tc * s;
                if (lane == 0) sm.Tsm[c * G::LDT + c] = tc;
                __syncwarp();
            }
        }
        __syncthreads();
    }
}

}  // namespace tqr
