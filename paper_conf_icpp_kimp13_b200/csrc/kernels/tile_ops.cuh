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

#ifdef TQR_PHASE_PROF
// Probe-only instrumentation (tools/probes): per-phase clock64 totals of warp 0 of every CTA.
__device__ unsigned long long g_phase[16];
#define TQR_PH(i) do { if ((threadIdx.x & 255) == 0) { long long _c = clock64(); \
    atomicAdd(&g_phase[i], (unsigned long long)(_c - _ph)); _ph = _c; } } while (0)
#define TQR_PH0() long long _ph = clock64()
__device__ unsigned long long g_fphase[4];
#define TQR_FP(i) do { if (threadIdx.x == 0 && blockIdx.x == gridDim.x - 1) { long long _c = clock64(); \
    atomicAdd(&g_fphase[i], (unsigned long long)(_c - _fp)); _fp = _c; } } while (0)
#define TQR_FP0() long long _fp = clock64()
// column-step phases of factor_block (thread 0 of the last CTA): g_cphase[0] shuffle + scale,
// [1] dots + record, [2] barrier, [3] sums + sqrt/div, [4] w_j, [5] update + store
__device__ unsigned long long g_cphase[8];
#define TQR_FC(i) do { if (threadIdx.x == 0 && blockIdx.x == gridDim.x - 1) { long long _c = clock64(); \
    atomicAdd(&g_cphase[i], (unsigned long long)(_c - _fc)); _fc = _c; } } while (0)
#define TQR_FC0() long long _fc = clock64()
#else
#define TQR_FC(i) do {} while (0)
#define TQR_FC0() do {} while (0)
#define TQR_FP(i) do {} while (0)
#define TQR_FP0() do {} while (0)
#define TQR_PH(i) do {} while (0)
#define TQR_PH0() do {} while (0)
#endif

constexpr int kThreads = 256;
constexpr int kWarps = 8;

template <int NB, int W, int IB>
struct Geom {
    static constexpr int RW = NB / kWarps;   // rows per warp
    static constexpr int NF = RW / 8;        // 8-row fragments per warp
    static constexpr int MF = W / 8;         // 8-column fragments
    static constexpr int JF = IB / 8;        // 8-wide ib fragments
    static constexpr int HC = IB / 2;        // ib columns per V staging half
    static constexpr int JC = JF / 2;        // ib fragments per GEMM1 pass (one pass per half)
    static constexpr int LDR = IB + 4;       // red[slot][col][ib]
    static constexpr int LDW = IB + 4;       // Wsm[col][ib]      (== 4 mod 16: conflict-free A-frag loads)
    static constexpr int LDT = IB;           // Tsm[i][c] (factor output)
    static constexpr int LDT2 = IB + 2;      // Traw[c][r'] (cp.async target, 16-byte aligned columns)
    static constexpr int SWZ = (RW >= 16) ? 4 : 0;   // V staging: 16-byte chunk index ^= SWZ*(col&1)
    static constexpr int CPC = RW / 2;       // 16-byte chunks per staged column
    static constexpr int NQ = (HC * CPC + 31) / 32;   // chunks per lane per half
    static constexpr int VSTN = kWarps * 2 * HC * RW;
    static constexpr int GRAMN = kWarps * IB * LDR;  // factor_block Gram partials (Vst + red + pad)
    static_assert(NB % 64 == 0 && W % 8 == 0 && IB % 16 == 0 && NB % IB == 0, "tile geometry");
};

// Shared-memory workspace of one CTA.  FACT = panel kernel (factor_block members, 4-slot
// two-stage reduction); !FACT = update kernel (8-slot single-stage reduction).
//   Vst  : per-warp staging of the warp's RW rows of the current V block, two ib-halves,
//          filled by one cp.async.bulk (8 KB at nb=512) per warp and half from the
//          pre-swizzled "stage image" of V that the panel kernel writes (vimg_off), so the
//          GEMM1 16-byte / GEMM2 8-byte fragment reads are conflict-free / 2-way with no
//          per-lane copy instructions.  Half B of block s is issued at the start of block s,
//          half A of block s+1 as soon as GEMM2 has finished reading half A of block s.
//   red  : NSLOT slots of W x IB GEMM1 partials.
template <int NB, int W, int IB, bool FACT>
struct Smem {
    using G = Geom<NB, W, IB>;
    static constexpr int NSLOT = FACT ? 4 : 8;
    static constexpr int REDN = NSLOT * W * G::LDR;
    static constexpr int PADN = (FACT && G::GRAMN > G::VSTN + REDN) ? G::GRAMN - G::VSTN - REDN : 2;
    uint64_t mbar[kWarps][2];          // bulk-copy completion of Vst[w][h]; first member, so every
                                       // workspace variant (panel apply W / factor IB) shares it and
                                       // no other use ever overwrites it
    double Vst[kWarps][2][G::HC][G::RW];
    double red[REDN];
    double gram_pad[PADN];             // Vst..gram_pad is the contiguous Gram scratch of factor_block
    double Wsm[W * G::LDW];            // -op(T) W  (A operand of GEMM2), element (ib, col) at col*LDW + ib
    double Traw[IB * G::LDT2];         // T block s, element (r', r) at r*LDT2 + r'
    double topsm[W * G::LDW];          // top rows X1 (IB x W), element (r, c) at c*LDW + r
    double Tsm[FACT ? IB * G::LDT : 2];   // factor_block output T(i, c) at i*LDT + c
    double Rsm[FACT ? IB * IB : 2];       // TSQRT diagonal R block (row c, col j) at c*IB + j
    double tau[FACT ? IB : 2];
    double wvec[FACT ? IB : 2];
    double red1[FACT ? kWarps : 2];
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
    // rows >= r0min only (r0min a multiple of 8)
    __device__ __forceinline__ void store_rows_from(double* P, int64_t ld, int r0min) const {
        const int g = lane_id() >> 2, t = lane_id() & 3, rw = warp_id() * G::RW;
#pragma unroll
        for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
            for (int nf = 0; nf < G::NF; ++nf)
                if (rw + nf * 8 + 8 > r0min)
                    st2(P + (int64_t)(mf * 8 + g) * ld + rw + 2 * t + nf * 8, acc[mf][nf][0], acc[mf][nf][1]);
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

// Element (r, c) of one warp's staging half: chunk-swizzled column-major.
template <int NB, int W, int IB>
__device__ __forceinline__ int vst_off(int r, int c) {
    using G = Geom<NB, W, IB>;
    return c * G::RW + 2 * ((r >> 1) ^ (G::SWZ * (c & 1))) + (r & 1);
}

// Stage image of a V tile (NB x NB, written by the panel kernel): ib block s, warp rows q, half h
// is the contiguous HC*RW chunk at s*IB*NB + (q*2 + h)*HC*RW, laid out exactly like Vst[q][h].
template <int NB, int W, int IB>
__device__ __forceinline__ int64_t vimg_off(int s, int q, int h, int r, int c) {
    using G = Geom<NB, W, IB>;
    return (int64_t)s * IB * NB + (q * 2 + h) * (G::HC * G::RW) + vst_off<NB, W, IB>(r, c);
}

// Per-warp bulk staging of half h of block image `blk` (lane 0 issues; WAR-safe after the
// warp's own reads of that half: __syncwarp + async-proxy fence).
template <int NB, int W, int IB, bool FACT>
__device__ __forceinline__ void stage_bulk(Smem<NB, W, IB, FACT>& sm, const double* blk, int h) {
    using G = Geom<NB, W, IB>;
    const int wq = warp_id();
    __syncwarp();
    if (lane_id() == 0) {
        fence_proxy_async_shared();
        bulk_g2s(&sm.Vst[wq][h][0][0], blk + (wq * 2 + h) * (G::HC * G::RW), G::HC * G::RW * 8, &sm.mbar[wq][h]);
    }
}
template <int NB, int W, int IB, bool FACT>
__device__ __forceinline__ void stage_init(Smem<NB, W, IB, FACT>& sm) {
    if (lane_id() == 0) {
        mbar_init(&sm.mbar[warp_id()][0], 1);
        mbar_init(&sm.mbar[warp_id()][1], 1);
        fence_mbar_init();
    }
    __syncwarp();
}
// Prologue of a block sequence: half A of the first block.
template <int NB, int W, int IB, bool FACT>
__device__ __forceinline__ void stage_first(Smem<NB, W, IB, FACT>& sm, const double* blk) {
    stage_bulk(sm, blk, 0);
}

// ---------------------------------------------------------------- apply one ib block
// X (registers, NB x W) <- H_s X where H_s = I - V_s T_s^T V_s^T (TRANS) or I - V_s T_s V_s^T.
//   Vs   : stage image of V block s (vimg_off); rows < kmin are zero (their DMMAs skipped).
//          Half A must be in flight (stage_first, or `next` of the previous call).
//   vph  : the warp's mbarrier phase bits (bit h for half h), carried across calls.
//   Ts   : T block s (IB x IB column-major, ld = IB) = T_tile + s*IB*IB (zeros below diagonal).
//   top  : if non-null, the X1 rows (IB x W, element (r, c) at top[c*ldtop + r]).
//   next : stage image of the following call's block -- its half A is staged here -- or null.
//   KM   : kmin may be > 0 (UNMQR / GEQRT blocks) or kmax < NB (TT merges: a triangular bottom
//          keeps V and X zero on rows >= kmax); false compiles the TS path branch-free.
template <int NB, int W, int IB, bool FACT, bool TRANS, bool CG, bool KM>
__device__ __forceinline__ void apply_block(Slice<NB, W, IB>& X, Smem<NB, W, IB, FACT>& sm,
                                            const double* __restrict__ Vs,
                                            const double* __restrict__ Ts,
                                            double* top, int64_t ldtop, int kmin,
                                            const double* next, unsigned& vph, int kmax = 1 << 30) {
    using G = Geom<NB, W, IB>;
    using SM = Smem<NB, W, IB, FACT>;
    const int lane = lane_id(), g = lane >> 2, t = lane & 3, wq = warp_id();
    const int rbase = wq * G::RW;
    const int tid = threadIdx.x;
    // 8 slots: -W'(col, r) lives in the 4 padding doubles (ib IB..IB+3) of slot r/4, column col;
    // A-fragment loads hit banks (4g + t) mod 16 (two wavefronts)
    static_assert(SM::NSLOT != 8 || G::LDR - IB == 4 && IB <= 4 * SM::NSLOT, "padding holds -W'");
    auto pad_off = [](int col, int r) { return (r >> 2) * (W * G::LDR) + col * G::LDR + IB + (r & 3); };
    TQR_PH0();

    // ---- (0) half B of V (bulk), T block and top rows (LDGSTS group, waited before barrier 1)
    stage_bulk(sm, Vs, 1);                    // half B of this block (its buffer was read last call)
    {
        constexpr int TCH = IB * IB / 2;      // 16-byte chunks of the T block
        for (int id = tid; id < TCH; id += kThreads) {
            const int c = id / (IB / 2), r2 = id % (IB / 2);
            cp_async16<CG>(&sm.Traw[c * G::LDT2 + 2 * r2], Ts + c * IB + 2 * r2);
        }
        if (top) {
            constexpr int XCH = W * IB / 2;   // 16-byte chunks of the top rows
            for (int id = tid; id < XCH; id += kThreads) {
                const int c = id / (IB / 2), r2 = id % (IB / 2);
                cp_async16<true>(&sm.topsm[c * G::LDW + 2 * r2], top + (int64_t)c * ldtop + 2 * r2);
            }
        }
        cp_async_commit();
    }
    TQR_PH(0);

    // ---- (1) GEMM1: partial W^T(col, ib) = sum_{my rows} X(row, col) V(row, ib), one pass per half.
    //      Narrow slices (MF <= 2: the lookahead and panel sub-slices) have only MF * JC accumulator
    //      chains per half; they get a second set for odd row fragments (NP = 2) so consecutive
    //      DMMAs do not wait on each other's results, summed once at the end.
#ifdef TQR_GEMM1_SPLIT
    constexpr int NP = (G::MF <= 2) ? 2 : 1;
#else
    constexpr int NP = 1;
#endif
    double c1[2][G::MF][G::JC][2];
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        mbar_wait(&sm.mbar[wq][h], (vph >> h) & 1u);
        vph ^= 1u << h;
        TQR_PH(h == 0 ? 5 : 11);                  // (probe) staging wait of V half h
        const double* vh = &sm.Vst[wq][h][0][0];
        double cp[NP][G::MF][G::JC][2];
#pragma unroll
        for (int pp = 0; pp < NP; ++pp)
#pragma unroll
            for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
                for (int j = 0; j < G::JC; ++j) cp[pp][mf][j][0] = cp[pp][mf][j][1] = 0.0;
#pragma unroll
        for (int nf = 0; nf < G::NF; ++nf) {
            if (KM && (rbase + nf * 8 + 8 <= kmin || rbase + nf * 8 >= kmax)) continue;  // V rows all zero (warp-uniform)
            const int pp = (NP == 2) ? (nf & 1) : 0;
            double2 b[G::JC];
#pragma unroll
            for (int j = 0; j < G::JC; ++j)
                b[j] = *reinterpret_cast<const double2*>(vh + vst_off<NB, W, IB>(nf * 8 + 2 * t, j * 8 + g));
#pragma unroll
            for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
                for (int j = 0; j < G::JC; ++j) dmma(cp[pp][mf][j][0], cp[pp][mf][j][1], X.acc[mf][nf][0], b[j].x);
#pragma unroll
            for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
                for (int j = 0; j < G::JC; ++j) dmma(cp[pp][mf][j][0], cp[pp][mf][j][1], X.acc[mf][nf][1], b[j].y);
        }
#pragma unroll
        for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
            for (int j = 0; j < G::JC; ++j) {
                c1[h][mf][j][0] = cp[0][mf][j][0];
                c1[h][mf][j][1] = cp[0][mf][j][1];
                if (NP == 2) {
                    c1[h][mf][j][0] += cp[NP - 1][mf][j][0];
                    c1[h][mf][j][1] += cp[NP - 1][mf][j][1];
                }
            }
        TQR_PH(1 + h);
    }
    // c1[h][mf][j] = W^T[col mf*8+g][ib h*HC + j*8 + 2t + e]
    // ---- (2) GEMM1 partials -> smem slots (8 slots, or 4 with a pairwise add for the panel)
    auto frag_ptr = [&](int slot, int h, int mf, int j) {
        return sm.red + slot * (W * G::LDR) + (mf * 8 + g) * G::LDR + h * G::HC + j * 8 + 2 * t;
    };
    cp_async_wait<0>();                       // this thread's T-block / top-row chunks landed
    if constexpr (SM::NSLOT == 8) {
#pragma unroll
        for (int h = 0; h < 2; ++h)
#pragma unroll
            for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
                for (int j = 0; j < G::JC; ++j) st2(frag_ptr(wq, h, mf, j), c1[h][mf][j][0], c1[h][mf][j][1]);
        __syncthreads();
        TQR_PH(3);
    } else {   // 4 slots: warps 4..7 store, warps 0..3 add
        if (wq >= 4) {
#pragma unroll
            for (int h = 0; h < 2; ++h)
#pragma unroll
                for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
                    for (int j = 0; j < G::JC; ++j) st2(frag_ptr(wq - 4, h, mf, j), c1[h][mf][j][0], c1[h][mf][j][1]);
        }
        __syncthreads();
        TQR_PH(3);
        if (wq < 4) {
#pragma unroll
            for (int h = 0; h < 2; ++h)
#pragma unroll
                for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
                    for (int j = 0; j < G::JC; ++j) {
                        double* pp = frag_ptr(wq, h, mf, j);
                        const double2 o = *reinterpret_cast<const double2*>(pp);
                        st2(pp, o.x + c1[h][mf][j][0], o.y + c1[h][mf][j][1]);
                    }
        }
        __syncthreads();
    }
    TQR_PH(4);
    // ---- (3) fused reduction + T multiply on DMMA: W'^T = (top + sum_slots P)^T op(T)^T,
    //      C[m = col][n = r] = sum_k W^T[col][k] B[k][n],  B = T (TRANS: W' = T^T W) or T^T.
    //      The A operand (W^T fragment) is summed from the partial slots as it is loaded; each
    //      warp owns fragments with one column block mf so it sums that A operand once.
    //      Wsm = -W' (GEMM2 operand); top -= W' written straight from the fragments.
    if constexpr (SM::NSLOT == 8) {
        // 8 slots (update kernel): reduce-scatter of the slots (+ top) into Wsm = W -- every
        // element read once, 16-byte pairs, eight consecutive threads on 128 contiguous bytes --
        // then the T multiply with A from Wsm (one load per k-step instead of nine) and the k-steps
        // past a fragment's triangle skipped (exact zeros); -W' overwrites Wsm after a barrier.
        // (Same sum order and products as the fused form below, which the 4-slot panel keeps.)
        constexpr int NPAIR = W * IB / 2;
        for (int idx = tid; idx < NPAIR; idx += kThreads) {
            const int col = idx / (IB / 2), ib = 2 * (idx % (IB / 2));
            double2 sv = top ? ld2(&sm.topsm[col * G::LDW + ib]) : make_double2(0.0, 0.0);
#pragma unroll
            for (int sl = 0; sl < SM::NSLOT; ++sl) {
                const double2 pv = ld2(&sm.red[sl * (W * G::LDR) + col * G::LDR + ib]);
                sv.x += pv.x;
                sv.y += pv.y;
            }
            st2(&sm.Wsm[col * G::LDW + ib], sv.x, sv.y);
        }
        __syncthreads();
        constexpr int NFRAG = G::MF * G::JF;
        constexpr int FPW = (NFRAG + kWarps - 1) / kWarps;
        const int f0 = wq * FPW, mf = f0 / G::JF;
        double acc0[FPW][2], acc1[FPW][2];
#pragma unroll
        for (int u = 0; u < FPW; ++u) acc0[u][0] = acc0[u][1] = acc1[u][0] = acc1[u][1] = 0.0;
        if (wq * FPW < NFRAG) {
#pragma unroll
            for (int kk = 0; kk < IB; kk += 4) {
                const double av = sm.Wsm[(mf * 8 + g) * G::LDW + kk + t];
#pragma unroll
                for (int u = 0; u < FPW; ++u) {
                    const int jf = (f0 + u) % G::JF;
                    if (TRANS && kk >= jf * 8 + 8) continue;
                    if (!TRANS && kk + 4 <= jf * 8) continue;
                    double bv;
                    if constexpr (TRANS) bv = sm.Traw[(jf * 8 + g) * G::LDT2 + kk + t];
                    else                 bv = sm.Traw[(kk + t) * G::LDT2 + jf * 8 + g];
                    if ((kk >> 2) & 1) dmma(acc1[u][0], acc1[u][1], av, bv);
                    else               dmma(acc0[u][0], acc0[u][1], av, bv);
                }
            }
        }
        // -W' goes to the padding of the partial slots (pad_off), which no GEMM1 store writes, so no
        // barrier is needed between the reads of Wsm above and these writes
        if (wq * FPW < NFRAG) {
#pragma unroll
            for (int u = 0; u < FPW; ++u) {
                const int jf = (f0 + u) % G::JF;
                const double w0 = acc0[u][0] + acc1[u][0], w1 = acc0[u][1] + acc1[u][1];
                const int col = mf * 8 + g, r = jf * 8 + 2 * t;
                st2(&sm.red[pad_off(col, r)], -w0, -w1);
                if (top) st2(top + (int64_t)col * ldtop + r, sm.topsm[col * G::LDW + r] - w0,
                             sm.topsm[col * G::LDW + r + 1] - w1);
            }
        }
    } else {
        constexpr int NFRAG = G::MF * G::JF;
        constexpr int FPW = (NFRAG + kWarps - 1) / kWarps;   // fragments per warp (JF % FPW == 0)
        static_assert(NFRAG <= kWarps || G::JF % FPW == 0, "fragment assignment");
        if (wq * FPW < NFRAG) {
            const int f0 = wq * FPW;
            const int mf = f0 / G::JF;
            double acc0[FPW][2], acc1[FPW][2];
#pragma unroll
            for (int u = 0; u < FPW; ++u) acc0[u][0] = acc0[u][1] = acc1[u][0] = acc1[u][1] = 0.0;
            const double* wa = sm.red + (mf * 8 + g) * G::LDR + t;
            const double* ta = sm.topsm + (mf * 8 + g) * G::LDW + t;
#pragma unroll
            for (int kk = 0; kk < IB; kk += 4) {
                double av = top ? ta[kk] : 0.0;
#pragma unroll
                for (int sl = 0; sl < SM::NSLOT; ++sl) av += wa[sl * (W * G::LDR) + kk];
#pragma unroll
                for (int u = 0; u < FPW; ++u) {
                    const int jf = (f0 + u) % G::JF;
                    double bv;
                    if constexpr (TRANS) bv = sm.Traw[(jf * 8 + g) * G::LDT2 + kk + t];   // T(kk+t, r)
                    else                 bv = sm.Traw[(kk + t) * G::LDT2 + jf * 8 + g];   // T(r, kk+t)
                    if ((kk >> 2) & 1) dmma(acc1[u][0], acc1[u][1], av, bv);
                    else               dmma(acc0[u][0], acc0[u][1], av, bv);
                }
            }
#pragma unroll
            for (int u = 0; u < FPW; ++u) {
                const int jf = (f0 + u) % G::JF;
                const double w0 = acc0[u][0] + acc1[u][0], w1 = acc0[u][1] + acc1[u][1];
                const int col = mf * 8 + g, r = jf * 8 + 2 * t;
                st2(&sm.Wsm[col * G::LDW + r], -w0, -w1);
                if (top) st2(top + (int64_t)col * ldtop + r, sm.topsm[col * G::LDW + r] - w0,
                             sm.topsm[col * G::LDW + r + 1] - w1);
            }
        }
    }
    __syncthreads();
    TQR_PH(6);
    TQR_PH(7);
    // ---- (4) GEMM2: X^T(col, row) += (-W'^T)(col, ib) V^T(ib, row); half A of `next` staged
    //      inside the half-B loop (half A of this block is no longer read there)
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        if (h == 1 && next != nullptr) stage_bulk(sm, next, 0);   // half A of the next block
        const double* vh = &sm.Vst[wq][h][0][0];
#pragma unroll
        for (int kk = 0; kk < G::HC; kk += 4) {
            double a[G::MF];
#pragma unroll
            for (int mf = 0; mf < G::MF; ++mf)
                a[mf] = (SM::NSLOT == 8) ? sm.red[pad_off(mf * 8 + g, h * G::HC + kk + t)]
                                         : sm.Wsm[(mf * 8 + g) * G::LDW + h * G::HC + kk + t];
#pragma unroll
            for (int nf = 0; nf < G::NF; ++nf) {
                if (KM && (rbase + nf * 8 + 8 <= kmin || rbase + nf * 8 >= kmax)) continue;
                const double b = vh[vst_off<NB, W, IB>(nf * 8 + g, kk + t)];
#pragma unroll
                for (int mf = 0; mf < G::MF; ++mf) dmma(X.acc[mf][nf][0], X.acc[mf][nf][1], a[mf], b);
            }
        }
        TQR_PH(8 + h);
    }
    // Exit: at most one bulk copy (half A of `next`) in flight.  The next call's first
    // barrier is preceded only by warp-private Vst traffic and red stores into slots that every
    // warp finished reading before this call's last barrier.
}

// ---------------------------------------------------------------- factor ib columns
// Exact powers of two for the scaled norms of factor_block (reading Q26).
// 2^e for -1022 <= e <= 1023, built from the exponent bits; 0 for e < -1022 (a contribution
// scaled that far down is below the smallest normal relative to the column's largest entry).
__device__ __forceinline__ double pow2s(int e) {
    return e < -1022 ? 0.0 : __longlong_as_double((long long)(e + 1023) << 52);
}
// floor(log2 |x|) for normal x, -1022 for subnormal x, kNoExp for 0
constexpr int kNoExp = -4096;
__device__ __forceinline__ int exp2_floor(double x) {
    const int f = (int)((__double_as_longlong(x) >> 52) & 0x7ff);
    return x == 0.0 ? kNoExp : (f == 0 ? 1 : f) - 1023;
}

// SCALED = false (fast path): unscaled sums; returns true -- before touching sm.Rsm or building
// the Gram -- when some column left the range where they are exact (an entry of the block above
// 2^490, or a sub-column norm outside [2^-100, 2^100]); the caller then restores X and calls the
// SCALED = true version, which scales every column as described below and never fails.
template <int NB, int IB, bool GE, bool SCALED = false>
__device__ __forceinline__ bool factor_block(Slice<NB, IB, IB>& X, Smem<NB, IB, IB, true>& sm, int dbase) {
    using G = Geom<NB, IB, IB>;
    const int lane = lane_id(), g = lane >> 2, t = lane & 3, wq = warp_id();
    const int rbase = wq * G::RW + 2 * t;   // row of acc[.][nf][e] = rbase + nf*8 + e
    bool bad = false;
    double wmax = 0.0;                      // fast path: largest |entry| of the block (incl. the TS top)
    if constexpr (!SCALED) {
#pragma unroll
        for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
            for (int nf = 0; nf < G::NF; ++nf)
                wmax = fmax(wmax, fmax(fabs(X.acc[mf][nf][0]), fabs(X.acc[mf][nf][1])));
        if (!GE)
            for (int idx = lane; idx < IB * IB; idx += 32) wmax = fmax(wmax, fabs(sm.Rsm[idx]));
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) wmax = fmax(wmax, __shfl_xor_sync(0xffffffffu, wmax, o));
    }
    // One barrier per column: each warp publishes, for column c, the partial ||x_below||^2, the
    // unscaled dots x^T a_j of every column j of the block and (GEQRT) the row-d entries a_dj;
    // after the barrier every thread forms beta, tau, scale = 1/(x0 - beta) and
    // w_j = a_dj (GEQRT) or R(c, j) (TSQRT) + scale * sum_w (x^T a_j)_w itself (v = scale x).
    // Column record, double-buffered by column parity (fb + (c & 1) * RECN), laid out for the reads
    // after the barrier: dots[j][w] (warp partials of x^T a_j, warp index fastest, row stride 10 so
    // the writers' banks differ and each thread reads its columns' 8 partials as four double2), then
    // ||x_w||^2[w], e_w[w] (or, fast path at c = 0, the block max) and the GEQRT diagonal row a_dj
    // (written once, by the warp that owns row d).
    constexpr int DLD = 10;                   // dots row stride (doubles)
    constexpr int OSS = IB * DLD, OEX = OSS + kWarps, ODG = OEX + kWarps;
    constexpr int RECN = ODG + IB + 2;        // + pad: every buffer starts 16-byte aligned
    static_assert(RECN % 2 == 0 && 2 * RECN <= Smem<NB, IB, IB, true>::REDN, "factor record buffer");
    double* fb = sm.red;
    double* Rout = sm.topsm;                  // TSQRT: R rows written as they are finished
    static_assert(IB * IB <= IB * G::LDW, "Rout buffer");
    TQR_FP0();
    // Scaled norms and dots (dlarfg / dnrm2 semantics, reading Q26) at no extra barrier: each warp
    // scales its part of x by the exact power of two 2^-e_w of its own largest |x| before forming
    // ||x_w||^2 and x_w^T a_j, and records e_w; after the barrier the partials are brought to the
    // column's common scale 2^-e, e = max(e_w, e(x0)), by exact power-of-two factors.  Nothing can
    // overflow (scaled |x| < 2) and nothing that matters can underflow (a term is lost only when it
    // is below 2^-1022 relative to the column's largest entry).  Powers of two are exact, so in the
    // normal range every quantity is bitwise the unscaled formula's.
    // Sum of the 8 warp partials at p8 (times fw[w] = 2^(e_w - ec) when scaled), as a tree:
    // ((p0 + p1) + (p2 + p3)) + ((p4 + p5) + (p6 + p7)); four 16-byte loads.  (Splitting the loads
    // across a lane quad + two butterflies measured slower: profiles/r02_factor_phases.txt.)
    auto sum8 = [](const double* p8, const double* f) {
        const double2 a0 = *reinterpret_cast<const double2*>(p8), a1 = *reinterpret_cast<const double2*>(p8 + 2);
        const double2 a2 = *reinterpret_cast<const double2*>(p8 + 4), a3 = *reinterpret_cast<const double2*>(p8 + 6);
        if (f == nullptr)
            return ((a0.x + a0.y) + (a1.x + a1.y)) + ((a2.x + a2.y) + (a3.x + a3.y));
        return ((a0.x * f[0] + a0.y * f[1]) + (a1.x * f[2] + a1.y * f[3])) +
               ((a2.x * f[4] + a2.y * f[5]) + (a3.x * f[6] + a3.y * f[7]));
    };

#pragma unroll
    for (int mfc = 0; mfc < G::MF; ++mfc) {
#pragma unroll 1
        for (int gc = 0; gc < 8; ++gc) {
            const int c = mfc * 8 + gc;
            const int d = dbase + c;
            double* fbp = fb + (c & 1) * RECN;
            TQR_FC0();
            // 1. x = column c on my rows (from the lane holding it, same t), masked to rows > d (GEQRT),
            //    scaled by 2^-ew (ew = exponent of the warp's largest |x|)
            double xv[G::NF][2];
#pragma unroll
            for (int nf = 0; nf < G::NF; ++nf)
#pragma unroll
                for (int e = 0; e < 2; ++e) {
                    const double x = __shfl_sync(0xffffffffu, X.acc[mfc][nf][e], gc * 4 + t);
                    const int r = rbase + nf * 8 + e;
                    xv[nf][e] = (!GE || r > d) ? x : 0.0;
                }
            int ew = 0;
            if constexpr (SCALED) {
                double xm = 0.0;
#pragma unroll
                for (int nf = 0; nf < G::NF; ++nf) xm = fmax(xm, fmax(fabs(xv[nf][0]), fabs(xv[nf][1])));
                xm = fmax(xm, __shfl_xor_sync(0xffffffffu, xm, 1));
                xm = fmax(xm, __shfl_xor_sync(0xffffffffu, xm, 2));
                ew = exp2_floor(xm);
                const int eu = (ew == kNoExp) ? 0 : ew;                   // x == 0 on this warp: unscaled
                const double sw = pow2s(-eu / 2) * pow2s(eu / 2 - eu);   // 2^-ew in two exact factors
#pragma unroll
                for (int nf = 0; nf < G::NF; ++nf) {
                    xv[nf][0] *= sw;
                    xv[nf][1] *= sw;
                }
            }
            TQR_FC(0);
            // ||x_w||^2 and the dots x_w^T a_j of the columns of groups >= mfc, two accumulators each
            double ss0 = 0.0, ss1 = 0.0;
            if (g == 0) {
#pragma unroll
                for (int nf = 0; nf < G::NF; ++nf) {
                    ss0 += xv[nf][0] * xv[nf][0];
                    ss1 += xv[nf][1] * xv[nf][1];
                }
            }
            double ss = ss0 + ss1;
            // GEQRT: the warp owning row d publishes the diagonal row a_dj (j = mf*8 + g) once
            const bool own_d = GE && (d / G::RW) == wq;
            const int td = ((d % G::RW) % 8) >> 1, ed = d & 1;
            double pd[G::MF];
#pragma unroll
            for (int mf = mfc; mf < G::MF; ++mf) {
                double s0 = 0.0, s1 = 0.0, sdiag = 0.0;
#pragma unroll
                for (int nf = 0; nf < G::NF; ++nf) {
                    s0 += xv[nf][0] * X.acc[mf][nf][0];
                    s1 += xv[nf][1] * X.acc[mf][nf][1];
                    if (GE) {
                        if (rbase + nf * 8 == d) sdiag = X.acc[mf][nf][0];
                        if (rbase + nf * 8 + 1 == d) sdiag = X.acc[mf][nf][1];
                    }
                }
                double sdot = s0 + s1;
                sdot += __shfl_xor_sync(0xffffffffu, sdot, 1);
                sdot += __shfl_xor_sync(0xffffffffu, sdot, 2);
                pd[mf] = sdot;
                if (GE) {
                    sdiag = __shfl_sync(0xffffffffu, sdiag, g * 4 + td);
                    if (own_d && t == 0) fbp[ODG + mf * 8 + g] = sdiag;
                }
            }
            (void)ed;
            ss += __shfl_xor_sync(0xffffffffu, ss, 1);
            ss += __shfl_xor_sync(0xffffffffu, ss, 2);
            if (t == 0) {
#pragma unroll
                for (int mf = mfc; mf < G::MF; ++mf) fbp[(mf * 8 + g) * DLD + wq] = pd[mf];
                if (g == 0) {
                    fbp[OSS + wq] = ss;
                    if (SCALED) fbp[OEX + wq] = (double)ew;
                    else if (c == 0) fbp[OEX + wq] = wmax;
                }
            }
            TQR_FC(1);
            __syncthreads();
            TQR_FC(2);
            // 2. reflector (dlarfg convention, readings Q1/Q4): beta = -sgn(x0) ||(x0, x)||, in units
            //    of 2^ec; fw[w] = 2^(e_w - ec) brings warp w's partials to that scale
            // the dots of my columns first (independent of the reflector: overlaps sqrt / div)
            double fw[kWarps];
            double fwq = 1.0;
            int ec = 0;
            const double x0 = GE ? fbp[ODG + c] : sm.Rsm[c * IB + c];
            if constexpr (SCALED) {
                int ewv[kWarps];
                ec = kNoExp;
#pragma unroll
                for (int w = 0; w < kWarps; ++w) {
                    ewv[w] = (int)fbp[OEX + w];
                    ec = max(ec, ewv[w]);
                }
                ec = max(ec, exp2_floor(x0));
                if (ec == kNoExp) ec = 0;                                 // x == 0 and x0 == 0
#pragma unroll
                for (int w = 0; w < kWarps; ++w) fw[w] = pow2s(ewv[w] - ec);
                fwq = pow2s(ew - ec);
            }
            double dsum[G::MF], basev[G::MF];
#pragma unroll
            for (int mf = mfc; mf < G::MF; ++mf) {
                const int j = mf * 8 + g;
                dsum[mf] = sum8(fbp + j * DLD, SCALED ? fw : nullptr);
                basev[mf] = GE ? fbp[ODG + j] : sm.Rsm[c * IB + j];
            }
            double xn2;
            if constexpr (SCALED) {
                double f2[kWarps];
#pragma unroll
                for (int w = 0; w < kWarps; ++w) f2[w] = fw[w] * fw[w];
                xn2 = sum8(fbp + OSS, f2);
            } else {
                xn2 = sum8(fbp + OSS, nullptr);
                if (c == 0) {
                    double bm = 0.0;
#pragma unroll
                    for (int w = 0; w < kWarps; ++w) bm = fmax(bm, fbp[OEX + w]);
                    bad = bad || !(bm <= 0x1p490);
                }
                // GEQRT's last tile column has no sub-column (legitimately x = 0, tau = 0)
                if (!(GE && d == NB - 1)) bad = bad || !(xn2 >= 0x1p-200) || !(x0 * x0 + xn2 <= 0x1p200);
            }
            const double se = SCALED ? pow2s(-ec / 2) * pow2s(ec / 2 - ec) : 1.0;   // 2^-ec
            const double x0s = x0 * se;
            double beta = x0, tau = 0.0, scale = 0.0;
            if (xn2 > 0.0) {
                const double nrm = sqrt(x0s * x0s + xn2);
                const double bs = (x0s < 0.0) ? nrm : -nrm;   // beta = -sgn(x0) ||x||, sgn(0)=+1
                tau = (bs - x0s) / bs;                         // correctly rounded: tau ||v||^2 = 2 decides
                scale = 1.0 / (x0s - bs);                      // the orthogonality of I - tau v v^T
                beta = SCALED ? bs * pow2s(ec / 2) * pow2s(ec - ec / 2) : bs;   // back to the caller's scale
            }
            // v on my rows = (x 2^-ew) 2^(ew - ec) scale (+ e_d); |v| <= 1
            const double vfac = SCALED ? scale * fwq : scale;
            TQR_FC(3);
            // 3. w_j for my columns j > c, then X(:, j) -= tau v w_j with v = x / (x0 - beta) (+ e_d)
            double tw[G::MF];
#pragma unroll
            for (int mf = mfc; mf < G::MF; ++mf) {
                const int j = mf * 8 + g;
                tw[mf] = 0.0;
                if (j > c) {
                    const double wj = basev[mf] + scale * dsum[mf];
                    tw[mf] = tau * wj;
                    if (!GE && wq == 0 && t == 0) Rout[c * IB + j] = basev[mf] - tau * wj;
                }
            }
            TQR_FC(4);
#pragma unroll
            for (int mf = mfc; mf < G::MF; ++mf) {
#pragma unroll
                for (int nf = 0; nf < G::NF; ++nf)
#pragma unroll
                    for (int e = 0; e < 2; ++e) {
                        const double v = vfac * xv[nf][e] + ((GE && rbase + nf * 8 + e == d) ? 1.0 : 0.0);
                        X.acc[mf][nf][e] -= tw[mf] * v;
                    }
            }
            // column c itself: v below the diagonal, beta on it
            if (g == gc) {
#pragma unroll
                for (int nf = 0; nf < G::NF; ++nf)
#pragma unroll
                    for (int e = 0; e < 2; ++e) {
                        const int r = rbase + nf * 8 + e;
                        if (!GE || r > d) X.acc[mfc][nf][e] = vfac * xv[nf][e];
                        else if (r == d) X.acc[mfc][nf][e] = beta;
                    }
            }
            if (threadIdx.x == 0) {
                sm.tau[c] = tau;
                if (!GE) Rout[c * IB + c] = beta;
            }
            TQR_FC(5);
        }
    }
    if (!SCALED && bad) {                   // CTA-uniform: sm.Rsm untouched, the caller redoes the block
        __syncthreads();
        return true;
    }
    if (!GE) {   // finished R rows -> Rsm (upper triangle)
        __syncthreads();
        for (int idx = threadIdx.x; idx < IB * IB; idx += kThreads) {
            const int c = idx / IB, j = idx % IB;
            if (j >= c) sm.Rsm[c * IB + j] = Rout[c * IB + j];
        }
    }
    __syncthreads();

    TQR_FP(0);
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
        // 8 warp partials in the (idle) V staging + reduction area (contiguous members)
        using SM = Smem<NB, IB, IB, true>;
        static_assert(G::GRAMN <= G::VSTN + SM::REDN + SM::PADN, "Gram scratch");
        double* scratch = &sm.Vst[0][0][0][0];
        double* rw = scratch + wq * (IB * G::LDR);
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
            for (int w = 0; w < kWarps; ++w) s += scratch[w * (IB * G::LDR) + cp * G::LDR + c];
            sm.Wsm[cp * G::LDW + c] = s;   // Gram(c', c)
        }
        __syncthreads();
        TQR_FP(1);
        // Gram in sm.Wsm; T is built by build_T (after the caller has stored X, freeing registers)
    }
    return false;
}

// Forward dlarft recurrence T(c,c) = tau_c, T(0:c, c) = -tau_c T(0:c, 0:c) G(0:c, c), one row per
// lane of warp 0 held in registers: row i only needs its own earlier entries, so the 32 rows run
// independently with broadcast reads of the Gram matrix (no inter-lane traffic, no barriers).
template <int NB, int IB>
__device__ __forceinline__ void build_T(Smem<NB, IB, IB, true>& sm) {
    using G = Geom<NB, IB, IB>;
    TQR_FP0();
    if (warp_id() == 0 && lane_id() < IB) {
        const int i = lane_id();
        double trow[IB];
#pragma unroll
        for (int c = 0; c < IB; ++c) {
            double s0 = 0.0, s1 = 0.0;
#pragma unroll
            for (int l = 0; l < c; ++l) {
                const double gl = sm.Wsm[l * G::LDW + c];
                if (l & 1) s1 += trow[l] * gl; else s0 += trow[l] * gl;
            }
            const double tc = sm.tau[c];
            trow[c] = (i < c) ? -tc * (s0 + s1) : (i == c ? tc : 0.0);
        }
#pragma unroll
        for (int c = 0; c < IB; ++c) sm.Tsm[i * G::LDT + c] = trow[c];
    }
    __syncthreads();
    TQR_FP(2);
}

}  // namespace tqr
