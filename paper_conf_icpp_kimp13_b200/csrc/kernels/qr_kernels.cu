// qr_kernels.cu -- the sm_100a hot path of the tiled Householder QR.
//
//   panel_kernel  : GEQRT(k,k) followed by the flat-TS chain TSQRT(i,k), i = k+1..p-1
//                   (Eqs. 4-5, 7-8; Fig. 3 DAG P:L332-345; reading Q7: flat,
//                   top-down).  One CTA per ib-wide column block of panel k; CTA b applies
//                   the reflector blocks b' < b of tile i as soon as CTA b' publishes them
//                   (inter-CTA release/acquire flags), then factors its own block.  The chain
//                   over i therefore runs as a wavefront across the NB/IB CTAs.
//   update_kernel : UNMQR(k,j) + TSMQR(i,j,k), i = k+1..p-1, for every trailing column j
//                   (Eqs. 6 and 9).  One CTA per W-wide column slice; the slice of A_ij lives
//                   in registers for all ib blocks of Q_ik, A_kj stays L2-resident as the
//                   "top" row block of every TS pair.  Also used (TRANS / reverse order) for
//                   Q^T B and Q B in tqr_apply_qt.
//   layout kernels: column-major <-> tile-major (128-bit when aligned), R out with zeroed
//                   lower part (the back substitution of tqr_solve_ls is in trsm.cu).
#include <algorithm>
#include <cstdio>
#include <cstring>
#include <type_traits>
#include "tile_ops.cuh"
#include "tile_w16.cuh"
#include "../tqr_internal.h"

namespace tqr {

#ifdef TQR_PHASE_PROF
// panel phases of the last column block's leader (the chain that bounds the panel):
// g_phase[12] flag waits, [13] applies, [14] gather + factor, [15] publish
__device__ unsigned long long g_pphase[8];
#define TQR_PP(i) do { if (threadIdx.x == 0 && blockIdx.x == gridDim.x - 1) { long long _c = clock64(); \
    atomicAdd(&g_pphase[i], (unsigned long long)(_c - _pp)); _pp = _c; } } while (0)
#define TQR_PP0() long long _pp = clock64()
#else
#define TQR_PP(i) do {} while (0)
#define TQR_PP0() do {} while (0)
#endif

#ifdef TQR_DEBUG_WAIT
#define TQR_TRACE(...) do { if (threadIdx.x == 0) printf(__VA_ARGS__); } while (0)
#else
#define TQR_TRACE(...) do {} while (0)
#endif

// ============================================================================ panel kernel
// Grid: NBLK * (S + 1) CTAs.  For column block b: S "apply" CTAs (u = 0..S-1) own the W = IB/S
// columns [b*IB + u*W, b*IB + (u+1)*W) of every tile of panel k and apply the published
// reflector blocks b' < b of tile i to them (the chain that bounds the panel, split S ways); the
// "factor" CTA (u = S) gathers the IB columns and factors them while the apply CTAs already
// continue with tile i+1.  Flags (release/acquire): F(i, b) = block b of tile i factored,
// G(i, b, u) = sub-slice (b, u) of tile i updated.  CTA index b*(S+1) + u: a CTA waits only on
// lower-indexed CTAs, so in-order dispatch cannot deadlock.
template <int NB, int IB, int W>
__global__ void __launch_bounds__(kThreads, 1) panel_kernel(PanelArgs a) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    using SA = Smem<NB, W, IB, true>;      // apply workspace (mbarriers live here)
    using SF = Smem<NB, IB, IB, true>;     // factor workspace (same memory, used after the applies)
    auto& sa = *reinterpret_cast<SA*>(smem_raw);
    auto& sf = *reinterpret_cast<SF*>(smem_raw);
    using G = Geom<NB, IB, IB>;
    constexpr int NBLK = NB / IB;
    constexpr int S = IB / W;
    // multi-job launch (tree mode): job = domain [head, end) of the panel column, its own wavefront
    const int job = blockIdx.x / (NBLK * (S + 1));
    const int cta = blockIdx.x % (NBLK * (S + 1));
    const int b = cta / (S + 1), u = cta % (S + 1);
    const bool leader = (u == S);              // the factor CTA of block b
    const int64_t tile = (int64_t)NB * NB;
    const int head = a.L > 0 ? a.k + job * a.L : a.k;
    const int end = a.L > 0 ? min(head + a.L, a.p) : a.p;
    double* col = a.col;                       // tiles of panel column k: tile i at col + i*stride*tile
    const int st = a.stride;
    double* Akk = (a.top && job == 0) ? a.top : col + (int64_t)head * st * tile;
    double* Vexp = (head == a.k) ? a.Vexp : a.Vimg + (int64_t)head * tile;
    unsigned* F = a.flags;                                   // p * NBLK
    // G(slot, b, u) at Gf + (slot*NBLK + b)*4 + u: independent of S, so launches of one epoch with
    // different splits (the two merge levels) never alias each other's flags
    unsigned* Gf = a.flags + (int64_t)(a.fslots > 0 ? a.fslots : a.p) * NBLK;
    static_assert(S <= 4, "G flag stride");
    const int g = lane_id() >> 2, t = lane_id() & 3, wq = warp_id();
    unsigned vph = 0;
    stage_init(sa);
    TQR_PP0();

    for (int ic = head + a.skip_ge; ic < end; ++ic) {
        const int i = ic * st;                 // slot of chain index ic
        double* Ai = col + (int64_t)i * tile;
        double* Ti = a.T + (int64_t)i * IB * NB;
        const bool ge = (ic == head);
        const int c0 = b * IB + u * W;         // first column of this sub-slice
        if (!leader && b > 0) {
            Slice<NB, W, IB> X;
            X.load_cg(Ai + (int64_t)c0 * NB, NB);
            for (int bp = 0; bp < b; ++bp) {
                TQR_TRACE("cta %d (b%d u%d) tile %d wait F(%d)\n", blockIdx.x, b, u, i, bp);
                TQR_PP(1);
                flag_wait_geq(F + (int64_t)i * NBLK + bp, a.epoch);
                TQR_PP(0);
                const double* Vb = (ge ? Vexp : a.Vimg + (int64_t)i * tile) + (int64_t)bp * IB * NB;
                if (lane_id() == 0) fence_proxy_async_global();   // sibling CTA's generic stores -> bulk copy
                stage_first(sa, Vb);
                if (ge)
                    apply_block<NB, W, IB, true, true, true, true>(X, sa, Vb, Ti + (int64_t)bp * IB * IB, nullptr,
                                                                   0, bp * IB, nullptr, vph);
                else if (a.skip_ge)   // TT merge: bottom triangular, rows >= (bp+1)*IB of V and X are zero
                    apply_block<NB, W, IB, true, true, true, true>(X, sa, Vb, Ti + (int64_t)bp * IB * IB,
                                                                   Akk + (int64_t)c0 * NB + bp * IB, NB, 0,
                                                                   nullptr, vph, (bp + 1) * IB);
                else
                    apply_block<NB, W, IB, true, true, true, false>(X, sa, Vb, Ti + (int64_t)bp * IB * IB,
                                                                    Akk + (int64_t)c0 * NB + bp * IB, NB, 0,
                                                                    nullptr, vph);
            }
            X.store(Ai + (int64_t)c0 * NB, NB);
        }
        if (!leader) {
            if (b > 0) {
                __threadfence();
                __syncthreads();
                if (threadIdx.x == 0) flag_release(Gf + ((int64_t)i * NBLK + b) * 4 + u, a.epoch);
                TQR_TRACE("cta %d (b%d u%d) tile %d published G\n", blockIdx.x, b, u, i);
            }
            continue;
        }
        // ---- leader: gather the IB columns of block b and factor them
        TQR_TRACE("cta %d (b%d u%d) tile %d leader waits G\n", blockIdx.x, b, u, i);
        if (b > 0)
            for (int up = 0; up < S; ++up) flag_wait_geq(Gf + ((int64_t)i * NBLK + b) * 4 + up, a.epoch);
        TQR_TRACE("cta %d (b%d u%d) tile %d leader factors\n", blockIdx.x, b, u, i);
        TQR_PP(0);
        Slice<NB, IB, IB> Xf;
        Xf.load_cg(Ai + (int64_t)b * IB * NB, NB);
        if (ge) {
            // rare redo with scaled norms (reading Q26) from the block as loaded (nobody else writes
            // its rows >= b*IB; rows above are R, untouched by a GEQRT block)
            if (factor_block<NB, IB, true>(Xf, sf, b * IB)) {
                Xf.load_cg(Ai + (int64_t)b * IB * NB, NB);
                factor_block<NB, IB, true, true>(Xf, sf, b * IB);
            }
        } else {
            for (int idx = threadIdx.x; idx < IB * IB; idx += kThreads) {
                const int c = idx / IB, j = idx % IB;
                sf.Rsm[c * IB + j] = (j >= c) ? ld_cg(Akk + (int64_t)(b * IB + j) * NB + b * IB + c) : 0.0;
            }
            __syncthreads();
            if (factor_block<NB, IB, false>(Xf, sf, b * IB)) {
                Xf.load_cg(Ai + (int64_t)b * IB * NB, NB);
                factor_block<NB, IB, false, true>(Xf, sf, b * IB);
            }
        }
        TQR_PP(2);
        // publish: reflectors (LAPACK layout in the tile), their stage image (TSQRT: V2 of tile i;
        // GEQRT: explicit unit-lower V of the diagonal tile), the T block, the R block (TSQRT)
        // GEQRT: rows < b*IB of these columns are R rows finished by the sub-slice applies and may
        // already be updated as TS "tops" of tile k+1 by the sub-slice CTAs: store rows >= b*IB only.
        Xf.store_rows_from(Ai + (int64_t)b * IB * NB, NB, ge ? b * IB : 0);
        double* img = ge ? Vexp : a.Vimg + (int64_t)i * tile;
#pragma unroll
        for (int mf = 0; mf < IB / 8; ++mf) {
            const int cb = mf * 8 + g;                 // column within the block
            const int dc = b * IB + cb;                // column within the tile
#pragma unroll
            for (int nf = 0; nf < G::NF; ++nf) {
                const int rl = nf * 8 + 2 * t;         // row within this warp's rows
                const int r = wq * G::RW + rl;
                double v0 = Xf.acc[mf][nf][0], v1 = Xf.acc[mf][nf][1];
                if (ge) {
                    v0 = (r > dc) ? v0 : (r == dc ? 1.0 : 0.0);
                    v1 = (r + 1 > dc) ? v1 : (r + 1 == dc ? 1.0 : 0.0);
                }
                st2(img + vimg_off<NB, IB, IB>(b, wq, cb / G::HC, rl, cb % G::HC), v0, v1);
            }
        }
        if (!ge) {
            for (int idx = threadIdx.x; idx < IB * IB; idx += kThreads) {
                const int j = idx / IB, c = idx % IB;
                if (c <= j) Akk[(int64_t)(b * IB + j) * NB + b * IB + c] = sf.Rsm[c * IB + j];
            }
        }
        build_T<NB, IB>(sf);
        for (int idx = threadIdx.x; idx < IB * IB; idx += kThreads) {
            const int c = idx / IB, r = idx % IB;   // T(r, c) -> column-major block b
            Ti[(int64_t)b * IB * IB + c * IB + r] = sf.Tsm[r * IB + c];
        }
        fence_proxy_async_global();
        __threadfence();
        __syncthreads();
        if (threadIdx.x == 0) flag_release(F + (int64_t)i * NBLK + b, a.epoch);
        TQR_TRACE("cta %d (b%d u%d) tile %d published F\n", blockIdx.x, b, u, i);
        TQR_PP(3);
    }
}

// ============================================================================ domain kernel
// TS-domain factorisation (tree mode): one CTA per domain, which runs the whole GEQRT(head) +
// TSQRT(i, head) chain of its tiles alone -- per tile and ib column block b: the block's NB x IB
// columns in registers, the b earlier reflector blocks of the same tile applied (apply_block,
// DMMA), then factor_block -- with no inter-CTA flags.  Many domains run at once (one per SM),
// which is what the flat chain of a tall panel lacks (C4: parallelism 1).
template <int NB, int IB>
__global__ void __launch_bounds__(kThreads, 1) domain_kernel(DomainArgs a) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    auto& sf = *reinterpret_cast<Smem<NB, IB, IB, true>*>(smem_raw);
    using G = Geom<NB, IB, IB>;
    constexpr int NBLK = NB / IB;
    const int64_t tile = (int64_t)NB * NB;
    const int head = a.k + (a.dom0 + (int)blockIdx.x) * a.L;
    const int end = min(head + a.L, a.p);
    double* Ah = a.col + (int64_t)head * tile;
    double* himg = (head == a.k) ? a.Vexp : a.Vimg + (int64_t)head * tile;
    const int g = lane_id() >> 2, t = lane_id() & 3, wq = warp_id();
    unsigned vph = 0;
    stage_init(sf);
    TQR_PP0();
    for (int i = head; i < end; ++i) {
        double* Ai = a.col + (int64_t)i * tile;
        double* Ti = a.T + (int64_t)i * IB * NB;
        const bool ge = (i == head);
        double* img = ge ? himg : a.Vimg + (int64_t)i * tile;
        for (int b = 0; b < NBLK; ++b) {
            Slice<NB, IB, IB> X;
            X.load_cg(Ai + (int64_t)b * IB * NB, NB);
            for (int bp = 0; bp < b; ++bp) {
                const double* Vb = img + (int64_t)bp * IB * NB;
                const double* nxt = (bp + 1 < b) ? img + (int64_t)(bp + 1) * IB * NB : nullptr;
                if (bp == 0) {
                    if (lane_id() == 0) fence_proxy_async_global();   // this CTA's image stores -> bulk copy
                    stage_first(sf, Vb);
                }
                if (ge)
                    apply_block<NB, IB, IB, true, true, true, true>(X, sf, Vb, Ti + (int64_t)bp * IB * IB, nullptr, 0,
                                                                   bp * IB, nxt, vph);
                else
                    apply_block<NB, IB, IB, true, true, true, false>(X, sf, Vb, Ti + (int64_t)bp * IB * IB,
                                                                    Ah + (int64_t)b * IB * NB + bp * IB, NB, 0, nxt,
                                                                    vph);
            }
            __syncthreads();   // top rows written by the applies -> Rsm reads below
            TQR_PP(4);
            // X (after the applies) is kept in the idle staging area for the rare scaled redo (Q26)
            double* keep = &sf.Vst[0][0][0][0];
            static_assert(sizeof(sf.Vst) / sizeof(double) >= NB * IB, "redo copy of the block");
#pragma unroll
            for (int mf = 0; mf < IB / 8; ++mf)
#pragma unroll
                for (int nf = 0; nf < G::NF; ++nf) {
                    keep[((mf * G::NF + nf) * 2 + 0) * kThreads + threadIdx.x] = X.acc[mf][nf][0];
                    keep[((mf * G::NF + nf) * 2 + 1) * kThreads + threadIdx.x] = X.acc[mf][nf][1];
                }
            auto restore = [&]() {
#pragma unroll
                for (int mf = 0; mf < IB / 8; ++mf)
#pragma unroll
                    for (int nf = 0; nf < G::NF; ++nf) {
                        X.acc[mf][nf][0] = keep[((mf * G::NF + nf) * 2 + 0) * kThreads + threadIdx.x];
                        X.acc[mf][nf][1] = keep[((mf * G::NF + nf) * 2 + 1) * kThreads + threadIdx.x];
                    }
            };
            if (ge) {
                if (factor_block<NB, IB, true>(X, sf, b * IB)) {
                    restore();
                    factor_block<NB, IB, true, true>(X, sf, b * IB);
                }
            } else {
                for (int idx = threadIdx.x; idx < IB * IB; idx += kThreads) {
                    const int c = idx / IB, j = idx % IB;
                    sf.Rsm[c * IB + j] = (j >= c) ? ld_cg(Ah + (int64_t)(b * IB + j) * NB + b * IB + c) : 0.0;
                }
                __syncthreads();
                if (factor_block<NB, IB, false>(X, sf, b * IB)) {
                    restore();
                    factor_block<NB, IB, false, true>(X, sf, b * IB);
                }
            }
            TQR_PP(5);
            X.store(Ai + (int64_t)b * IB * NB, NB);
#pragma unroll
            for (int mf = 0; mf < IB / 8; ++mf) {
                const int cb = mf * 8 + g;
                const int dc = b * IB + cb;
#pragma unroll
                for (int nf = 0; nf < G::NF; ++nf) {
                    const int rl = nf * 8 + 2 * t;
                    const int r = wq * G::RW + rl;
                    double v0 = X.acc[mf][nf][0], v1 = X.acc[mf][nf][1];
                    if (ge) {
                        v0 = (r > dc) ? v0 : (r == dc ? 1.0 : 0.0);
                        v1 = (r + 1 > dc) ? v1 : (r + 1 == dc ? 1.0 : 0.0);
                    }
                    st2(img + vimg_off<NB, IB, IB>(b, wq, cb / G::HC, rl, cb % G::HC), v0, v1);
                }
            }
            if (!ge) {
                for (int idx = threadIdx.x; idx < IB * IB; idx += kThreads) {
                    const int j = idx / IB, c = idx % IB;
                    if (c <= j) Ah[(int64_t)(b * IB + j) * NB + b * IB + c] = sf.Rsm[c * IB + j];
                }
            }
            build_T<NB, IB>(sf);
            for (int idx = threadIdx.x; idx < IB * IB; idx += kThreads) {
                const int c = idx / IB, r = idx % IB;
                Ti[(int64_t)b * IB * IB + c * IB + r] = sf.Tsm[r * IB + c];
            }
            __threadfence_block();
            __syncthreads();
            TQR_PP(6);
        }
    }
}

// Mt[e] = triu(tile k + e*L of the column), zeros below the diagonal (e = 1..ndom-1): the dense
// "bottom" of merge e, factored against the head tile k by the panel kernel (skip_ge).
__global__ void merge_prep_kernel(const double* __restrict__ col, double* __restrict__ Mt, int nb, int k, int L) {
    const int e = blockIdx.y + 1;
    const int64_t tile = (int64_t)nb * nb;
    const double* s = col + (int64_t)(k + e * L) * tile;
    double* d = Mt + (int64_t)e * tile;
    for (int64_t x = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; x < tile; x += (int64_t)gridDim.x * blockDim.x) {
        const int c = (int)(x / nb), r = (int)(x % nb);
        d[x] = (r <= c) ? s[x] : 0.0;
    }
}

// ============================================================================ update kernel
// Forward (TRANS = true, Q^T): for each slice: [UNMQR on row tile k]; for i = k+1..p-1 TSMQR.
// Backward (TRANS = false, Q):  for i = p-1..k+1 TSMQR (blocks descending); then UNMQR.
template <int NB, int W, int IB, bool TRANS>
__global__ void __launch_bounds__(kThreads, 1) update_kernel(UpdateArgs a) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    auto& sm = *reinterpret_cast<Smem<NB, W, IB, false>*>(smem_raw);
    constexpr int SPG = NB / W;     // slices per column group
    constexpr int NBLK = NB / IB;
    // wavefront apply (nsteps > 1): CTA = (step offset st, slice); step k = a.k +- st with its own
    // reflector column (V, T, Vexp + k * column strides); tile i of step k waits until the
    // previous step's CTA of the same slice has finished tile i (progress flags, lower CTA index)
    // tree jobs (domL > 0): CTA = (job d, slice); job d is the chain of row tiles
    // [k + d*domL, min(k + (d+1)*domL, p)) against its own head (the TS domains of a tree panel,
    // or the level-1 merge groups over merge slots) -- independent row ranges, one launch
    const bool jobs = a.domL > 0;
    const int st = a.nsteps > 1 ? (int)(blockIdx.x / a.nslc) : 0;
    const int jd = jobs ? (int)(blockIdx.x / a.nslc) : 0;
    const int bid = (a.nsteps > 1 || jobs) ? (int)(blockIdx.x % a.nslc) : (int)blockIdx.x;
    const int k = jobs ? a.k + jd * a.domL : (TRANS ? a.k + st : a.k - st);
    const int pend = jobs ? min(k + a.domL, a.p) : a.p;
    const double* __restrict__ Vb = a.V + (int64_t)st * (TRANS ? 1 : -1) * a.vcol;
    const double* __restrict__ Tb = a.T + (int64_t)st * (TRANS ? 1 : -1) * a.tcol;
    const double* __restrict__ Eb = (jobs && jd > 0) ? a.V + (int64_t)k * a.vstride * NB * NB
                                                     : a.Vexp + (int64_t)st * (TRANS ? 1 : -1) * a.ecol;
    const int grp = bid / SPG;
    const int c0 = (bid % SPG) * W;
    double* Xg = a.X + (int64_t)(a.group0 + grp * a.gstride) * a.col_stride + (int64_t)c0 * a.ld;
    double* Xk = Xg + (int64_t)k * a.tile_stride;
    const int64_t vtile = (int64_t)NB * NB;
    Slice<NB, W, IB> X;
    stage_init(sm);
    unsigned vph = 0;

    // Reflector blocks in application order; block q of the sequence is staged (cp.async) while
    // block q-1's GEMM2 runs.  Forward: UNMQR blocks 0..NBLK-1, then for i = k+1..p-1 blocks
    // 0..NBLK-1 of V_i.  Backward: i = p-1..k+1 blocks NBLK-1..0, then UNMQR blocks NBLK-1..0.
    const int ntiles = pend - k - 1 + (a.do_unmqr ? 1 : 0);
    auto tile_of = [&](int q) -> int {            // q-th tile of the sequence; -1 = UNMQR (row tile k)
        if (TRANS) return a.do_unmqr ? (q == 0 ? -1 : k + q) : k + 1 + q;
        return (q < pend - k - 1) ? pend - 1 - q : -1;
    };
    auto vblock = [&](int ti, int s) -> const double* {
        return (ti < 0 ? Eb : Vb + (int64_t)ti * a.vstride * vtile) + (int64_t)s * IB * NB;
    };
    // progress of the previous step's CTA needed before row tile ti: forward, the previous step
    // (k-1) runs k-1, k, k+1, ..; backward (Q), the previous step (k+1) runs p-1, .., k+1
    auto wait_prev = [&](int ti) {
        if (st > 0 && !(!TRANS && ti < 0)) {      // backward UNMQR row k: untouched by step k+1
            const int row = ti < 0 ? k : ti;
            const unsigned need = TRANS ? (unsigned)(row - k + 2) : (unsigned)(a.p - row);
            flag_wait_geq(a.prog + (int64_t)(st - 1) * a.nslc + bid, need);
        }
    };
    auto blk = [&](int si) { return TRANS ? si : NBLK - 1 - si; };
    auto wait_tile = [&](int ti) {   // lookahead overlapped with the panel: tile ti published?
        if (a.wflags) {
            flag_wait_geq(a.wflags + (int64_t)(ti < 0 ? k : ti) * NBLK + NBLK - 1, a.wepoch);
            if (lane_id() == 0) fence_proxy_async_global();   // panel's generic stores -> bulk copies
        }
        if (a.cflags) {                  // trailing a remote panel: tile ti's chunk landed in the slot?
            const unsigned long long* f = a.cflags + ((ti < 0 ? k : ti) - k) / a.cchunk;
            if (threadIdx.x == 0) {
                for (;;) {
                    unsigned long long x;
                    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(x) : "l"(f) : "memory");
                    if ((long long)(x - a.cval) >= 0) break;
                    __nanosleep(128);
                }
                fence_proxy_async_global();
            }
            __syncthreads();
        }
    };
    if (ntiles > 0) {
        wait_tile(tile_of(0));
        stage_first(sm, vblock(tile_of(0), blk(0)));
    }
    for (int q = 0; q < ntiles; ++q) {
        const int ti = tile_of(q);
        double* Xi = (ti < 0) ? Xk : Xg + (int64_t)ti * a.tile_stride;
        const double* Tt = Tb + (int64_t)(ti < 0 ? k : ti * a.vstride) * IB * NB;
        if (a.nsteps > 1) {
            wait_prev(ti);
            X.load_cg(Xi, a.ld);     // written by another CTA: L2, not a stale L1 line
        } else {
            X.load(Xi, a.ld);
        }
        for (int si = 0; si < NBLK; ++si) {
            const int s = blk(si);
            const double* nxt = nullptr;
            if (si + 1 < NBLK) nxt = vblock(ti, blk(si + 1));
            else if (q + 1 < ntiles) {
                wait_tile(tile_of(q + 1));
                nxt = vblock(tile_of(q + 1), blk(0));
            }
            if (ti < 0)
                apply_block<NB, W, IB, false, TRANS, false, true>(X, sm, vblock(ti, s), Tt + (int64_t)s * IB * IB,
                                                                  nullptr, a.ld, s * IB, nxt, vph);
            else
                apply_block<NB, W, IB, false, TRANS, false, false>(X, sm, vblock(ti, s), Tt + (int64_t)s * IB * IB,
                                                                   Xk + s * IB, a.ld, 0, nxt, vph);
        }
        X.store(Xi, a.ld);
        if (a.nsteps > 1) __threadfence();
        __syncthreads();   // row tile k (the TS "top") is re-read by other threads
        if (a.nsteps > 1 && threadIdx.x == 0) flag_release(a.prog + (int64_t)st * a.nslc + bid, (unsigned)(q + 1));
    }
}

// ============================================================================ 16-warp bulk update
// update_kernel's Q^T chain with the 32-column slice split over 16 warps (tile_w16.cuh): plain
// launches and the forward wavefront of tqr_apply_qt (nsteps > 1: CTA = (step offset, slice), tile i
// of step k only after the step-(k-1) CTA of the same slice has finished it; progress flags, lower
// CTA index, so in-order dispatch cannot deadlock).  No jobs, no lookahead flags.
template <int NB, int IB>
__global__ void __launch_bounds__(kThreads16, 1) update_kernel16(UpdateArgs a) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    auto& sm = *reinterpret_cast<Smem16<NB, IB>*>(smem_raw);
    constexpr int SPG = NB / 32, NBLK = NB / IB;
    const int st = a.nsteps > 1 ? (int)(blockIdx.x / a.nslc) : 0;
    const int bid = a.nsteps > 1 ? (int)(blockIdx.x % a.nslc) : (int)blockIdx.x;
    const int k = a.k + st;
    const double* __restrict__ Vb = a.V + (int64_t)st * a.vcol;
    const double* __restrict__ Tb = a.T + (int64_t)st * a.tcol;
    const double* __restrict__ Eb = a.Vexp + (int64_t)st * a.ecol;
    const int grp = bid / SPG, c0 = (bid % SPG) * 32;
    double* Xg = a.X + (int64_t)(a.group0 + grp * a.gstride) * a.col_stride + (int64_t)c0 * a.ld;
    double* Xk = Xg + (int64_t)k * a.tile_stride;
    const int64_t vtile = (int64_t)NB * NB;
    if (warp_id() < 8 && lane_id() == 0) {
        mbar_init(&sm.mbar[warp_id()][0], 1);
        mbar_init(&sm.mbar[warp_id()][1], 1);
        fence_mbar_init();
    }
    __syncthreads();
    unsigned vph = 0;
    const int ntiles = a.p - k - 1 + (a.do_unmqr ? 1 : 0);
    auto tile_of = [&](int q) -> int { return a.do_unmqr ? (q == 0 ? -1 : k + q) : k + 1 + q; };
    auto vblock = [&](int ti, int s) -> const double* {
        return (ti < 0 ? Eb : Vb + (int64_t)ti * a.vstride * vtile) + (int64_t)s * IB * NB;
    };
    Slice16<NB, IB> X;
    if (ntiles > 0) stage16(sm, vblock(tile_of(0), 0), 0);
    for (int q = 0; q < ntiles; ++q) {
        const int ti = tile_of(q);
        double* Xi = (ti < 0) ? Xk : Xg + (int64_t)ti * a.tile_stride;
        const double* Tt = Tb + (int64_t)(ti < 0 ? k : ti * a.vstride) * IB * NB;
        if (a.nsteps > 1) {
            if (st > 0) flag_wait_geq(a.prog + (int64_t)(st - 1) * a.nslc + bid, (unsigned)((ti < 0 ? k : ti) - k + 2));
            X.load_cg(Xi, a.ld);   // written by another CTA: L2, not a stale L1 line
        } else {
            X.load(Xi, a.ld);
        }
        for (int s = 0; s < NBLK; ++s) {
            const double* nxt = nullptr;
            if (s + 1 < NBLK) nxt = vblock(ti, s + 1);
            else if (q + 1 < ntiles) nxt = vblock(tile_of(q + 1), 0);
            if (ti < 0)
                apply_block16<NB, IB, true>(X, sm, vblock(ti, s), Tt + (int64_t)s * IB * IB, nullptr, a.ld, s * IB,
                                            nxt, vph);
            else
                apply_block16<NB, IB, false>(X, sm, vblock(ti, s), Tt + (int64_t)s * IB * IB, Xk + s * IB, a.ld, 0,
                                             nxt, vph);
        }
        X.store(Xi, a.ld);
        if (a.nsteps > 1) __threadfence();
        __syncthreads();   // row tile k (the X1 rows) is re-read by other threads
        if (a.nsteps > 1 && threadIdx.x == 0) flag_release(a.prog + (int64_t)st * a.nslc + bid, (unsigned)(q + 1));
    }
}

// ============================================================================ layout kernels
// a1: column-major source -> tile-major column storage, zero-padded to whole tiles (rows >= m_valid
// and global columns >= n_valid are written as 0: a padded zero column gets tau = 0 and padded zero
// rows stay zero under every reflector, so Q = diag(Q_m, I) and R(0:n, 0:n) is unchanged).
// Source group of local column lc at src + (local_src ? lc : cols[lc])*src_group_stride (ld = lda);
// destination tile i of local column lc at dst + lc*dst_col_stride + i*nb*nb, element (r, c) at
// + c*nb + r.  blockIdx.x = chunk*nb + c, blockIdx.y = lc.  VEC elements per 16-byte access when
// lda, the group stride, m_valid and the pointer allow it: a warp moves 512 contiguous bytes per
// instruction on both sides.
template <class T, int VEC>
__global__ void to_tiles_kernel(const T* __restrict__ src, int64_t lda, int64_t src_group_stride,
                                T* __restrict__ dst, const int32_t* __restrict__ cols, int local_src,
                                int64_t dst_col_stride, int nb, int p, int64_t m_valid, int64_t n_valid) {
    using V = typename std::conditional<VEC == 1, T, typename std::conditional<sizeof(T) == 8, double2, float4>::type>::type;
    const int lc = blockIdx.y;
    const int c = blockIdx.x % nb;
    const int chunk = blockIdx.x / nb, nchunk = gridDim.x / nb;
    const int64_t gcol = (int64_t)cols[lc] * nb + c;
    const bool colv = gcol < n_valid;
    const T* s = src + (int64_t)(local_src ? lc : cols[lc]) * src_group_stride + (int64_t)c * lda;
    T* d = dst + (int64_t)lc * dst_col_stride + (int64_t)c * nb;
    const int64_t tile = (int64_t)nb * nb;
    const int64_t m = (int64_t)p * nb;
    for (int64_t r = VEC * ((int64_t)chunk * blockDim.x + threadIdx.x); r < m; r += VEC * (int64_t)nchunk * blockDim.x) {
        V v{};
        if (colv && r < m_valid) v = __ldcs(reinterpret_cast<const V*>(s + r));
        *reinterpret_cast<V*>(d + (r / nb) * tile + (r % nb)) = v;
    }
}

// a8: tile-major -> column-major rows [0, m_rows) of the global columns < n_valid: R on and above
// the diagonal, 0 below.  Destination group at dst + (local_dst ? lc : cols[lc])*dst_group_stride.
template <class T, int VEC>
__global__ void from_tiles_kernel(T* __restrict__ dst, int64_t lda, int64_t dst_group_stride,
                                  const T* __restrict__ src, const int32_t* __restrict__ cols,
                                  int64_t src_col_stride, int nb, int64_t m_rows, int64_t n_valid, int local_dst) {
    const int lc = blockIdx.y;
    const int c = blockIdx.x % nb;
    const int chunk = blockIdx.x / nb, nchunk = gridDim.x / nb;
    const int64_t gcol = (int64_t)cols[lc] * nb + c;
    if (gcol >= n_valid) return;
    T* d = dst + (int64_t)(local_dst ? lc : cols[lc]) * dst_group_stride + (int64_t)c * lda;
    const T* s = src + (int64_t)lc * src_col_stride + (int64_t)c * nb;
    const int64_t tile = (int64_t)nb * nb;
    for (int64_t r = VEC * ((int64_t)chunk * blockDim.x + threadIdx.x); r < m_rows; r += VEC * (int64_t)nchunk * blockDim.x) {
        T v[VEC];
#pragma unroll
        for (int e = 0; e < VEC; ++e) v[e] = T(0);
        if (r <= gcol) {
            if constexpr (VEC == 1) {
                v[0] = s[(r / nb) * tile + (r % nb)];
            } else {
                const T* sp = s + (r / nb) * tile + (r % nb);
#pragma unroll
                for (int e = 0; e < VEC; ++e) v[e] = (r + e <= gcol) ? sp[e] : T(0);
            }
        }
        if constexpr (VEC == 1) {
            d[r] = v[0];
        } else if constexpr (sizeof(T) == 8) {
            __stcs(reinterpret_cast<double2*>(d + r), make_double2(v[0], v[1]));
        } else {
            __stcs(reinterpret_cast<float4*>(d + r), make_float4(v[0], v[1], v[2], v[3]));
        }
    }
}

// Row-split stage 2 input: the stacked R_g blocks (nb rows each, ld) keep only their upper
// triangles: entry (r, c) with r % nb > c is zeroed (the reflectors stored below R_g's diagonal).
template <class T>
__global__ void zero_below_blocks_kernel(T* __restrict__ a, int64_t ld, int64_t rows, int64_t cols, int nb) {
    const int64_t tot = rows * cols;
    for (int64_t x = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; x < tot; x += (int64_t)gridDim.x * blockDim.x) {
        const int64_t c = x / rows, r = x % rows;
        if (r % nb > c) a[c * ld + r] = T(0);
    }
}

// ============================================================================ launchers
template <int NB, int IB, int W>
static cudaError_t launch_panel_t(const PanelArgs& a, cudaStream_t s, int njobs) {
    const size_t smem = std::max(sizeof(Smem<NB, IB, IB, true>), sizeof(Smem<NB, W, IB, true>));
    auto kern = panel_kernel<NB, IB, W>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    kern<<<njobs * (NB / IB) * (IB / W + 1), kThreads, smem, s>>>(a);
    return cudaGetLastError();
}

template <int NB, int W, int IB>
static cudaError_t launch_update_t(const UpdateArgs& a, int nslices, bool trans, cudaStream_t s) {
    const size_t smem = sizeof(Smem<NB, W, IB, false>);
    const int grid = nslices;
    if (grid <= 0) return cudaSuccess;
    if constexpr (W == 32 && NB >= 256) {
        // 16 warps per CTA for the Q^T chain, plain or wavefront (C5 1629 -> 1592 ms, C3 229 -> 225 ms)
        if (a.w16 && trans && a.domL == 0 && !a.wflags && !a.cflags) {
            const size_t sm16 = sizeof(Smem16<NB, IB>);
            auto kern = update_kernel16<NB, IB>;
            cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm16);
            if (e != cudaSuccess) return e;
            kern<<<grid, kThreads16, sm16, s>>>(a);
            return cudaGetLastError();
        }
    }
    if (trans) {
        auto kern = update_kernel<NB, W, IB, true>;
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        kern<<<grid, kThreads, smem, s>>>(a);
    } else {
        auto kern = update_kernel<NB, W, IB, false>;
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        kern<<<grid, kThreads, smem, s>>>(a);
    }
    return cudaGetLastError();
}

#define TQR_NBIB_DISPATCH(NB_, IB_, CALL)                              \
    if (nb == NB_ && ib == IB_) { return CALL; }

template <int NB, int IB, int W>
static cudaError_t launch_panel_chk(const PanelArgs& a, cudaStream_t s, int njobs) {
    if constexpr (W >= 8) return launch_panel_t<NB, IB, W>(a, s, njobs);
    else return cudaErrorInvalidValue;
}

// split: sub-slices per ib column block (1, 2 or 4; W = ib / split >= 8)
cudaError_t launch_panel(int nb, int ib, int split, const PanelArgs& a, cudaStream_t s, int njobs) {
#define TQR_PAN(NB_, IB_)                                                          \
    if (nb == NB_ && ib == IB_) {                                                  \
        if (split == 1) return launch_panel_chk<NB_, IB_, IB_>(a, s, njobs);      \
        if (split == 2) return launch_panel_chk<NB_, IB_, IB_ / 2>(a, s, njobs);  \
        if (split == 4) return launch_panel_chk<NB_, IB_, IB_ / 4>(a, s, njobs);  \
        return cudaErrorInvalidValue;                                              \
    }
    TQR_PAN(64, 16) TQR_PAN(64, 32) TQR_PAN(128, 16) TQR_PAN(128, 32)
    TQR_PAN(256, 16) TQR_PAN(256, 32) TQR_PAN(512, 16) TQR_PAN(512, 32)
#undef TQR_PAN
    return cudaErrorInvalidValue;
}

template <int NB, int IB>
static cudaError_t launch_domains_t(const DomainArgs& a, int ndom, cudaStream_t s) {
    const size_t smem = sizeof(Smem<NB, IB, IB, true>);
    auto kern = domain_kernel<NB, IB>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    kern<<<ndom, kThreads, smem, s>>>(a);
    return cudaGetLastError();
}

cudaError_t launch_domains(int nb, int ib, const DomainArgs& a, int ndom, cudaStream_t s) {
    if (ndom <= 0) return cudaSuccess;
#define TQR_DOM(NB_, IB_) if (nb == NB_ && ib == IB_) return launch_domains_t<NB_, IB_>(a, ndom, s);
    TQR_DOM(64, 16) TQR_DOM(64, 32) TQR_DOM(128, 16) TQR_DOM(128, 32)
    TQR_DOM(256, 16) TQR_DOM(256, 32) TQR_DOM(512, 16) TQR_DOM(512, 32)
#undef TQR_DOM
    return cudaErrorInvalidValue;
}

cudaError_t launch_merge_prep(int nb, const double* col, double* Mt, int k, int L, int ndom, cudaStream_t s) {
    if (ndom <= 1) return cudaSuccess;
    dim3 grid(std::max(1, std::min(64, nb * nb / 2048)), ndom - 1);
    merge_prep_kernel<<<grid, 256, 0, s>>>(col, Mt, nb, k, L);
    return cudaGetLastError();
}

// w: slice width (8, 16, 32).  Narrow slices raise CTA count for the lookahead column.
cudaError_t launch_update(int nb, int ib, int w, const UpdateArgs& a, int nslices, bool trans, cudaStream_t s) {
#define TQR_UPD(NB_, IB_)                                                                 \
    if (nb == NB_ && ib == IB_) {                                                         \
        if (w == 8) return launch_update_t<NB_, 8, IB_>(a, nslices, trans, s);            \
        if (w == 16) return launch_update_t<NB_, 16, IB_>(a, nslices, trans, s);          \
        if (w == 32) return launch_update_t<NB_, 32, IB_>(a, nslices, trans, s);          \
        return cudaErrorInvalidValue;                                                     \
    }
    TQR_UPD(64, 16)
    TQR_UPD(64, 32)
    TQR_UPD(128, 16)
    TQR_UPD(128, 32)
    TQR_UPD(256, 16)
    TQR_UPD(256, 32)
    TQR_UPD(512, 16)
    TQR_UPD(512, 32)
#undef TQR_UPD
    return cudaErrorInvalidValue;
}

static int layout_chunks(int64_t m, int vec, int threads) {
    int64_t chunks = (m / vec + threads - 1) / threads;
    return (int)(chunks > 16 ? 16 : (chunks < 1 ? 1 : chunks));
}

template <class T>
cudaError_t launch_to_tiles(const T* src, int64_t lda, int64_t src_group_stride, T* dst, const int32_t* cols_dev,
                            int local_src, int ncols, int64_t dst_col_stride, int nb, int p, int64_t m_valid,
                            int64_t n_valid, cudaStream_t s) {
    if (ncols <= 0) return cudaSuccess;
    constexpr int VEC = 16 / sizeof(T);
    const bool vec = (lda % VEC) == 0 && (src_group_stride % VEC) == 0 && (m_valid % VEC) == 0 &&
                     (((uintptr_t)src) % 16) == 0;
    const int threads = 256;
    dim3 grid(nb * layout_chunks((int64_t)p * nb, vec ? VEC : 1, threads), ncols);
    if (vec)
        to_tiles_kernel<T, VEC><<<grid, threads, 0, s>>>(src, lda, src_group_stride, dst, cols_dev, local_src,
                                                        dst_col_stride, nb, p, m_valid, n_valid);
    else
        to_tiles_kernel<T, 1><<<grid, threads, 0, s>>>(src, lda, src_group_stride, dst, cols_dev, local_src,
                                                      dst_col_stride, nb, p, m_valid, n_valid);
    return cudaGetLastError();
}

template <class T>
cudaError_t launch_from_tiles(T* dst, int64_t lda, int64_t dst_group_stride, const T* src, const int32_t* cols_dev,
                              int ncols, int64_t src_col_stride, int nb, int64_t m_rows, int64_t n_valid,
                              int local_dst, cudaStream_t s) {
    if (ncols <= 0 || m_rows <= 0) return cudaSuccess;
    constexpr int VEC = 16 / sizeof(T);
    const bool vec = (lda % VEC) == 0 && (dst_group_stride % VEC) == 0 && (m_rows % VEC) == 0 &&
                     (((uintptr_t)dst) % 16) == 0;
    const int threads = 256;
    dim3 grid(nb * layout_chunks(m_rows, vec ? VEC : 1, threads), ncols);
    if (vec)
        from_tiles_kernel<T, VEC><<<grid, threads, 0, s>>>(dst, lda, dst_group_stride, src, cols_dev, src_col_stride,
                                                          nb, m_rows, n_valid, local_dst);
    else
        from_tiles_kernel<T, 1><<<grid, threads, 0, s>>>(dst, lda, dst_group_stride, src, cols_dev, src_col_stride,
                                                        nb, m_rows, n_valid, local_dst);
    return cudaGetLastError();
}
template cudaError_t launch_to_tiles<double>(const double*, int64_t, int64_t, double*, const int32_t*, int, int,
                                             int64_t, int, int, int64_t, int64_t, cudaStream_t);
template cudaError_t launch_to_tiles<float>(const float*, int64_t, int64_t, float*, const int32_t*, int, int,
                                            int64_t, int, int, int64_t, int64_t, cudaStream_t);
template cudaError_t launch_from_tiles<double>(double*, int64_t, int64_t, const double*, const int32_t*, int,
                                               int64_t, int, int64_t, int64_t, int, cudaStream_t);
template cudaError_t launch_from_tiles<float>(float*, int64_t, int64_t, const float*, const int32_t*, int,
                                              int64_t, int, int64_t, int64_t, int, cudaStream_t);

template <class T>
cudaError_t launch_zero_below_blocks(T* a, int64_t ld, int64_t rows, int64_t cols, int nb, cudaStream_t s) {
    if (rows <= 0 || cols <= 0) return cudaSuccess;
    const int grid = (int)std::min<int64_t>((rows * cols + 255) / 256, 148 * 8);
    zero_below_blocks_kernel<T><<<grid, 256, 0, s>>>(a, ld, rows, cols, nb);
    return cudaGetLastError();
}
template cudaError_t launch_zero_below_blocks<double>(double*, int64_t, int64_t, int64_t, int, cudaStream_t);
template cudaError_t launch_zero_below_blocks<float>(float*, int64_t, int64_t, int64_t, int, cudaStream_t);

size_t panel_smem_bytes(int nb, int ib) {
#define TQR_PS(NB_, IB_) if (nb == NB_ && ib == IB_) return sizeof(Smem<NB_, IB_, IB_, true>);
    TQR_PS(64, 16) TQR_PS(64, 32) TQR_PS(128, 16) TQR_PS(128, 32)
    TQR_PS(256, 16) TQR_PS(256, 32) TQR_PS(512, 16) TQR_PS(512, 32)
#undef TQR_PS
    return 0;
}

size_t update_smem_bytes(int nb, int ib, int w) {
#define TQR_US(NB_, IB_) if (nb == NB_ && ib == IB_) { \
        if (w == 8) return sizeof(Smem<NB_, 8, IB_, false>); \
        if (w == 16) return sizeof(Smem<NB_, 16, IB_, false>); \
        if (w == 32) return sizeof(Smem<NB_, 32, IB_, false>); }
    TQR_US(64, 16) TQR_US(64, 32) TQR_US(128, 16) TQR_US(128, 32)
    TQR_US(256, 16) TQR_US(256, 32) TQR_US(512, 16) TQR_US(512, 32)
#undef TQR_US
    return 0;
}

}  // namespace tqr

#ifdef TQR_PHASE_PROF
extern "C" int tqr_probe_phases(unsigned long long* out, int reset) {
    cudaMemcpyFromSymbol(out, tqr::g_phase, sizeof(unsigned long long) * 16);
    cudaMemcpyFromSymbol(out + 16, tqr::g_pphase, sizeof(unsigned long long) * 8);
    cudaMemcpyFromSymbol(out + 24, tqr::g_fphase, sizeof(unsigned long long) * 4);
    cudaMemcpyFromSymbol(out + 28, tqr::g_cphase, sizeof(unsigned long long) * 8);
    if (reset) {
        unsigned long long z[16] = {0};
        cudaMemcpyToSymbol(tqr::g_phase, z, sizeof(z));
        cudaMemcpyToSymbol(tqr::g_pphase, z, sizeof(unsigned long long) * 8);
        cudaMemcpyToSymbol(tqr::g_fphase, z, sizeof(unsigned long long) * 4);
        cudaMemcpyToSymbol(tqr::g_cphase, z, sizeof(unsigned long long) * 8);
    }
    return (int)cudaGetLastError();
}
#endif

// Every instantiated workspace must fit the sm_100a opt-in limit of 227 KB dynamic smem per CTA.
namespace tqr {
constexpr size_t kMaxSmem = 232448;
#define TQR_FITS(NB_, IB_)                                                             \
    static_assert(sizeof(Smem<NB_, IB_, IB_, true>) <= kMaxSmem, "panel smem");        \
    static_assert(sizeof(Smem<NB_, IB_ / 2, IB_, true>) <= kMaxSmem, "panel smem S=2"); \
    static_assert(sizeof(Smem<NB_, 8, IB_, false>) <= kMaxSmem, "update smem W=8");    \
    static_assert(sizeof(Smem<NB_, 16, IB_, false>) <= kMaxSmem, "update smem W=16");  \
    static_assert(sizeof(Smem<NB_, 32, IB_, false>) <= kMaxSmem, "update smem W=32");
TQR_FITS(64, 16) TQR_FITS(64, 32) TQR_FITS(128, 16) TQR_FITS(128, 32)
TQR_FITS(256, 16) TQR_FITS(256, 32) TQR_FITS(512, 16) TQR_FITS(512, 32)
#undef TQR_FITS
}  // namespace tqr
