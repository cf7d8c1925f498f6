// tile_ops_tf32.cuh -- FP32 block-reflector apply on the tensor cores with split TF32 ("3xTF32").
//
// The FP32 trailing update (UNMQR, Eq. 6; TSMQR, Eq. 9, applied as Q^T -- reading Q5) with the same
// register-resident structure as the FP64 DMMA path (tile_ops.cuh), on legacy mma.sync
// m16n8k8 TF32 (measured 277.6 TFLOP/s on this pool's B200 vs 72.5 for FFMA): every FP32 operand
// x is split x = hi + lo with hi = rna_tf32(x), lo = x - hi, and a product is formed as
// lo_a*hi_b + hi_a*lo_b + hi_a*hi_b with FP32 accumulation (the dropped lo*lo term and the TF32
// truncation of lo are ~2^-22 relative: FP32-level accuracy, unlike plain TF32's 2^-11).
//
// Register layout ("transposed accumulator", as common.cuh for FP64): warp q owns rows
// q*RW .. q*RW + RW - 1 of the NB x W slice X; acc[mf][nf][e] is the m16n8 C fragment of X^T
// (m = column mf*16 + g (+8 for e >= 2), n = row nf*8 + 2t + (e & 1)).  With the K index of GEMM1
// permuted (k = t <-> row 2t, k = t + 4 <-> row 2t + 1) the same registers are GEMM1's A fragment
// {c0, c2, c1, c3}; GEMM2 (X^T += Wn^T V^T) accumulates straight into them.
//
// V stage image (written by the FP32 panel narrowing): per tile, ib block s, warp row range q and
// ib half h, the RW x IB/2 rows x columns as 8x8 blocks (row block nf, column block jj) of 128
// floats (hi/lo interleaved), element (r, c, hl) of a block at tf32_blk_off(r, c, hl): conflict-free
// 16-byte reads for GEMM1's (rows 2t, 2t+1; column g) and 8-byte reads for GEMM2's (row g;
// columns t, t+4).  One cp.async.bulk per warp and half (8 KB), double-buffered by halves exactly
// like the FP64 kernel.
#pragma once
#include "common.cuh"

namespace tqr {
namespace tf32 {

constexpr int kThreads = 256;
constexpr int kWarps = 8;

__host__ __device__ __forceinline__ int blk_off(int r, int c, int hl) {   // r, c in 0..7
    return c * 16 + (((r >> 2) ^ ((c >> 1) & 1)) << 3) + (((r >> 1) & 1) << 2) + ((r & 1) << 1) + hl;
}

template <int NB, int W, int IB>
struct Geom {
    static constexpr int RW = NB / kWarps;    // rows per warp
    static constexpr int NF = RW / 8;         // n8 row fragments per warp
    static constexpr int MF = W / 16;         // m16 column fragments
    static constexpr int JF = IB / 8;         // 8-wide ib fragments
    static constexpr int HC = IB / 2;         // ib columns per staging half
    static constexpr int JH = JF / 2;         // ib fragments per half
    static constexpr int HALF = RW * HC * 2;  // floats of one warp-half image (hi + lo)
    static constexpr int LDR = IB + 4;        // red / Wsm / Wn / topsm / Tsm pitch
    static constexpr int K4 = IB / 4;
    static_assert(NB % 64 == 0 && W % 16 == 0 && IB % 16 == 0 && NB % IB == 0, "tile geometry");
    static_assert(W * K4 <= kThreads, "reduction mapping");
};

// image offset of element (r, c) (hi or lo) of a V tile
template <int NB, int IB>
__host__ __device__ __forceinline__ int64_t img_off(int r, int c, int hl) {
    using G = Geom<NB, 16, IB>;
    const int s = c / IB, cc = c % IB, q = r / G::RW, rl = r % G::RW, h = cc / G::HC, ch = cc % G::HC;
    return (int64_t)s * NB * IB * 2 + (int64_t)q * G::RW * IB * 2 + h * G::HALF +
           ((rl >> 3) * G::JH + (ch >> 3)) * 128 + blk_off(rl & 7, ch & 7, hl);
}
template <int NB, int IB>
__host__ __device__ constexpr int64_t img_tile() { return (int64_t)NB * NB * 2; }

template <int NB, int W, int IB>
struct Smem {
    using G = Geom<NB, W, IB>;
    uint64_t mbar[kWarps][2];
    float Vst[kWarps][2][G::HALF];
    float red[kWarps][W][G::LDR];       // GEMM1 partials W^T(col, ib) per warp
    float Wsm[W][G::LDR];               // W = X1 + V^T X, [col][ib]
    float Wn[W][G::LDR];                // -op(T) W, [col][ib]  (GEMM2 A operand)
    float Tsm[IB][G::LDR];              // Tsm[c][r] = T(r, c)
    float topsm[W][G::LDR];             // topsm[c][r] = X1(r, c)
};

__device__ __forceinline__ unsigned tf32_rna(float x) {
    unsigned r;
    asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
    return r;
}
// d += a*b, m16n8k8 TF32 (row.col), FP32 accumulate
__device__ __forceinline__ void mma_tf32(float (&d)[4], unsigned a0, unsigned a1, unsigned a2, unsigned a3,
                                         unsigned b0, unsigned b1) {
    asm volatile("mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3},{%4,%5,%6,%7},{%8,%9},{%0,%1,%2,%3};"
                 : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
                 : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}
// round to TF32 (10 explicit mantissa bits), ties away from zero; two integer ops (cvt.rna.tf32 is
// emulated by a 5-instruction sequence on sm_100a).  Finite inputs only (inf / NaN never occur).
__device__ __forceinline__ unsigned tf32_round(float x) { return (__float_as_uint(x) + 0x1000u) & 0xffffe000u; }
// split x = hi + lo into TF32 operands, both rounded (lo carries the next 11 bits)
__device__ __forceinline__ void split(float x, unsigned& hi, unsigned& lo) {
    hi = tf32_round(x);
    lo = tf32_round(x - __uint_as_float(hi));
}

template <int NB, int W, int IB>
struct Slice {
    using G = Geom<NB, W, IB>;
    float acc[G::MF][G::NF][4];
    // element (r, c) at P[c*ld + r]
    __device__ __forceinline__ void load(const float* P, int64_t ld) {
        const int g = lane_id() >> 2, t = lane_id() & 3, r0 = warp_id() * G::RW + 2 * t;
#pragma unroll
        for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
            for (int nf = 0; nf < G::NF; ++nf) {
                const float2 v0 = *reinterpret_cast<const float2*>(P + (int64_t)(mf * 16 + g) * ld + r0 + nf * 8);
                const float2 v1 = *reinterpret_cast<const float2*>(P + (int64_t)(mf * 16 + g + 8) * ld + r0 + nf * 8);
                acc[mf][nf][0] = v0.x; acc[mf][nf][1] = v0.y; acc[mf][nf][2] = v1.x; acc[mf][nf][3] = v1.y;
            }
    }
    __device__ __forceinline__ void store(float* P, int64_t ld) const {
        const int g = lane_id() >> 2, t = lane_id() & 3, r0 = warp_id() * G::RW + 2 * t;
#pragma unroll
        for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
            for (int nf = 0; nf < G::NF; ++nf) {
                *reinterpret_cast<float2*>(P + (int64_t)(mf * 16 + g) * ld + r0 + nf * 8) =
                    make_float2(acc[mf][nf][0], acc[mf][nf][1]);
                *reinterpret_cast<float2*>(P + (int64_t)(mf * 16 + g + 8) * ld + r0 + nf * 8) =
                    make_float2(acc[mf][nf][2], acc[mf][nf][3]);
            }
    }
};

template <int NB, int W, int IB>
__device__ __forceinline__ void stage_init(Smem<NB, W, IB>& sm) {
    if (lane_id() == 0) {
        mbar_init(&sm.mbar[warp_id()][0], 1);
        mbar_init(&sm.mbar[warp_id()][1], 1);
        fence_mbar_init();
    }
    __syncwarp();
}
// half h of block image `blk` (warp w's part) -> Vst[w][h]
template <int NB, int W, int IB>
__device__ __forceinline__ void stage(Smem<NB, W, IB>& sm, const float* blk, int h) {
    using G = Geom<NB, W, IB>;
    const int w = warp_id();
    __syncwarp();
    if (lane_id() == 0) {
        fence_proxy_async_shared();
        bulk_g2s(&sm.Vst[w][h][0], blk + (int64_t)w * G::RW * IB * 2 + h * G::HALF, G::HALF * 4, &sm.mbar[w][h]);
    }
}

// X <- (I - V_s op(T_s) V_s^T) X (+ X1 rows); op = T^T (TRANS) or T.  Half A of block s in flight
// on entry (stage(.., 0) of the previous call or the prologue); `next` = following block image.
template <int NB, int W, int IB, bool TRANS>
__device__ __forceinline__ void apply_block(Slice<NB, W, IB>& X, Smem<NB, W, IB>& sm, const float* __restrict__ Vs,
                                            const float* __restrict__ Ts, float* top, int64_t ldtop, int kmin,
                                            const float* next, unsigned& vph) {
    using G = Geom<NB, W, IB>;
    const int lane = lane_id(), g = lane >> 2, t = lane & 3, wq = warp_id(), tid = threadIdx.x;
    const bool active = (wq + 1) * G::RW > kmin;
    const int nf0 = active ? max(0, (kmin - wq * G::RW) >> 3) : G::NF;   // first row fragment with V != 0

    // ---- (0) half B of V, T block, X1 rows
    stage(sm, Vs, 1);
    for (int id = tid; id < IB * IB / 4; id += kThreads) {
        const int c = id / (IB / 4), r4 = id % (IB / 4);
        cp_async16<true>(&sm.Tsm[c][4 * r4], Ts + c * IB + 4 * r4);
    }
    if (top)
        for (int id = tid; id < W * IB / 4; id += kThreads) {
            const int c = id / (IB / 4), r4 = id % (IB / 4);
            cp_async16<true>(&sm.topsm[c][4 * r4], top + (int64_t)c * ldtop + 4 * r4);
        }
    cp_async_commit();

    // ---- (1) GEMM1: partial W^T(col, ib) = sum over my rows X^T(col, row) V(row, ib).  The hi*hi
    //      products and the two correction products go to separate accumulators, and each group of
    //      MMAs cycles over MF x JH independent accumulators, so dependent MMAs are never adjacent.
    float c1[G::MF][G::JF][4], cc[G::MF][G::JF][4];
#pragma unroll
    for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
        for (int j = 0; j < G::JF; ++j)
#pragma unroll
            for (int e = 0; e < 4; ++e) c1[mf][j][e] = cc[mf][j][e] = 0.f;
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        mbar_wait(&sm.mbar[wq][h], (vph >> h) & 1u);
        vph ^= 1u << h;
        const float* vh = &sm.Vst[wq][h][0];
#pragma unroll
        for (int nf = 0; nf < G::NF; ++nf) {
            if (nf < nf0) continue;
            unsigned ah[G::MF][4], al[G::MF][4];
#pragma unroll
            for (int mf = 0; mf < G::MF; ++mf) {
                split(X.acc[mf][nf][0], ah[mf][0], al[mf][0]);
                split(X.acc[mf][nf][2], ah[mf][1], al[mf][1]);
                split(X.acc[mf][nf][1], ah[mf][2], al[mf][2]);
                split(X.acc[mf][nf][3], ah[mf][3], al[mf][3]);
            }
            unsigned bh[G::JH][2], bl[G::JH][2];
#pragma unroll
            for (int jj = 0; jj < G::JH; ++jj) {
                // B: V(rows 2t, 2t+1 of fragment nf; ib column g of fragment jj) = {hi, lo, hi, lo}
                const float4 v = *reinterpret_cast<const float4*>(vh + (nf * G::JH + jj) * 128 + blk_off(2 * t, g, 0));
                bh[jj][0] = __float_as_uint(v.x); bl[jj][0] = __float_as_uint(v.y);
                bh[jj][1] = __float_as_uint(v.z); bl[jj][1] = __float_as_uint(v.w);
            }
#pragma unroll
            for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
                for (int jj = 0; jj < G::JH; ++jj)
                    mma_tf32(c1[mf][h * G::JH + jj], ah[mf][0], ah[mf][1], ah[mf][2], ah[mf][3], bh[jj][0], bh[jj][1]);
#pragma unroll
            for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
                for (int jj = 0; jj < G::JH; ++jj)
                    mma_tf32(cc[mf][h * G::JH + jj], al[mf][0], al[mf][1], al[mf][2], al[mf][3], bh[jj][0], bh[jj][1]);
#pragma unroll
            for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
                for (int jj = 0; jj < G::JH; ++jj)
                    mma_tf32(cc[mf][h * G::JH + jj], ah[mf][0], ah[mf][1], ah[mf][2], ah[mf][3], bl[jj][0], bl[jj][1]);
        }
    }
#pragma unroll
    for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
        for (int j = 0; j < G::JF; ++j)
#pragma unroll
            for (int e = 0; e < 4; ++e) c1[mf][j][e] += cc[mf][j][e];
    // c1[mf][j] = W^T[col mf*16 + g (+8)][ib j*8 + 2t (+1)]
#pragma unroll
    for (int mf = 0; mf < G::MF; ++mf)
#pragma unroll
        for (int j = 0; j < G::JF; ++j) {
            *reinterpret_cast<float2*>(&sm.red[wq][mf * 16 + g][j * 8 + 2 * t]) = make_float2(c1[mf][j][0], c1[mf][j][1]);
            *reinterpret_cast<float2*>(&sm.red[wq][mf * 16 + g + 8][j * 8 + 2 * t]) = make_float2(c1[mf][j][2], c1[mf][j][3]);
        }
    cp_async_wait<0>();
    __syncthreads();

    // ---- (2) W(col, k4..k4+3) = X1 + sum of the warp partials
    const bool rth = tid < W * G::K4;
    const int rc = tid / G::K4, rk = (tid % G::K4) * 4;
    if (rth) {
        float4 acc = top ? *reinterpret_cast<const float4*>(&sm.topsm[rc][rk]) : make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
        for (int w = 0; w < kWarps; ++w) {
            const float4 v = *reinterpret_cast<const float4*>(&sm.red[w][rc][rk]);
            acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
        }
        *reinterpret_cast<float4*>(&sm.Wsm[rc][rk]) = acc;
    }
    __syncthreads();
    // ---- (3) W' = op(T) W (explicit zeros below the diagonal of T); X1 -= W'; Wn = -W'
    if (rth) {
        float o[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
        for (int k4 = 0; k4 < IB; k4 += 4) {
            const float4 w = *reinterpret_cast<const float4*>(&sm.Wsm[rc][k4]);
            const float wv[4] = {w.x, w.y, w.z, w.w};
            if constexpr (TRANS) {
#pragma unroll
                for (int e = 0; e < 4; ++e) {   // T(kp, rk + e), kp = k4..k4+3 contiguous in Tsm[rk + e]
                    const float4 tv = *reinterpret_cast<const float4*>(&sm.Tsm[rk + e][k4]);
                    o[e] = fmaf(tv.x, wv[0], fmaf(tv.y, wv[1], fmaf(tv.z, wv[2], fmaf(tv.w, wv[3], o[e]))));
                }
            } else {
#pragma unroll
                for (int j = 0; j < 4; ++j) {   // T(rk + e, kp) for e = 0..3 contiguous in Tsm[kp]
                    const float4 tv = *reinterpret_cast<const float4*>(&sm.Tsm[k4 + j][rk]);
                    o[0] = fmaf(tv.x, wv[j], o[0]); o[1] = fmaf(tv.y, wv[j], o[1]);
                    o[2] = fmaf(tv.z, wv[j], o[2]); o[3] = fmaf(tv.w, wv[j], o[3]);
                }
            }
        }
        *reinterpret_cast<float4*>(&sm.Wn[rc][rk]) = make_float4(-o[0], -o[1], -o[2], -o[3]);
        if (top) {
            const float4 tp = *reinterpret_cast<const float4*>(&sm.topsm[rc][rk]);
            *reinterpret_cast<float4*>(top + (int64_t)rc * ldtop + rk) =
                make_float4(tp.x - o[0], tp.y - o[1], tp.z - o[2], tp.w - o[3]);
        }
    }
    __syncthreads();

    // ---- (4) GEMM2: X^T(col, row) += Wn^T(col, ib) V^T(ib, row); half A of `next` staged once
    //      half A of this block has been consumed
#pragma unroll
    for (int h = 0; h < 2; ++h) {
        if (h == 1 && next != nullptr) stage(sm, next, 0);
        const float* vh = &sm.Vst[wq][h][0];
#pragma unroll
        for (int jj = 0; jj < G::JH; ++jj) {
            const int kk = (h * G::JH + jj) * 8;
            unsigned ah[G::MF][4], al[G::MF][4];
#pragma unroll
            for (int mf = 0; mf < G::MF; ++mf) {
                split(sm.Wn[mf * 16 + g][kk + t], ah[mf][0], al[mf][0]);
                split(sm.Wn[mf * 16 + g + 8][kk + t], ah[mf][1], al[mf][1]);
                split(sm.Wn[mf * 16 + g][kk + t + 4], ah[mf][2], al[mf][2]);
                split(sm.Wn[mf * 16 + g + 8][kk + t + 4], ah[mf][3], al[mf][3]);
            }
            // B: V^T(ib kk + t (+4), row nf*8 + g) = V(row g, column t / t + 4) of block (nf, jj), all nf
            unsigned bh[G::NF][2], bl[G::NF][2];
#pragma unroll
            for (int nf = 0; nf < G::NF; ++nf) {
                const float* bp = vh + (nf * G::JH + jj) * 128;
                const float2 v0 = *reinterpret_cast<const float2*>(bp + blk_off(g, t, 0));
                const float2 v1 = *reinterpret_cast<const float2*>(bp + blk_off(g, t + 4, 0));
                bh[nf][0] = __float_as_uint(v0.x); bl[nf][0] = __float_as_uint(v0.y);
                bh[nf][1] = __float_as_uint(v1.x); bl[nf][1] = __float_as_uint(v1.y);
            }
            // three passes over the MF x NF independent accumulators (hi*hi, lo*hi, hi*lo)
#pragma unroll
            for (int nf = 0; nf < G::NF; ++nf) {
                if (nf < nf0) continue;
#pragma unroll
                for (int mf = 0; mf < G::MF; ++mf)
                    mma_tf32(X.acc[mf][nf], ah[mf][0], ah[mf][1], ah[mf][2], ah[mf][3], bh[nf][0], bh[nf][1]);
            }
#pragma unroll
            for (int nf = 0; nf < G::NF; ++nf) {
                if (nf < nf0) continue;
#pragma unroll
                for (int mf = 0; mf < G::MF; ++mf)
                    mma_tf32(X.acc[mf][nf], al[mf][0], al[mf][1], al[mf][2], al[mf][3], bh[nf][0], bh[nf][1]);
            }
#pragma unroll
            for (int nf = 0; nf < G::NF; ++nf) {
                if (nf < nf0) continue;
#pragma unroll
                for (int mf = 0; mf < G::MF; ++mf)
                    mma_tf32(X.acc[mf][nf], ah[mf][0], ah[mf][1], ah[mf][2], ah[mf][3], bl[nf][0], bl[nf][1]);
            }
        }
    }
}

}  // namespace tf32
}  // namespace tqr
