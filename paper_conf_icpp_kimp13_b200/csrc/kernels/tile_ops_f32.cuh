// tile_ops_f32.cuh -- FP32 block-reflector apply on the SIMT FFMA pipe.
//
// The FP32 trailing update (UNMQR, Eq. 6, and TSMQR, Eq. 9 -- applied as Q^T, reading Q5) has the
// same structure as the FP64 DMMA path (tile_ops.cuh): one CTA owns an NB x W column slice X of a
// trailing tile column in registers and, per ib-wide reflector block s,
//     W  = X1 + V_s^T X           (GEMM1, K = NB rows; per-warp reduce-scatter over shuffles,
//                                  then an 8-slot shared-memory sum)
//     W' = op(T_s) W              (ib x ib triangular)
//     X1 -= W' ;  X -= V_s W'     (GEMM2, K = ib)
// sm_100a has no FP32-accurate tensor-core kind (TF32 keeps 10 mantissa bits, too few for the
// 1e-5 residual bar), so both GEMMs are FFMA: thread (rg, cg) of warp w owns the R = RW/RG rows
// w*RW + rg + RG*i (interleaved) of the column quad 4cg..4cg+3.  Every 16-byte shared-memory
// read of V (4 consecutive k of one row, broadcast to the CG lanes sharing the row) feeds 16 FFMAs
// in both GEMMs, which keeps the shared-memory pipe (2 wavefronts per such read: one per
// half-warp) below the FFMA pipe (measured: 2 columns per thread made the kernel smem-bound).
// GEMM1 runs in k-chunks of 16 so the partial sums fit in registers next to X.  V is staged per warp (each warp only reads its own RW rows) by one
// cp.async.bulk from the "stage image" the panel step writes: block s of a tile is NB rows of
// IBP = IB + 4 floats (k contiguous, 4 floats of padding), so the RG adjacent rows read together
// fall in distinct 16-byte bank groups without a swizzle.  Two buffers per warp: block s+1 is in
// flight while block s is computed.
#pragma once
#include "common.cuh"

namespace tqr {
namespace f32 {

constexpr int kThreads = 256;
constexpr int kWarps = 8;

template <int NB, int W, int IB>
struct G32 {
    static constexpr int RW = NB / kWarps;      // rows per warp
    static constexpr int CG = W / 4;            // column quads (lanes % CG)
    static constexpr int RG = 32 / CG;          // row groups per warp
    static constexpr int R = RW / RG;           // rows per thread
    static constexpr int KC = IB / 4;           // 16-byte chunks per V row
    static constexpr int KCH = 16;              // GEMM1 k-chunk
    static constexpr int NCH = IB / KCH;        // GEMM1 chunks
    static constexpr int KPL = KCH / RG;        // k values per lane and chunk after the reduce-scatter
    static constexpr int IBP = IB + 4;          // padded V row (floats)
    static constexpr int VBLK = RW * IBP;       // one warp's staged rows of one block (floats)
    static constexpr int LDT = IB + 4;          // Tsm / topsm row pitch (16-byte aligned, bank-skewed)
    static constexpr int W4 = W / 4;            // float4 column groups in the reduction
    static constexpr bool ok = (W % 8 == 0) && (32 % CG == 0) && (RW >= RG) && (KCH % RG == 0) && (IB % KCH == 0);
    static_assert(IB * W4 <= kThreads, "reduction mapping");
};

// Stage image of a V tile (NB x NB reflectors): block s = columns [s*IB, s*IB + IB) is NB rows
// of IBP floats; element (r, c) at img_off(r, c).  Warp w's rows of block s are the contiguous
// VBLK floats at s*NB*IBP + w*VBLK.
template <int NB, int IB>
__host__ __device__ constexpr int64_t img_tile() { return (int64_t)(NB / IB) * NB * (IB + 4); }
template <int NB, int IB>
__host__ __device__ __forceinline__ int64_t img_off(int r, int c) {
    return (int64_t)(c / IB) * NB * (IB + 4) + (int64_t)r * (IB + 4) + (c % IB);
}

template <int NB, int W, int IB>
struct Smem32 {
    static_assert(G32<NB, W, IB>::ok, "f32 geometry");
    using G = G32<NB, W, IB>;
    uint64_t mbar[kWarps][2];                   // bulk-copy completion of vbuf[w][b]
    float vbuf[kWarps][2][G::VBLK];
    float red[kWarps][IB][W];                   // per-warp GEMM1 sums (after the reduce-scatter)
    float Wsm[IB][W];                           // W = X1 + V^T X
    float Wn[IB][W];                            // -op(T) W   (GEMM2 operand)
    float Tsm[IB][G::LDT];                      // T block: Tsm[c][r] = T(r, c)
    float topsm[W][G::LDT];                     // X1: topsm[c][r] = X1(r, c)
};

template <int NB, int W, int IB>
struct Slice32 {
    using G = G32<NB, W, IB>;
    float x[G::R][4];
    // element (r, c) of the slice at P[c*ld + r]
    __device__ __forceinline__ void load(const float* P, int64_t ld) {
        const int lane = lane_id(), cg = lane % G::CG, rg = lane / G::CG, rb = warp_id() * G::RW + rg;
#pragma unroll
        for (int i = 0; i < G::R; ++i)
#pragma unroll
            for (int c = 0; c < 4; ++c) x[i][c] = P[(int64_t)(4 * cg + c) * ld + rb + G::RG * i];
    }
    __device__ __forceinline__ void store(float* P, int64_t ld) const {
        const int lane = lane_id(), cg = lane % G::CG, rg = lane / G::CG, rb = warp_id() * G::RW + rg;
#pragma unroll
        for (int i = 0; i < G::R; ++i)
#pragma unroll
            for (int c = 0; c < 4; ++c) P[(int64_t)(4 * cg + c) * ld + rb + G::RG * i] = x[i][c];
    }
};

template <int NB, int W, int IB>
__device__ __forceinline__ void stage_init32(Smem32<NB, W, IB>& sm) {
    if (lane_id() == 0) {
        mbar_init(&sm.mbar[warp_id()][0], 1);
        mbar_init(&sm.mbar[warp_id()][1], 1);
        fence_mbar_init();
    }
    __syncwarp();
}
// Warp w's rows of block image `blk` -> vbuf[w][b] (lane 0 issues after the warp's reads of the
// buffer: __syncwarp + async-proxy fence).
template <int NB, int W, int IB>
__device__ __forceinline__ void stage32(Smem32<NB, W, IB>& sm, const float* blk, int b) {
    using G = G32<NB, W, IB>;
    const int w = warp_id();
    __syncwarp();
    if (lane_id() == 0) {
        fence_proxy_async_shared();
        bulk_g2s(&sm.vbuf[w][b][0], blk + w * G::VBLK, G::VBLK * 4, &sm.mbar[w][b]);
    }
}

// X <- (I - V_s op(T_s) V_s^T) X (+ X1 rows), op = T^T (TRANS, Q^T) or T (Q).
//   Vs   : stage image of block s (already in flight into vbuf[w][buf]).
//   next : image of the following block (staged here into vbuf[w][buf^1]) or null.
//   Ts   : T block (IB x IB column-major, zeros below the diagonal).
//   top  : X1 (IB x W, element (r, c) at top[c*ldtop + r]) or null (UNMQR).
//   kmin : rows < kmin of V are zero (UNMQR blocks); warps whose rows are all < kmin skip both
//          GEMMs.  A runtime value (not a template flag) so the kernel holds one copy of this body.
template <int NB, int W, int IB, bool TRANS>
__device__ __forceinline__ void apply_block32(Slice32<NB, W, IB>& X, Smem32<NB, W, IB>& sm,
                                              const float* __restrict__ Ts, float* top, int64_t ldtop,
                                              int kmin, const float* next, unsigned& vph, int& buf) {
    using G = G32<NB, W, IB>;
    const int lane = lane_id(), w = warp_id(), tid = threadIdx.x;
    const int cg = lane % G::CG, rg = lane / G::CG;
    const bool active = (w + 1) * G::RW > kmin;

    // ---- (0) T block and X1 rows (LDGSTS, waited before barrier 1); next block's V (bulk)
    for (int id = tid; id < IB * IB / 4; id += kThreads) {
        const int c = id / (IB / 4), r4 = id % (IB / 4);
        cp_async16<true>(&sm.Tsm[c][4 * r4], Ts + c * IB + 4 * r4);
    }
    if (top) {
        for (int id = tid; id < W * IB / 4; id += kThreads) {
            const int c = id / (IB / 4), r4 = id % (IB / 4);
            cp_async16<true>(&sm.topsm[c][4 * r4], top + (int64_t)c * ldtop + 4 * r4);
        }
    }
    cp_async_commit();
    mbar_wait(&sm.mbar[w][buf], (vph >> buf) & 1u);
    vph ^= 1u << buf;
    if (next) stage32(sm, next, buf ^ 1);
    const float* vb = &sm.vbuf[w][buf][0];

    // ---- (1) GEMM1 per k-chunk: P(k, c) = sum over my rows of V(r, k) X(r, c), then a
    //      reduce-scatter over the RG lanes sharing a column quad (xor 16, 8, .., CG): each level
    //      halves the k range a lane keeps; one float4 store per kept k
#pragma unroll 1
    for (int ch = 0; ch < G::NCH; ++ch) {     // runtime loop: keeps the body in the instruction cache
        float P[G::KCH][4];
#pragma unroll
        for (int k = 0; k < G::KCH; ++k)
#pragma unroll
            for (int c = 0; c < 4; ++c) P[k][c] = 0.f;
        if (active) {
#pragma unroll
            for (int i = 0; i < G::R; ++i) {
                const float4* vr = reinterpret_cast<const float4*>(vb + (rg + G::RG * i) * G::IBP + ch * G::KCH);
                float4 v[G::KCH / 4];
#pragma unroll
                for (int q = 0; q < G::KCH / 4; ++q) v[q] = vr[q];
#pragma unroll
                for (int q = 0; q < G::KCH / 4; ++q)
#pragma unroll
                    for (int c = 0; c < 4; ++c) {
                        const float xc = X.x[i][c];
                        P[4 * q + 0][c] = fmaf(v[q].x, xc, P[4 * q + 0][c]);
                        P[4 * q + 1][c] = fmaf(v[q].y, xc, P[4 * q + 1][c]);
                        P[4 * q + 2][c] = fmaf(v[q].z, xc, P[4 * q + 2][c]);
                        P[4 * q + 3][c] = fmaf(v[q].w, xc, P[4 * q + 3][c]);
                    }
            }
        }
        int k0 = ch * G::KCH;
#pragma unroll
        for (int j = 0; (1 << j) < G::RG; ++j) {
            const int m = 16 >> j;
            const int H = (G::KCH >> j) / 2;
            const bool up = (lane & m) != 0;
#pragma unroll
            for (int e = 0; e < H; ++e)
#pragma unroll
                for (int c = 0; c < 4; ++c) {
                    const float send = up ? P[e][c] : P[e + H][c];
                    const float keep = up ? P[e + H][c] : P[e][c];
                    P[e][c] = keep + __shfl_xor_sync(0xffffffffu, send, m);
                }
            if (up) k0 += H;
        }
#pragma unroll
        for (int e = 0; e < G::KPL; ++e)
            *reinterpret_cast<float4*>(&sm.red[w][k0 + e][4 * cg]) = make_float4(P[e][0], P[e][1], P[e][2], P[e][3]);
    }
    cp_async_wait<0>();
    __syncthreads();

    // ---- (3) W(k, c4..c4+3) = X1 + sum over the 8 warp slots
    const bool rth = tid < IB * G::W4;
    const int rk = tid / G::W4, rc = (tid % G::W4) * 4;
    if (rth) {
        float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
        if (top) acc = make_float4(sm.topsm[rc][rk], sm.topsm[rc + 1][rk], sm.topsm[rc + 2][rk], sm.topsm[rc + 3][rk]);
#pragma unroll
        for (int ww = 0; ww < kWarps; ++ww) {
            const float4 v = *reinterpret_cast<const float4*>(&sm.red[ww][rk][rc]);
            acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
        }
        *reinterpret_cast<float4*>(&sm.Wsm[rk][rc]) = acc;
    }
    __syncthreads();
    // ---- (4) W' = op(T) W (T upper triangular, explicit zeros below); X1 -= W'; Wn = -W'
    if (rth) {
        float4 o = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll 8
        for (int kp = 0; kp < IB; ++kp) {
            const float t = TRANS ? sm.Tsm[rk][kp] : sm.Tsm[kp][rk];   // T(kp, rk) : T(rk, kp)
            const float4 v = *reinterpret_cast<const float4*>(&sm.Wsm[kp][rc]);
            o.x = fmaf(t, v.x, o.x); o.y = fmaf(t, v.y, o.y); o.z = fmaf(t, v.z, o.z); o.w = fmaf(t, v.w, o.w);
        }
        *reinterpret_cast<float4*>(&sm.Wn[rk][rc]) = make_float4(-o.x, -o.y, -o.z, -o.w);
        if (top) {
            top[(int64_t)(rc + 0) * ldtop + rk] = sm.topsm[rc + 0][rk] - o.x;
            top[(int64_t)(rc + 1) * ldtop + rk] = sm.topsm[rc + 1][rk] - o.y;
            top[(int64_t)(rc + 2) * ldtop + rk] = sm.topsm[rc + 2][rk] - o.z;
            top[(int64_t)(rc + 3) * ldtop + rk] = sm.topsm[rc + 3][rk] - o.w;
        }
    }
    __syncthreads();

    // ---- (5) GEMM2: X(r, c) += sum_k V(r, k) Wn(k, c)
    if (active) {
#pragma unroll 1
        for (int kc = 0; kc < G::KC; ++kc) {   // runtime loop (instruction-cache footprint)
            float4 wv[4];
#pragma unroll
            for (int e = 0; e < 4; ++e) wv[e] = *reinterpret_cast<const float4*>(&sm.Wn[4 * kc + e][4 * cg]);
#pragma unroll
            for (int i = 0; i < G::R; ++i) {
                const float4 v = reinterpret_cast<const float4*>(vb + (rg + G::RG * i) * G::IBP)[kc];
                float a0 = X.x[i][0], a1 = X.x[i][1], a2 = X.x[i][2], a3 = X.x[i][3];
                a0 = fmaf(v.x, wv[0].x, a0); a1 = fmaf(v.x, wv[0].y, a1); a2 = fmaf(v.x, wv[0].z, a2); a3 = fmaf(v.x, wv[0].w, a3);
                a0 = fmaf(v.y, wv[1].x, a0); a1 = fmaf(v.y, wv[1].y, a1); a2 = fmaf(v.y, wv[1].z, a2); a3 = fmaf(v.y, wv[1].w, a3);
                a0 = fmaf(v.z, wv[2].x, a0); a1 = fmaf(v.z, wv[2].y, a1); a2 = fmaf(v.z, wv[2].z, a2); a3 = fmaf(v.z, wv[2].w, a3);
                a0 = fmaf(v.w, wv[3].x, a0); a1 = fmaf(v.w, wv[3].y, a1); a2 = fmaf(v.w, wv[3].z, a2); a3 = fmaf(v.w, wv[3].w, a3);
                X.x[i][0] = a0; X.x[i][1] = a1; X.x[i][2] = a2; X.x[i][3] = a3;
            }
        }
    }
    buf ^= 1;
    // Exit: the next call's red / Wsm / Wn writes follow its own barriers; every read of those
    // buffers in this call precedes this call's last barrier.
}

}  // namespace f32
}  // namespace tqr
