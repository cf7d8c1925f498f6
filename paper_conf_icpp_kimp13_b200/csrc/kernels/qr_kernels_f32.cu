// qr_kernels_f32.cu -- the FP32 path of the tiled Householder QR (configs C5 FP32).
//
//   update_kernel32 : UNMQR(k,j) + TSMQR(i,j,k) chain for every trailing column slice (Eqs. 6
//                     and 9, reading Q5), FFMA apply of tile_ops_f32.cuh; also Q^T B / Q B.
//   panel step      : the panel column (tiles k..p-1 of column k) is widened to FP64, factored by
//                     the FP64 panel kernel (GEQRT + TSQRT chain, Eqs. 4-5, 7-8) and written back:
//                     R / reflectors in place (FP32), T factors (FP32) and the FP32 stage images of
//                     the reflectors the update kernel streams.  The panel is <= 2 % of the flops at
//                     C5; computing it in FP64 keeps its Householder vectors orthogonal to FP64
//                     accuracy before the single rounding to FP32.
#include <algorithm>
#include <cstdio>
#include "tile_ops_f32.cuh"
#include "../tqr_internal.h"

namespace tqr {
namespace f32 {

// Same block order as the FP64 update_kernel (qr_kernels.cu): forward UNMQR blocks 0..NBLK-1 of
// row tile k, then TSMQR blocks 0..NBLK-1 of tiles k+1..p-1; backward the exact reverse.
template <int NB, int W, int IB, bool TRANS>
__global__ void __launch_bounds__(kThreads, 1) update_kernel32(UpdateArgsT<float> a) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    auto& sm = *reinterpret_cast<Smem32<NB, W, IB>*>(smem_raw);
    constexpr int SPG = NB / W;
    constexpr int NBLK = NB / IB;
    constexpr int64_t VT = img_tile<NB, IB>();
    const int grp = blockIdx.x / SPG;
    const int c0 = (blockIdx.x % SPG) * W;
    float* Xg = a.X + (int64_t)(a.group0 + grp * a.gstride) * a.col_stride + (int64_t)c0 * a.ld;
    float* Xk = Xg + (int64_t)a.k * a.tile_stride;
    Slice32<NB, W, IB> X;
    stage_init32(sm);
    unsigned vph = 0;
    int buf = 0;
    const int ntiles = a.p - a.k - 1 + (a.do_unmqr ? 1 : 0);
    auto tile_of = [&](int q) -> int {
        if (TRANS) return a.do_unmqr ? (q == 0 ? -1 : a.k + q) : a.k + 1 + q;
        return (q < a.p - a.k - 1) ? a.p - 1 - q : -1;
    };
    auto vblock = [&](int ti, int s) -> const float* {
        return (ti < 0 ? a.Vexp : a.V + (int64_t)ti * VT) + (int64_t)s * NB * (IB + 4);
    };
    auto blk = [&](int si) { return TRANS ? si : NBLK - 1 - si; };
    if (ntiles > 0) stage32(sm, vblock(tile_of(0), blk(0)), 0);
    for (int q = 0; q < ntiles; ++q) {
        const int ti = tile_of(q);
        float* Xi = (ti < 0) ? Xk : Xg + (int64_t)ti * a.tile_stride;
        const float* Tt = a.T + (int64_t)(ti < 0 ? a.k : ti) * IB * NB;
        X.load(Xi, a.ld);
        for (int si = 0; si < NBLK; ++si) {
            const int s = blk(si);
            const float* nxt = nullptr;
            if (si + 1 < NBLK) nxt = vblock(ti, blk(si + 1));
            else if (q + 1 < ntiles) nxt = vblock(tile_of(q + 1), blk(0));
            apply_block32<NB, W, IB, TRANS>(X, sm, Tt + (int64_t)s * IB * IB, ti < 0 ? nullptr : Xk + s * IB, a.ld,
                                            ti < 0 ? s * IB : 0, nxt, vph, buf);
        }
        X.store(Xi, a.ld);
        __syncthreads();   // row tile k (the TS "top") is re-read by other threads
    }
}

// Panel in: FP32 tiles -> FP64 scratch (same tile layout), n elements, 16-byte loads.
__global__ void widen_kernel(const float* __restrict__ src, double* __restrict__ dst, int64_t n4) {
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x) {
        const float4 v = reinterpret_cast<const float4*>(src)[i];
        reinterpret_cast<double2*>(dst)[2 * i] = make_double2(v.x, v.y);
        reinterpret_cast<double2*>(dst)[2 * i + 1] = make_double2(v.z, v.w);
    }
}

// Panel out: one CTA per (tile i >= k, ib block s, 128-row chunk).  Reads the FP64 scratch tile
// (reflectors in place: GEQRT tile k = R above / unit-lower V below the diagonal, TSQRT tiles = V2)
// column by column, writes the FP32 tile (same layout) and, through a shared-memory transpose, the
// FP32 stage image rows (k contiguous) -- explicit unit-lower V for tile k (Vexp), V2 otherwise.
// CTA (i, s, chunk 0) also narrows the T block s of tile i.
template <int NB, int IB>
__global__ void __launch_bounds__(256) narrow_panel_kernel(const double* __restrict__ sc, const double* __restrict__ T64,
                                                          float* __restrict__ tiles, float* __restrict__ T32,
                                                          float* __restrict__ Vimg, float* __restrict__ Vexp, int k) {
    constexpr int RC = NB < 128 ? NB : 128;       // rows per CTA
    constexpr int IBP = IB + 4;
    __shared__ float st[RC][IBP + 1];
    const int nch = NB / RC;
    const int chunk = blockIdx.x % nch, s = (blockIdx.x / nch) % (NB / IB), i = k + blockIdx.x / (nch * (NB / IB));
    const int64_t tile = (int64_t)NB * NB;
    const bool ge = (i == k);
    const double* src = sc + (int64_t)i * tile;
    float* dt = tiles + (int64_t)i * tile;
    const int r0 = chunk * RC;
    for (int e = threadIdx.x; e < IB * RC; e += blockDim.x) {
        const int kk = e / RC, rl = e % RC;
        const int c = s * IB + kk, r = r0 + rl;
        const double v = src[(int64_t)c * NB + r];
        dt[(int64_t)c * NB + r] = (float)v;
        st[rl][kk] = ge ? (r > c ? (float)v : (r == c ? 1.f : 0.f)) : (float)v;
    }
    __syncthreads();
    float* img = (ge ? Vexp : Vimg + (int64_t)i * img_tile<NB, IB>()) + (int64_t)s * NB * IBP + (int64_t)r0 * IBP;
    for (int e = threadIdx.x; e < RC * IBP; e += blockDim.x) {
        const int rl = e / IBP, kk = e % IBP;
        img[e] = (kk < IB) ? st[rl][kk] : 0.f;
    }
    if (chunk == 0) {
        const double* ts = T64 + (int64_t)i * IB * NB + (int64_t)s * IB * IB;
        float* td = T32 + (int64_t)i * IB * NB + (int64_t)s * IB * IB;
        for (int e = threadIdx.x; e < IB * IB; e += blockDim.x) td[e] = (float)ts[e];
    }
}

template <int NB, int W, int IB>
static cudaError_t launch_update32_t(const UpdateArgsT<float>& a, int nslices, bool trans, cudaStream_t s) {
  if constexpr (!G32<NB, W, IB>::ok) {
    return cudaErrorInvalidValue;     // slice too narrow for the tile (nb = 64, w = 8)
  } else {
    const size_t smem = sizeof(Smem32<NB, W, IB>);
    if (nslices <= 0) return cudaSuccess;
    if (trans) {
        auto kern = update_kernel32<NB, W, IB, true>;
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        kern<<<nslices, kThreads, smem, s>>>(a);
    } else {
        auto kern = update_kernel32<NB, W, IB, false>;
        cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        if (e != cudaSuccess) return e;
        kern<<<nslices, kThreads, smem, s>>>(a);
    }
    return cudaGetLastError();
  }
}

constexpr size_t kMaxSmem = 232448;
template <int NB, int W, int IB>
constexpr bool fits() {
    if constexpr (G32<NB, W, IB>::ok) return sizeof(Smem32<NB, W, IB>) <= kMaxSmem;
    else return true;
}
#define TQR_FITS32(NB_, IB_)                                                \
    static_assert(fits<NB_, 8, IB_>(), "f32 update smem W=8");              \
    static_assert(fits<NB_, 16, IB_>(), "f32 update smem W=16");            \
    static_assert(fits<NB_, 32, IB_>(), "f32 update smem W=32");
TQR_FITS32(64, 16) TQR_FITS32(64, 32) TQR_FITS32(128, 16) TQR_FITS32(128, 32)
TQR_FITS32(256, 16) TQR_FITS32(256, 32) TQR_FITS32(512, 16) TQR_FITS32(512, 32)
#undef TQR_FITS32

}  // namespace f32



cudaError_t launch_update_f32(int nb, int ib, int w, const UpdateArgsT<float>& a, int nslices, bool trans,
                              cudaStream_t s) {
#define TQR_UPD32(NB_, IB_)                                                                   \
    if (nb == NB_ && ib == IB_) {                                                             \
        if (w == 8) return f32::launch_update32_t<NB_, 8, IB_>(a, nslices, trans, s);         \
        if (w == 16) return f32::launch_update32_t<NB_, 16, IB_>(a, nslices, trans, s);       \
        if (w == 32) return f32::launch_update32_t<NB_, 32, IB_>(a, nslices, trans, s);       \
        return cudaErrorInvalidValue;                                                         \
    }
    TQR_UPD32(64, 16) TQR_UPD32(64, 32) TQR_UPD32(128, 16) TQR_UPD32(128, 32)
    TQR_UPD32(256, 16) TQR_UPD32(256, 32) TQR_UPD32(512, 16) TQR_UPD32(512, 32)
#undef TQR_UPD32
    return cudaErrorInvalidValue;
}

cudaError_t launch_widen(const float* src, double* dst, int64_t n, cudaStream_t s) {
    if (n <= 0) return cudaSuccess;
    if (n % 4) return cudaErrorInvalidValue;
    const int64_t n4 = n / 4;
    const int grid = (int)std::min<int64_t>((n4 + 255) / 256, 148 * 8);
    f32::widen_kernel<<<grid, 256, 0, s>>>(src, dst, n4);
    return cudaGetLastError();
}

cudaError_t launch_narrow_panel(int nb, int ib, const double* sc, const double* T64, float* tiles, float* T32,
                                float* Vimg, float* Vexp, int k, int p, cudaStream_t s) {
    const int ntiles = p - k;
    if (ntiles <= 0) return cudaSuccess;
#define TQR_NAR(NB_, IB_)                                                                                   \
    if (nb == NB_ && ib == IB_) {                                                                           \
        const int grid = ntiles * (NB_ / IB_) * (NB_ >= 128 ? NB_ / 128 : 1);                               \
        f32::narrow_panel_kernel<NB_, IB_><<<grid, 256, 0, s>>>(sc, T64, tiles, T32, Vimg, Vexp, k);        \
        return cudaGetLastError();                                                                          \
    }
    TQR_NAR(64, 16) TQR_NAR(64, 32) TQR_NAR(128, 16) TQR_NAR(128, 32) TQR_NAR(256, 16) TQR_NAR(256, 32) TQR_NAR(512, 16) TQR_NAR(512, 32)
#undef TQR_NAR
    return cudaErrorInvalidValue;
}

int64_t f32_img_tile(int nb, int ib) { return (int64_t)(nb / ib) * nb * (ib + 4); }

}  // namespace tqr
