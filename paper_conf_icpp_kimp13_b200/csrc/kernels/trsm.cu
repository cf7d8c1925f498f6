// trsm.cu -- back substitution R X = C of tqr_solve_ls (Eq. 3: "x = R^-1 Q^T b"),
// on the tile storage of R directly (no gather to column-major), one step per tile row i,
// i = q-1 .. 0 (NEXT-3):
//
//   trsm_diag_kernel   : X_i = R_ii^-1 C_i for one 32-wide right-hand-side slice per CTA.  The
//                        C_i slice stays in shared memory; the tile is walked bottom-up in 32-row
//                        blocks: the 32 x 32 diagonal block of R_ii is inverted by one warp (lane j
//                        back-substitutes column j of the inverse in registers, no barriers),
//                        X_blk = U^-1 C_blk, then the rows above the block inside the tile get
//                        C -= R_ii(rows, blk) X_blk.
//   trsm_update_kernel : C_r -= R_ri X_i for every row tile r < i: a 128 x 32 output block per
//                        CTA, the column tile i of R (tiles 0..i-1 stacked contiguously in the
//                        owner's column storage) streamed through shared memory in 32-deep k
//                        chunks, 4 x 4 register micro-tiles (FP64 / FP32 FMA).  HBM-bound for few
//                        right-hand sides (R is read once per 32 columns of X).
//
// Rows >= n_valid of the last tile row are the plan's zero padding (Q20): their diagonal is taken
// as 1 and their C rows as 0, so X is 0 there and the padded rows/columns of R (all zero) add
// nothing.  Exact zeros on the real diagonal are rejected by the caller (TQR_ERR_SINGULAR)
// before any of this runs.
#include <algorithm>
#include <cstdint>
#include "../tqr_internal.h"

namespace tqr {
namespace {

constexpr int kT = 256;   // threads per CTA
constexpr int RB = 32;    // diagonal block / RHS slice width

template <class T, int NB>
struct DiagSmem {
    T C[NB][RB + 1];      // C_i slice, row-major with padding (column reads conflict-free)
    T U[RB][RB + 1];      // diagonal block
    T Ui[RB][RB + 1];     // its inverse
    T X[RB][RB + 1];      // solved block rows
};

template <class T, int NB>
__global__ void __launch_bounds__(kT) trsm_diag_kernel(const T* __restrict__ Rii, T* __restrict__ C, int64_t ldc,
                                                      int n_valid) {
    extern __shared__ __align__(16) unsigned char smem_raw[];
    auto& sm = *reinterpret_cast<DiagSmem<T, NB>*>(smem_raw);
    const int tid = threadIdx.x;
    T* Cs = C + (int64_t)blockIdx.x * RB * ldc;
    for (int e = tid; e < NB * RB; e += kT) {
        const int c = e / NB, r = e % NB;
        sm.C[r][c] = (r < n_valid) ? Cs[(int64_t)c * ldc + r] : T(0);
    }
    for (int rb = NB / RB - 1; rb >= 0; --rb) {
        const int r0 = rb * RB;
        for (int e = tid; e < RB * RB; e += kT) {
            const int c = e / RB, r = e % RB;
            T u = (r <= c) ? Rii[(int64_t)(r0 + c) * NB + r0 + r] : T(0);
            if (r0 + r >= n_valid) u = (r == c) ? T(1) : T(0);   // zero padding: unit diagonal
            if (r0 + c >= n_valid && r != c) u = T(0);
            sm.U[r][c] = u;
        }
        __syncthreads();
        if (tid < RB) {
            // column j = tid of U^-1: U y = e_j, y_r = 0 for r > j, back substitution upward
            const int j = tid;
            T y[RB];
#pragma unroll
            for (int r = RB - 1; r >= 0; --r) {
                T s = (r == j) ? T(1) : T(0);
#pragma unroll
                for (int c = r + 1; c < RB; ++c) s -= sm.U[r][c] * y[c];
                y[r] = (r <= j) ? s / sm.U[r][r] : T(0);
            }
#pragma unroll
            for (int r = 0; r < RB; ++r) sm.Ui[r][j] = y[r];
        }
        __syncthreads();
        // X_blk (32 x 32) = U^-1 C_blk: thread -> column c = tid % 32, rows rr = tid / 32 + 8 m
        {
            const int c = tid % RB, rr0 = tid / RB;
#pragma unroll
            for (int m = 0; m < RB / 8; ++m) {
                const int r = rr0 + 8 * m;
                T s = T(0);
#pragma unroll 8
                for (int kk = r; kk < RB; ++kk) s += sm.Ui[r][kk] * sm.C[r0 + kk][c];
                sm.X[r][c] = s;
            }
        }
        __syncthreads();
        for (int e = tid; e < RB * RB; e += kT) {
            const int r = e / RB, c = e % RB;
            sm.C[r0 + r][c] = sm.X[r][c];
        }
        // rows above the block inside the tile: C(0:r0, :) -= R_ii(0:r0, blk) X_blk
        for (int r = tid; r < r0; r += kT) {
            T acc[RB];
#pragma unroll
            for (int c = 0; c < RB; ++c) acc[c] = sm.C[r][c];
#pragma unroll 4
            for (int kk = 0; kk < RB; ++kk) {
                const T a = Rii[(int64_t)(r0 + kk) * NB + r];
#pragma unroll
                for (int c = 0; c < RB; ++c) acc[c] -= a * sm.X[kk][c];
            }
#pragma unroll
            for (int c = 0; c < RB; ++c) sm.C[r][c] = acc[c];
        }
        __syncthreads();
    }
    for (int e = tid; e < NB * RB; e += kT) {
        const int c = e / NB, r = e % NB;
        if (r < n_valid) Cs[(int64_t)c * ldc + r] = sm.C[r][c];
        else Cs[(int64_t)c * ldc + r] = T(0);
    }
}

// C(0:rows, slice) -= A(0:rows, 0:NB) X(0:NB, slice); A = column i's tiles 0..i-1 stacked (tile r at
// A + r*NB*NB, column-major, ld NB); X = rows i*NB.. of the workspace (ld ldc).
constexpr int UM = 128, UK = 32;
template <class T, int NB>
__global__ void __launch_bounds__(kT) trsm_update_kernel(const T* __restrict__ A, T* __restrict__ C,
                                                        const T* __restrict__ X, int64_t ldc, int rows) {
    __shared__ __align__(16) T As[UK][UM + 4];
    __shared__ __align__(16) T Xs[UK][RB + 1];
    const int tid = threadIdx.x;
    const int row0 = blockIdx.x * UM;                 // first output row
    const int64_t tile = (int64_t)NB * NB;
    T* Cs = C + (int64_t)blockIdx.y * RB * ldc;
    const T* Xsl = X + (int64_t)blockIdx.y * RB * ldc;
    const int tr = tid % 32, tc = tid / 32;          // rows tr + 32 a (a < 4), columns tc + 8 b (b < 4)
    T acc[4][4];
#pragma unroll
    for (int a = 0; a < 4; ++a)
#pragma unroll
        for (int b = 0; b < 4; ++b) acc[a][b] = T(0);
    for (int k0 = 0; k0 < NB; k0 += UK) {
        for (int e = tid; e < UK * UM; e += kT) {
            const int kk = e / UM, r = e % UM, gr = row0 + r;
            As[kk][r] = (gr < rows) ? A[(int64_t)(gr / NB) * tile + (int64_t)(k0 + kk) * NB + gr % NB] : T(0);
        }
        for (int e = tid; e < UK * RB; e += kT) {
            const int c = e / UK, kk = e % UK;
            Xs[kk][c] = Xsl[(int64_t)c * ldc + k0 + kk];
        }
        __syncthreads();
#pragma unroll 8
        for (int kk = 0; kk < UK; ++kk) {
            T av[4], xv[4];
#pragma unroll
            for (int a = 0; a < 4; ++a) av[a] = As[kk][tr + 32 * a];
#pragma unroll
            for (int b = 0; b < 4; ++b) xv[b] = Xs[kk][tc + 8 * b];
#pragma unroll
            for (int a = 0; a < 4; ++a)
#pragma unroll
                for (int b = 0; b < 4; ++b) acc[a][b] += av[a] * xv[b];
        }
        __syncthreads();
    }
#pragma unroll
    for (int b = 0; b < 4; ++b)
#pragma unroll
        for (int a = 0; a < 4; ++a) {
            const int gr = row0 + tr + 32 * a;
            if (gr < rows) Cs[(int64_t)(tc + 8 * b) * ldc + gr] -= acc[a][b];
        }
}

// first zero on the real diagonal of the column tiles [one CTA per local column]: tile (j, j) of
// local column lc at tiles + lc*colsz + j*NB*NB
template <class T>
__global__ void diag_zero_tiles_kernel(const T* __restrict__ tiles, const int32_t* __restrict__ cols, int64_t colsz,
                                       int nb, int64_t n, unsigned long long* first_zero) {
    const int lc = blockIdx.x;
    const int64_t j = cols[lc];
    const T* d = tiles + (int64_t)lc * colsz + j * (int64_t)nb * nb;
    for (int c = threadIdx.x; c < nb; c += blockDim.x) {
        const int64_t g = j * nb + c;
        if (g < n && d[(int64_t)c * nb + c] == T(0)) atomicMin(first_zero, (unsigned long long)g);
    }
}

template <class T, int NB>
cudaError_t diag_t(const T* Rii, T* C, int64_t ldc, int n_valid, int nslices, cudaStream_t s) {
    const size_t smem = sizeof(DiagSmem<T, NB>);
    auto kern = trsm_diag_kernel<T, NB>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    kern<<<nslices, kT, smem, s>>>(Rii, C, ldc, n_valid);
    return cudaGetLastError();
}

}  // namespace

template <class T>
cudaError_t launch_trsm_step(int nb, const T* Rcol, int i, T* C, int64_t ldc, int64_t n, int nslices,
                             cudaStream_t s) {
    if (nslices <= 0) return cudaSuccess;
    const int64_t tile = (int64_t)nb * nb;
    const int n_valid = (int)std::min<int64_t>(nb, n - (int64_t)i * nb);
    T* Ci = C + (int64_t)i * nb;
    cudaError_t e = cudaErrorInvalidValue;
#define TQR_DG(NB_) if (nb == NB_) e = diag_t<T, NB_>(Rcol + (int64_t)i * tile, Ci, ldc, n_valid, nslices, s);
    TQR_DG(64) TQR_DG(128) TQR_DG(256) TQR_DG(512)
#undef TQR_DG
    if (e != cudaSuccess || i == 0) return e;
    const int rows = i * nb;
    const dim3 grid((unsigned)((rows + UM - 1) / UM), (unsigned)nslices);
#define TQR_UP(NB_) if (nb == NB_) trsm_update_kernel<T, NB_><<<grid, kT, 0, s>>>(Rcol, C, Ci, ldc, rows);
    TQR_UP(64) TQR_UP(128) TQR_UP(256) TQR_UP(512)
#undef TQR_UP
    return cudaGetLastError();
}

template <class T>
cudaError_t launch_diag_zero_tiles(const T* tiles, const int32_t* cols_dev, int ncols, int64_t colsz, int nb, int64_t n,
                                   unsigned long long* first_zero, cudaStream_t s) {
    if (ncols <= 0) return cudaSuccess;
    diag_zero_tiles_kernel<T><<<ncols, 256, 0, s>>>(tiles, cols_dev, colsz, nb, n, first_zero);
    return cudaGetLastError();
}

template cudaError_t launch_trsm_step<double>(int, const double*, int, double*, int64_t, int64_t, int, cudaStream_t);
template cudaError_t launch_trsm_step<float>(int, const float*, int, float*, int64_t, int64_t, int, cudaStream_t);
template cudaError_t launch_diag_zero_tiles<double>(const double*, const int32_t*, int, int64_t, int, int64_t,
                                                    unsigned long long*, cudaStream_t);
template cudaError_t launch_diag_zero_tiles<float>(const float*, const int32_t*, int, int64_t, int, int64_t,
                                                   unsigned long long*, cudaStream_t);

}  // namespace tqr
