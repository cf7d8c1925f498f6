// tqr_internal.h -- kernel argument blocks and launchers shared by the host runtime (tqr_api.cpp)
// and the sm_100a kernels (kernels/qr_kernels.cu).  Not part of the public ABI.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace tqr {

// Panel step k on the owner of column k: GEQRT(k,k) + TSQRT(i,k), i = k+1..p-1.
struct PanelArgs {
    double* col;       // the owner's tiles of column k: tile i at col + i*nb*nb (column-major nb x nb)
    double* T;         // T factors of column k: tile i at T + i*ib*nb (ib x nb, LAPACK dgeqrt layout)
    double* Vimg;      // stage images of column k's reflector tiles: tile i at Vimg + i*nb*nb (TSQRT writes)
    double* Vexp;      // stage image of the explicit unit-lower V of the diagonal tile (GEQRT writes)
    unsigned* flags;   // p * (nb/ib) * (1 + split) publication flags (F, then G)
    unsigned epoch;    // value published for this launch (monotone across launches)
    int k;             // step (tile column / diagonal tile row)
    int p;             // number of row tiles
    double* top = nullptr;   // TS "top" tile override (null: col + k*nb*nb)
    int skip_ge = 0;         // 1: tile k is already triangular (a merge chain): TSQRT tiles k+1..p-1 only
    int L = 0;               // > 0: multi-job (tree mode) -- job d = domain [k + d*L, min(k + (d+1)*L, p)),
                             //      head d's explicit V image in Vexp (d = 0) or Vimg slot k + d*L;
                             //      with skip_ge (merge groups) the top override applies to job 0 only,
                             //      job d > 0 merges into its own head slot
    int fslots = 0;          // > 0: slot rows of the F flag block (G flags follow it); 0 = p
    int stride = 1;          // chain index i addresses slot i*stride of col / T / Vimg / flags (the
                             //      second level of a two-level merge walks the group heads)
};

// TS-domain step (NEXT-1 tree; paper's TT elimination P:L409-419): one CTA per domain
// [k + d*L, min(k + (d+1)*L, p)) of panel column k: GEQRT of the domain head, then TSQRT of the
// domain's other tiles against it.  Head d's explicit V image goes to Vexp (d = 0) or to the
// head tile's own image slot (d > 0); its T to the head tile's T slot.
struct DomainArgs {
    double* col;
    double* T;
    double* Vimg;
    double* Vexp;
    int k, p, L;
    int dom0 = 0;      // first domain of this launch (CTA x factors domain dom0 + x)
};
cudaError_t launch_domains(int nb, int ib, const DomainArgs& a, int ndom, cudaStream_t s);
// merge inputs: Mt[e] = triu(tile k + e*L) (zeros below the diagonal), e = 1..ndom-1
cudaError_t launch_merge_prep(int nb, const double* col, double* Mt, int k, int L, int ndom, cudaStream_t s);

// Trailing update of step k over `ngroups` column groups (UNMQR + TSMQR chain), or the
// application of panel k's Q^T / Q to a right-hand side block (tqr_apply_qt).  T = element type.
template <class E>
struct UpdateArgsT {
    const E* V;          // stage images of panel k's reflector tiles (tile i at V + i*image tile, i > k used)
    const E* Vexp;       // stage image of the explicit V of the diagonal tile
    const E* T;          // T factors: tile i at T + i*ib*nb
    E* X;                // target: element (tile i, r, c) of group gidx at
                         //   X + gidx*col_stride + i*tile_stride + c*ld + r
    int64_t col_stride;
    int64_t tile_stride;
    int64_t ld;
    int group0;          // first group index
    int gstride;         // group index step between consecutive groups of this launch
    int k, p;
    int do_unmqr;        // 1: apply Q_kk (UNMQR) to row tile k as well
    int vstride = 1;     // reflector tile i at V + i*vstride*image tile, T + i*vstride*ib*nb
    // FP64 lookahead overlapped with its panel: before reading reflector tile i (i = k for UNMQR),
    // wait until the panel kernel has published F(i, last ib block) >= wepoch (every block of tile
    // i then is, by the panel's release/acquire chain); null = the stream dependency suffices
    const unsigned* wflags = nullptr;
    unsigned wepoch = 0;
    // Lookahead trailing a REMOTE panel (another owner's): before reading reflector tile i, wait
    // until the chunk flag cflags[(i - k) / cchunk] (64-bit, in this owner's memory, raised by the
    // transfer of that chunk of tiles into the receive slot) is >= cval; null = not trailing
    const unsigned long long* cflags = nullptr;
    unsigned long long cval = 0;
    int cchunk = 1;
    // FP64 wavefront apply of nsteps consecutive panels in one launch (tqr_apply_qt / solve_ls,
    // single owner, flat tree): grid = nsteps * nslc CTAs, step offset st = CTA / nslc processes
    // step k +- st (TRANS: +) with V, T, Vexp advanced by st * (vcol, tcol, ecol) elements; prog
    // (nsteps * nslc, zeroed) counts the chain tiles each CTA has finished
    int nsteps = 1;
    int nslc = 0;                        // slices per step (nsteps > 1) or per job (domL > 0)
    int domL = 0;                        // > 0: tree jobs of domL row tiles (see update_kernel)
    int64_t vcol = 0, tcol = 0, ecol = 0;
    unsigned* prog = nullptr;
    // FP64, W = 32, nb >= 256, plain Q^T chain: run update_kernel16 (the slice over 16 warps,
    // tile_w16.cuh) instead of the 8-warp update_kernel
    int w16 = 0;
};
using UpdateArgs = UpdateArgsT<double>;

// split = apply CTAs per ib column block (1, 2, 4): grid = (nb/ib) * (split + 1)
cudaError_t launch_panel(int nb, int ib, int split, const PanelArgs& a, cudaStream_t s, int njobs = 1);
// nslices CTAs; CTA b works on columns [b*w, b*w + w) counted from group0 (groups are nb wide)
cudaError_t launch_update(int nb, int ib, int w, const UpdateArgs& a, int nslices, bool trans, cudaStream_t s);
// a1: src column group of local column lc at src + (local_src ? lc : cols[lc])*src_group_stride
// (ld = lda) -> tiles at dst + lc*dst_col_stride; rows >= m_valid and global columns >= n_valid -> 0
template <class T>
cudaError_t launch_to_tiles(const T* src, int64_t lda, int64_t src_group_stride, T* dst, const int32_t* cols_dev,
                            int local_src, int ncols, int64_t dst_col_stride, int nb, int p, int64_t m_valid,
                            int64_t n_valid, cudaStream_t s);
// a8: tiles -> column-major rows [0, m_rows) of global columns < n_valid, zeros below the diagonal
// (global column group of local column lc is cols[lc]); destination group at
// dst + (local_dst ? lc : cols[lc])*dst_group_stride
template <class T>
cudaError_t launch_from_tiles(T* dst, int64_t lda, int64_t dst_group_stride, const T* src, const int32_t* cols_dev,
                              int ncols, int64_t src_col_stride, int nb, int64_t m_rows, int64_t n_valid,
                              int local_dst, cudaStream_t s);
// zero (r, c) with r % nb > c in a rows x cols column-major block stack (ld)
template <class T>
cudaError_t launch_zero_below_blocks(T* a, int64_t ld, int64_t rows, int64_t cols, int nb, cudaStream_t s);
// Step i of the tile back substitution (trsm.cu): X_i = R_ii^-1 C_i, then C_r -= R_ri X_i, r < i.
// Rcol = column tile i of R in tile storage (tile r at Rcol + r*nb*nb); C = mp x 32*nslices, ld ldc.
template <class T>
cudaError_t launch_trsm_step(int nb, const T* Rcol, int i, T* C, int64_t ldc, int64_t n, int nslices, cudaStream_t s);
// atomicMin of the first global diagonal index g < n with R(g, g) == 0 over the owned column tiles
template <class T>
cudaError_t launch_diag_zero_tiles(const T* tiles, const int32_t* cols_dev, int ncols, int64_t colsz, int nb, int64_t n,
                                   unsigned long long* first_zero, cudaStream_t s);

// ---- FP32 path (kernels/qr_kernels_f32.cu)
// FFMA trailing update; V / Vexp are FP32 stage images (f32_img_tile elements per tile)
cudaError_t launch_update_f32(int nb, int ib, int w, const UpdateArgsT<float>& a, int nslices, bool trans,
                              cudaStream_t s);
// FP32 -> FP64 copy of n elements (n % 4 == 0, 16-byte aligned)
cudaError_t launch_widen(const float* src, double* dst, int64_t n, cudaStream_t s);
// FP64 panel result of step k (scratch column sc, T64) -> FP32 tiles, T and stage images
cudaError_t launch_narrow_panel(int nb, int ib, const double* sc, const double* T64, float* tiles, float* T32,
                                float* Vimg, float* Vexp, int k, int p, cudaStream_t s);
int64_t f32_img_tile(int nb, int ib);

// ---- stream-ordered 64-bit flags of the CUDA-IPC transport (tqr_signal.cu)
// *addr = v after all prior work of s (addr may be peer / IPC-mapped memory)
cudaError_t sig_write(cudaStream_t s, uint64_t* addr, uint64_t v);
// later work of s waits until (int64_t)(*addr - v) >= 0 (addr: this process's device memory)
cudaError_t sig_wait_geq(cudaStream_t s, const uint64_t* addr, uint64_t v);
// 32-bit variant (the panel kernel's publication flags): later work waits until (int32_t)(*addr - v) >= 0
cudaError_t sig_wait_geq32(cudaStream_t s, const unsigned* addr, unsigned v);
bool signal_uses_memops();
size_t panel_smem_bytes(int nb, int ib);
size_t update_smem_bytes(int nb, int ib, int w);

}  // namespace tqr
