// common.cuh -- shared device helpers for the sm_100a tile kernels.
//
// FP64 tensor path on sm_100a: mma.sync.aligned.m8n8k4 f64 lowers to SASS DMMA.8x8x4 (there is
// no tcgen05 kind for f64).  Measured on this pool's B200 (profiles/r01_fp64_peak_probe.txt):
// 37.1 TFLOP/s chip-wide = 148 SM x 64 FMA/clk x 2 x 1.965 GHz, identical to the DFMA peak.
//
// Fragment layout (verified on the GPU by the same probe, layout_maxerr 0):
//   lane = 4*g + t  (g = lane>>2 in 0..7, t = lane&3 in 0..3)
//   A (8x4, M x K):  a = A[g][t]
//   B (4x8, K x N):  b = B[t][g]
//   C (8x8, M x N):  c0 = C[g][2t], c1 = C[g][2t+1]
//
// Register tile convention used by every kernel ("transposed accumulator"):
//   a CTA of 8 warps holds an NB x W column slice X of a tile; warp q owns rows
//   q*NB/8 .. q*NB/8 + NB/8 - 1; acc[mf][nf][e] = X[row = q*RW + nf*8 + 2t + e][col = mf*8 + g],
//   i.e. the C fragment of X^T (m = column, n = row).  The same registers are the A operand
//   of X^T * (.) when the contraction index k runs over rows {nf*8 + 2t + e}, t = 0..3
//   (a permutation of the K index, legal for a contraction), so no shared-memory transpose
//   is needed between the "W = V^T X" and "X -= V W" halves of a block-reflector apply.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <cstdio>

namespace tqr {

__device__ __forceinline__ void dmma(double& c0, double& c1, double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1},{%2},{%3},{%0,%1};"
                 : "+d"(c0), "+d"(c1) : "d"(a), "d"(b));
}

__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }
__device__ __forceinline__ int warp_id() { return threadIdx.x >> 5; }

// 16-byte aligned pair load/store (rows 2t, 2t+1 of one column: contiguous in column-major).
__device__ __forceinline__ double2 ld2(const double* p) { return *reinterpret_cast<const double2*>(p); }
__device__ __forceinline__ void st2(double* p, double x, double y) {
    *reinterpret_cast<double2*>(p) = make_double2(x, y);
}
// L2-only loads for data published by another CTA of the same grid (never stale in L1).
__device__ __forceinline__ double2 ld2_cg(const double* p) {
    double2 v;
    asm volatile("ld.global.cg.v2.f64 {%0,%1}, [%2];" : "=d"(v.x), "=d"(v.y) : "l"(p));
    return v;
}
__device__ __forceinline__ double ld_cg(const double* p) {
    double v;
    asm volatile("ld.global.cg.f64 %0, [%1];" : "=d"(v) : "l"(p));
    return v;
}

// cp.async (LDGSTS) 16-byte copies global -> shared, grouped per thread.  CG variant caches in
// L2 only (data published by sibling CTAs of the same grid is never stale in L1).
template <bool CG>
__device__ __forceinline__ void cp_async16(void* smem_dst, const void* gsrc) {
    const unsigned d = (unsigned)__cvta_generic_to_shared(smem_dst);
    if constexpr (CG)
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(gsrc) : "memory");
    else
        asm volatile("cp.async.ca.shared.global [%0], [%1], 16;" ::"r"(d), "l"(gsrc) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

// Bulk async copy engine (cp.async.bulk, SASS UBLKCP) with mbarrier completion.
__device__ __forceinline__ unsigned smem_u32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async_shared() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async_global() {
    asm volatile("fence.proxy.async.global;" ::: "memory");
}
// One thread: arm the barrier for `bytes` and launch the copy (16-byte aligned, bytes % 16 == 0).
__device__ __forceinline__ void bulk_g2s(void* smem_dst, const void* gsrc, unsigned bytes, uint64_t* bar) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_u32(smem_dst)), "l"(gsrc), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
#ifdef TQR_DEBUG_WAIT
__device__ __forceinline__ void mbar_wait(uint64_t* bar, unsigned parity) {
    unsigned ok = 0;
    for (long long spins = 0; !ok; ++spins) {
        asm volatile("{\n\t.reg .pred P;\n\tmbarrier.try_wait.parity.shared::cta.b64 P, [%1], %2;\n\t"
                     "selp.u32 %0, 1, 0, P;\n}" : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
        if (!ok && spins == (1ll << 22)) {
            printf("TQR_DEBUG_WAIT block %d warp %d mbarrier %p parity %u\n", blockIdx.x, threadIdx.x / 32,
                   (void*)bar, parity);
            __trap();
        }
    }
}
#else
__device__ __forceinline__ void mbar_wait(uint64_t* bar, unsigned parity) {
    asm volatile(
        "{\n\t.reg .pred P;\n"
        "WAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n\t"
        "@!P bra WAIT_%=;\n}" ::"r"(smem_u32(bar)), "r"(parity) : "memory");
}
#endif

// Inter-CTA flags (panel kernel wavefront).  Publisher: data stores, __threadfence, then a
// release store.  Consumer: acquire spin by one thread, fence, then __syncthreads.
__device__ __forceinline__ void flag_release(unsigned* f, unsigned v) {
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(f), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned flag_acquire(const unsigned* f) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(f) : "memory");
    return v;
}
__device__ __forceinline__ void flag_wait_geq(const unsigned* f, unsigned v) {
    if (threadIdx.x == 0) {
#ifdef TQR_DEBUG_WAIT
        long long spins = 0;
        while ((int)(flag_acquire(f) - v) < 0) {
            __nanosleep(64);
            if (++spins == (1ll << 24)) {
                printf("TQR_DEBUG_WAIT block %d flag %p value %u waiting for %u\n", blockIdx.x, (const void*)f,
                       flag_acquire(f), v);
                __trap();
            }
        }
#else
        while ((int)(flag_acquire(f) - v) < 0) __nanosleep(64);
#endif
        __threadfence();
    }
    __syncthreads();
}

}  // namespace tqr
