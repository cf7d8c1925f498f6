// tqr_signal.cu -- stream-ordered 64-bit flags for the CUDA-IPC panel transport (tqr_api.cpp).
//
// The multi-process transport (tqr_options.transport = TQR_TRANSPORT_IPC) moves panel k's V/T
// with plain device-to-device copies into the receivers' IPC-mapped slots (NVLink peer memory
// on a multi-GPU node, the same HBM for several processes on one GPU) and orders producer and
// consumer with monotone 64-bit flags: a stream writes a flag after the work it guards, another
// process's stream waits until the flag reaches a value.  Every wait is on the waiting rank's own
// memory; writes may target peer memory.
//
// Preferred mechanism: the driver's stream memory operations (cuStreamWaitValue64 /
// cuStreamWriteValue64, resolved with cudaGetDriverEntryPoint so the library keeps linking only
// the static runtime): the wait is performed by the GPU front end and occupies no SM, so it can
// never starve a kernel of another process time-sliced on the same GPU.  Fallback (entry points
// missing, or TQR_SIGNAL=kernel): one-warp kernels with st.release.sys / ld.acquire.sys spins.
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include "tqr_internal.h"

namespace tqr {

namespace {

using WaitFn = CUresult (*)(CUstream, CUdeviceptr, cuuint64_t, unsigned int);
using WriteFn = CUresult (*)(CUstream, CUdeviceptr, cuuint64_t, unsigned int);
using Wait32Fn = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);

struct MemOps {
    bool tried = false;
    WaitFn wait = nullptr;
    WriteFn write = nullptr;
    Wait32Fn wait32 = nullptr;
};

MemOps& memops() {
    static MemOps m;
    if (!m.tried) {
        m.tried = true;
        const char* e = getenv("TQR_SIGNAL");
        if (e && strcmp(e, "kernel") == 0) return m;
        void* fw = nullptr;
        void* fr = nullptr;
        cudaDriverEntryPointQueryResult q1 = cudaDriverEntryPointSymbolNotFound, q2 = cudaDriverEntryPointSymbolNotFound;
        if (cudaGetDriverEntryPoint("cuStreamWaitValue64", &fw, cudaEnableDefault, &q1) == cudaSuccess &&
            cudaGetDriverEntryPoint("cuStreamWriteValue64", &fr, cudaEnableDefault, &q2) == cudaSuccess &&
            q1 == cudaDriverEntryPointSuccess && q2 == cudaDriverEntryPointSuccess && fw && fr) {
            m.wait = reinterpret_cast<WaitFn>(fw);
            m.write = reinterpret_cast<WriteFn>(fr);
            void* f32 = nullptr;
            cudaDriverEntryPointQueryResult q3 = cudaDriverEntryPointSymbolNotFound;
            if (cudaGetDriverEntryPoint("cuStreamWaitValue32", &f32, cudaEnableDefault, &q3) == cudaSuccess &&
                q3 == cudaDriverEntryPointSuccess && f32)
                m.wait32 = reinterpret_cast<Wait32Fn>(f32);
        }
        cudaGetLastError();
    }
    return m;
}

__global__ void sig_write_kernel(uint64_t* addr, uint64_t v) {
    __threadfence_system();
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(addr), "l"(v) : "memory");
}

__global__ void sig_wait_kernel(const uint64_t* addr, uint64_t v) {
    if (threadIdx.x == 0) {
        for (;;) {
            uint64_t x;
            asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(x) : "l"(addr) : "memory");
            if ((int64_t)(x - v) >= 0) break;
            __nanosleep(256);
        }
        __threadfence_system();
    }
}

__global__ void sig_wait32_kernel(const unsigned* addr, unsigned v) {
    if (threadIdx.x == 0) {
        for (;;) {
            unsigned x;
            asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(x) : "l"(addr) : "memory");
            if ((int)(x - v) >= 0) break;
            __nanosleep(256);
        }
        __threadfence_system();
    }
}

}  // namespace

bool signal_uses_memops() { return memops().wait != nullptr; }

cudaError_t sig_wait_geq32(cudaStream_t s, const unsigned* addr, unsigned v) {
    MemOps& m = memops();
    if (m.wait32) {
        return m.wait32((CUstream)s, (CUdeviceptr)addr, (cuuint32_t)v, CU_STREAM_WAIT_VALUE_GEQ) == CUDA_SUCCESS
                   ? cudaSuccess : cudaErrorUnknown;
    }
    sig_wait32_kernel<<<1, 32, 0, s>>>(addr, v);
    return cudaGetLastError();
}

cudaError_t sig_write(cudaStream_t s, uint64_t* addr, uint64_t v) {
    MemOps& m = memops();
    if (m.write) {
        // default flags: the write is ordered after (and its memory barrier covers) all prior work
        return m.write((CUstream)s, (CUdeviceptr)addr, (cuuint64_t)v, CU_STREAM_WRITE_VALUE_DEFAULT) == CUDA_SUCCESS
                   ? cudaSuccess : cudaErrorUnknown;
    }
    sig_write_kernel<<<1, 1, 0, s>>>(addr, v);
    return cudaGetLastError();
}

cudaError_t sig_wait_geq(cudaStream_t s, const uint64_t* addr, uint64_t v) {
    MemOps& m = memops();
    if (m.wait) {
        return m.wait((CUstream)s, (CUdeviceptr)addr, (cuuint64_t)v, CU_STREAM_WAIT_VALUE_GEQ) == CUDA_SUCCESS
                   ? cudaSuccess : cudaErrorUnknown;
    }
    sig_wait_kernel<<<1, 32, 0, s>>>(addr, v);
    return cudaGetLastError();
}

}  // namespace tqr
