// Dependent-chain latency (cycles per op, one warp) of the FP64 operations on factor_block's
// column-step critical path: DFMA, DADD, sqrt, division, reciprocal, rsqrt, a shuffle of a double.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o fp64_latency fp64_latency.cu && ./fp64_latency
#include <cstdio>
#include <cuda_runtime.h>

template <int OP>
__global__ void chain(double* out, double x0, long long* cyc) {
    double x = x0 + threadIdx.x * 1e-9, y = 1.0000001;
    const int N = 1024;
    long long t0 = clock64();
#pragma unroll 16
    for (int i = 0; i < N; ++i) {
        if (OP == 0) x = fma(x, y, 1e-300);
        if (OP == 1) x = x + 1e-300;
        if (OP == 2) x = sqrt(x) + 1.0;            // keeps x ~ 2.6
        if (OP == 3) x = 3.0 / x + 0.5;            // keeps x bounded
        if (OP == 4) x = __drcp_rn(x) + 0.5;
        if (OP == 5) x = rsqrt(x) + 1.0;
        if (OP == 6) x = __shfl_xor_sync(0xffffffffu, x, 1) + 1e-300;
        if (OP == 7) x = __dsqrt_rn(x) + 1.0;
        if (OP == 8) x = __ddiv_rn(3.0, x) + 0.5;
    }
    long long t1 = clock64();
    out[threadIdx.x] = x;
    if (threadIdx.x == 0) *cyc = t1 - t0;
}

int main() {
    double* out; long long* cyc; long long h;
    cudaMalloc(&out, 32 * 8); cudaMalloc(&cyc, 8);
    const char* names[] = {"DFMA", "DADD", "sqrt", "3.0/x", "__drcp_rn", "rsqrt", "shfl f64 + DADD", "__dsqrt_rn", "__ddiv_rn"};
#define RUN(OP) chain<OP><<<1, 32>>>(out, 2.0, cyc); chain<OP><<<1, 32>>>(out, 2.0, cyc); cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost); \
    printf("%-18s %7.1f cycles/op (incl. the + where shown)\n", names[OP], h / 1024.0);
    RUN(0) RUN(1) RUN(2) RUN(3) RUN(4) RUN(5) RUN(6) RUN(7) RUN(8)
    return 0;
}
