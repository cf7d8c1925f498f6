// Probe: FP32 FFMA peak (the roofline denominator of the FP32 path) and, for context, legacy
// mma.sync m16n8k8 TF32 throughput on sm_100a.  Standalone, not product code.
#include <cstdio>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("CUDA %s @%d\n",cudaGetErrorString(e),__LINE__);return 1;}}while(0)

template<int NACC>
__global__ void k_ffma(float* out, int iters, float a, float b){
  float acc[NACC];
  #pragma unroll
  for(int i=0;i<NACC;i++) acc[i]=threadIdx.x+i;
  float av=a+threadIdx.x*1e-7f;
  for(int it=0;it<iters;it++){
    #pragma unroll
    for(int i=0;i<NACC;i++) acc[i]=fmaf(acc[i],av,b);
  }
  float s=0;
  #pragma unroll
  for(int i=0;i<NACC;i++) s+=acc[i];
  if(s==1.2345f) out[0]=s;
}
__device__ __forceinline__ void mma_tf32(float (&d)[4], const unsigned (&a)[4], const unsigned (&b)[2]){
  asm volatile("mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3},{%4,%5,%6,%7},{%8,%9},{%0,%1,%2,%3};"
    :"+f"(d[0]),"+f"(d[1]),"+f"(d[2]),"+f"(d[3]):"r"(a[0]),"r"(a[1]),"r"(a[2]),"r"(a[3]),"r"(b[0]),"r"(b[1]));
}
template<int NACC>
__global__ void k_tf32(float* out, int iters){
  float acc[NACC][4];
  #pragma unroll
  for(int i=0;i<NACC;i++) for(int j=0;j<4;j++) acc[i][j]=0.f;
  unsigned a[4]={0x3f800000u+threadIdx.x,0x3f800000u,0x3f800000u,0x3f800000u}, b[2]={0x3f800000u,0x3f800000u};
  for(int it=0;it<iters;it++){
    #pragma unroll
    for(int i=0;i<NACC;i++) mma_tf32(acc[i],a,b);
  }
  float s=0;
  #pragma unroll
  for(int i=0;i<NACC;i++) s+=acc[i][0]+acc[i][3];
  if(s==1.2345f) out[0]=s;
}
int main(){
  float* out; CK(cudaMalloc(&out,64));
  int dev; cudaGetDevice(&dev); cudaDeviceProp p; cudaGetDeviceProperties(&p,dev);
  printf("dev %s sms %d\n",p.name,p.multiProcessorCount);
  cudaEvent_t e0,e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  int iters=20000;
  for(int wpb: {8,16,32}) for(int bps: {1,2}){
    int blocks=p.multiProcessorCount*bps;
    k_ffma<16><<<blocks,wpb*32>>>(out,100,1.0f,1e-3f);
    cudaEventRecord(e0); k_ffma<16><<<blocks,wpb*32>>>(out,iters,1.0f,1e-3f); cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
    float ms; cudaEventElapsedTime(&ms,e0,e1);
    printf("FFMA warps/blk %d blk/sm %d : %.2f TFLOP/s\n",wpb,bps,2.0*16*(double)iters*wpb*32*blocks/ms/1e9);
  }
  for(int wpb: {4,8,16}){
    int blocks=p.multiProcessorCount*2;
    k_tf32<8><<<blocks,wpb*32>>>(out,100);
    cudaEventRecord(e0); k_tf32<8><<<blocks,wpb*32>>>(out,iters); cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
    float ms; cudaEventElapsedTime(&ms,e0,e1);
    printf("mma.sync TF32 m16n8k8 warps/blk %d blk/sm 2 : %.2f TFLOP/s\n",wpb,2.0*16*8*8*8*(double)iters*wpb*blocks/ms/1e9);
  }
  return 0;
}
