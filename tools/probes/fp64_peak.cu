// Probe: FP64 DMMA (mma.sync m8n8k4 f64) vs DFMA throughput on sm_100a, plus the
// m8n8k4 f64 fragment-layout check used by the tile kernels. Standalone, not product code.
#include <cstdio>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("CUDA %s @%d\n",cudaGetErrorString(e),__LINE__);return 1;}}while(0)

__device__ __forceinline__ void dmma(double& d0,double& d1,double a,double b){
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1},{%2},{%3},{%0,%1};"
               :"+d"(d0),"+d"(d1):"d"(a),"d"(b));
}
template<int NACC>
__global__ void k_dmma(double* out, int iters, double a, double b){
  double acc[NACC][2];
  #pragma unroll
  for(int i=0;i<NACC;i++){acc[i][0]=threadIdx.x; acc[i][1]=i;}
  double av=a+threadIdx.x*1e-9, bv=b;
  for(int it=0;it<iters;it++){
    #pragma unroll
    for(int i=0;i<NACC;i++) dmma(acc[i][0],acc[i][1],av,bv);
  }
  double s=0;
  #pragma unroll
  for(int i=0;i<NACC;i++) s+=acc[i][0]+acc[i][1];
  if(s==1.2345) out[0]=s;
}
template<int NACC>
__global__ void k_dfma(double* out, int iters, double a, double b){
  double acc[NACC];
  #pragma unroll
  for(int i=0;i<NACC;i++) acc[i]=threadIdx.x+i;
  double av=a+threadIdx.x*1e-9;
  for(int it=0;it<iters;it++){
    #pragma unroll
    for(int i=0;i<NACC;i++) acc[i]=fma(acc[i],av,b);
  }
  double s=0;
  #pragma unroll
  for(int i=0;i<NACC;i++) s+=acc[i];
  if(s==1.2345) out[0]=s;
}
// layout check: A[m][k]=m*10+k+1 (8x4), B[k][n]=(k+1)*0.5+n*100 (4x8); C=0
__global__ void k_layout(double* D, int* ok){
  int lane=threadIdx.x, g=lane>>2, t=lane&3;
  double a = g*10 + t + 1;            // A[g][t]
  double b = (t+1)*0.5 + g*100;        // B[t][g]
  double d0=0,d1=0;
  dmma(d0,d1,a,b);
  D[g*8+2*t]=d0; D[g*8+2*t+1]=d1;     // hypothesis: D[g][2t], D[g][2t+1]
}
int main(){
  double* out; CK(cudaMalloc(&out,64*8));
  int* ok; CK(cudaMalloc(&ok,4));
  k_layout<<<1,32>>>(out,ok); CK(cudaDeviceSynchronize());
  double h[64]; CK(cudaMemcpy(h,out,512,cudaMemcpyDeviceToHost));
  double maxerr=0;
  for(int m=0;m<8;m++)for(int n=0;n<8;n++){double e=0;for(int k=0;k<4;k++)e+=(m*10+k+1)*((k+1)*0.5+n*100);
    double d=h[m*8+n]-e; if(d<0)d=-d; if(d>maxerr)maxerr=d;}
  printf("layout_maxerr %g\n",maxerr);
  int dev; cudaGetDevice(&dev); cudaDeviceProp p; cudaGetDeviceProperties(&p,dev);
  printf("dev %s sms %d clock_khz %d\n",p.name,p.multiProcessorCount,p.clockRate);
  cudaEvent_t e0,e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  int iters=20000;
  for(int wpb: {4,8,16}){
    for(int bps: {1,2,4}){
      int blocks=p.multiProcessorCount*bps;
      k_dmma<8><<<blocks,wpb*32>>>(out,100,1.0,1e-3);
      cudaEventRecord(e0);
      k_dmma<8><<<blocks,wpb*32>>>(out,iters,1.0,1e-3);
      cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
      float ms; cudaEventElapsedTime(&ms,e0,e1);
      double fl=2.0*256*8*(double)iters*wpb*blocks;
      printf("DMMA warps/blk %d blk/sm %d : %.2f TFLOP/s (%.3f ms)\n",wpb,bps,fl/ms/1e9,ms);
    }
  }
  for(int wpb: {8,16,32}){
    int blocks=p.multiProcessorCount*2;
    k_dfma<16><<<blocks,wpb*32>>>(out,100,1.0,1e-3);
    cudaEventRecord(e0);
    k_dfma<16><<<blocks,wpb*32>>>(out,iters,1.0,1e-3);
    cudaEventRecord(e1); CK(cudaEventSynchronize(e1));
    float ms; cudaEventElapsedTime(&ms,e0,e1);
    double fl=2.0*16*(double)iters*wpb*32*blocks;
    printf("DFMA warps/blk %d blk/sm 2 : %.2f TFLOP/s\n",wpb,fl/ms/1e9);
  }
  // single-SM rates
  k_dmma<8><<<1,256>>>(out,iters,1.0,1e-3);
  cudaEventRecord(e0); k_dmma<8><<<1,256>>>(out,iters,1.0,1e-3); cudaEventRecord(e1); cudaEventSynchronize(e1);
  { float ms; cudaEventElapsedTime(&ms,e0,e1); printf("DMMA 1 SM 8 warps: %.1f GFLOP/s\n",2.0*256*8*(double)iters*8/ms/1e6);}
  return 0;
}
