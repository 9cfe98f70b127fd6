// Microbenchmark: FP32 issue throughput of FFMA (3-register form) vs FFMA2 (f32x2) on sm_100a.
// Each thread runs 8 independent dependency chains; reports lane-FMA/clk/SM.
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ unsigned long long pk(float a, float b){unsigned long long r; asm("mov.b64 %0,{%1,%2};":"=l"(r):"f"(a),"f"(b)); return r;}
__device__ __forceinline__ float2 upk(unsigned long long r){float a,b; asm("mov.b64 {%0,%1},%2;":"=f"(a),"=f"(b):"l"(r)); return make_float2(a,b);}
template<int MODE>
__global__ void k(float* out, float s, float t, int iters){
  float a[16]; unsigned long long p[8];
  for(int i=0;i<16;i++) a[i]=threadIdx.x*1e-3f+i;
  for(int i=0;i<8;i++) p[i]=pk(a[2*i],a[2*i+1]);
  unsigned long long S=pk(s,s), T=pk(t,t);
  float ss=s*(1+threadIdx.x), tt=t-threadIdx.x;
  for(int it=0; it<iters; it++){
    #pragma unroll
    for(int i=0;i<16;i++){
      if(MODE==0){ a[i]=fmaf(a[i],ss,tt); }
      else if(MODE==1){ if(i<8) asm volatile("fma.rn.f32x2 %0,%0,%1,%2;":"+l"(p[i]):"l"(S),"l"(T)); }
      else if(MODE==2){ if(i<8) asm volatile("add.rn.f32x2 %0,%0,%1;":"+l"(p[i]):"l"(T)); }
      else { a[i]=a[i]+tt; }
    }
  }
  float r=0; for(int i=0;i<16;i++) r+=a[i]; for(int i=0;i<8;i++){float2 q=upk(p[i]); r+=q.x+q.y;}
  out[blockIdx.x*blockDim.x+threadIdx.x]=r;
}
template<int M> void run(const char* name, float* d, int blocks, int threads){
  int iters=4096; cudaEvent_t e0,e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  k<M><<<blocks,threads>>>(d,1.0001f,0.5f,iters);
  cudaEventRecord(e0); k<M><<<blocks,threads>>>(d,1.0001f,0.5f,iters); cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms,e0,e1);
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  double lane_ops = (double)blocks*threads*iters*16;
  printf("%-6s threads/blk=%d: %.3f ms, %.1f Tlane-op/s (%.1f lane-op/clk/SM @ %.0f MHz nominal)\n", name, threads, ms,
         lane_ops/ms/1e9, lane_ops/(ms*1e-3)/148/(clk*1e3), clk/1e3);
}
int main(){ float* d; cudaMalloc(&d, 148*8*1024*4);
  for(int th: {256, 512, 1024}){ run<0>("FFMA",d,148*2,th); run<1>("FFMA2",d,148*2,th); run<3>("FADD",d,148*2,th); run<2>("FADD2",d,148*2,th);} return 0; }
