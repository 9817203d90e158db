#include <cstdio>
__device__ __forceinline__ unsigned long long pk(float a, float b){ unsigned long long r; asm("mov.b64 %0, {%1,%2};" : "=l"(r) : "f"(a), "f"(b)); return r;}
__device__ __forceinline__ unsigned long long ffma2(unsigned long long a, unsigned long long b, unsigned long long c){ unsigned long long d; asm volatile("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c)); return d;}
__device__ __forceinline__ unsigned long long fmul2(unsigned long long a, unsigned long long b){ unsigned long long d; asm volatile("mul.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b)); return d;}
__device__ __forceinline__ unsigned long long fadd2(unsigned long long a, unsigned long long b){ unsigned long long d; asm volatile("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b)); return d;}
__global__ void k2(float* out, int iters, float s){
  unsigned long long a[8]; unsigned long long b = pk(s, s*1.0001f), c = pk(0.999f, 0.998f);
  for(int i=0;i<8;i++) a[i]=pk(threadIdx.x*1e-3f+i, i*0.5f);
  for(int it=0; it<iters; it++){
#pragma unroll
    for(int i=0;i<8;i++) a[i]=ffma2(a[i],b,c);
  }
  float acc=0; for(int i=0;i<8;i++){ float x,y; asm("mov.b64 {%0,%1}, %2;" : "=f"(x),"=f"(y):"l"(a[i])); acc+=x+y;}
  out[blockIdx.x*blockDim.x+threadIdx.x]=acc;
}
__global__ void k1(float* out, int iters, float s){
  float a[16]; float b=s, c=0.999f;
  for(int i=0;i<16;i++) a[i]=threadIdx.x*1e-3f+i;
  for(int it=0; it<iters; it++){
#pragma unroll
    for(int i=0;i<16;i++) a[i]=fmaf(a[i],b,c);
  }
  float acc=0; for(int i=0;i<16;i++) acc+=a[i];
  out[blockIdx.x*blockDim.x+threadIdx.x]=acc;
}
__global__ void krcp(float* out, int iters, float s){
  float a[8]; for(int i=0;i<8;i++) a[i]=threadIdx.x*1e-3f+i+1.5f;
  for(int it=0; it<iters; it++){
#pragma unroll
    for(int i=0;i<8;i++){ float r; asm volatile("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(a[i])); a[i]=r+s; }
  }
  float acc=0; for(int i=0;i<8;i++) acc+=a[i];
  out[blockIdx.x*blockDim.x+threadIdx.x]=acc;
}
int main(){
  float* d; cudaMalloc(&d, 148*64*1024*4);
  cudaEvent_t e0,e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  int iters=20000; int blocks=148*8, threads=256;
  for(int rep=0;rep<2;rep++){
  k1<<<blocks,threads>>>(d,100,1.0f); cudaDeviceSynchronize();
  cudaEventRecord(e0); k1<<<blocks,threads>>>(d,iters,1.0f); cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms,e0,e1);
  double fmas=(double)blocks*threads*iters*16;
  printf("scalar FFMA: %.3f ms, %.2f TFMA-lane/s -> per SM per clk @1965: %.1f\n", ms, fmas/ms/1e9, fmas/(ms*1e-3)/148/1.965e9);
  k2<<<blocks,threads>>>(d,100,1.0f); cudaDeviceSynchronize();
  cudaEventRecord(e0); k2<<<blocks,threads>>>(d,iters,1.0f); cudaEventRecord(e1); cudaEventSynchronize(e1);
  cudaEventElapsedTime(&ms,e0,e1);
  fmas=(double)blocks*threads*iters*16;
  printf("FFMA2: %.3f ms, %.2f TFMA-lane/s -> per SM per clk @1965: %.1f\n", ms, fmas/ms/1e9, fmas/(ms*1e-3)/148/1.965e9);
  krcp<<<blocks,threads>>>(d,100,1.0f); cudaDeviceSynchronize();
  cudaEventRecord(e0); krcp<<<blocks,threads>>>(d,iters,1.0f); cudaEventRecord(e1); cudaEventSynchronize(e1);
  cudaEventElapsedTime(&ms,e0,e1);
  fmas=(double)blocks*threads*iters*8;
  printf("RCP(+FADD): %.3f ms, %.2f Trcp/s -> per SM per clk @1965: %.1f\n", ms, fmas/ms/1e9, fmas/(ms*1e-3)/148/1.965e9);
  }
  return 0;
}
