#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ float2 f2(float v){return make_float2(v,v);}
__device__ __forceinline__ float rcpa(float x){float r; asm("rcp.approx.ftz.f32 %0,%1;":"=f"(r):"f"(x)); return r;}
template<int KP, int MODE>
__global__ void __launch_bounds__(128, 4) k(float* out, int n, float r2min, float rc2, float c){
  float2 X[KP],Y[KP],Z[KP],Q[KP],A[KP],B[KP];
  for(int p=0;p<KP;p++){X[p]=make_float2(threadIdx.x*1e-3f+p, p*0.5f); Y[p]=make_float2(p*0.3f,1.f); Z[p]=make_float2(0.2f,p*0.1f); Q[p]=A[p]=B[p]=make_float2(0,0);}
  const float INF=__int_as_float(0x7f800000);
  float4 xq=make_float4(0.1f,0.2f,0.3f,0.4f), pp=make_float4(1.f,2.f,0,0);
  #pragma unroll 2
  for(int j=0;j<n;j++){
    xq.x += 0.001f; xq.y -= 0.0007f;
    #pragma unroll
    for(int p=0;p<KP;p++){
      float2 r2;
      if (MODE>=10){ float2 t=__fadd2_rn(Q[p], f2(xq.y)); t=__ffma2_rn(X[p],f2(xq.x),t); t=__ffma2_rn(Y[p],f2(xq.y),t); r2=__ffma2_rn(Z[p],f2(xq.z),t);} else {
      float2 dx=__fadd2_rn(X[p],f2(-xq.x)), dy=__fadd2_rn(Y[p],f2(-xq.y)), dz=__fadd2_rn(Z[p],f2(-xq.z));
      r2=__fmul2_rn(dx,dx); r2=__ffma2_rn(dy,dy,r2); r2=__ffma2_rn(dz,dz,r2);}
      if (MODE>=1){ r2.x=fmaxf(r2.x,r2min); r2.y=fmaxf(r2.y,r2min);}
      float2 r2u=r2; bool ix=true, iy=true;
      if (MODE>=2 && MODE!=6 && MODE!=10){ ix=r2.x<rc2; iy=r2.y<rc2; r2.x=ix?r2.x:INF; r2.y=iy?r2.y:INF; }
      float2 inv; inv.x=rcpa(r2.x); inv.y=rcpa(r2.y);
      float2 es=inv;
      if (MODE==2){ es=__fadd2_rn(__ffma2_rn(r2u,f2(c*c),inv),f2(-2.f*c)); es.x=ix?es.x:0.f; es.y=iy?es.y:0.f; }
      if (MODE==3){ float2 sh=__ffma2_rn(r2u,f2(-c),f2(1.f)); es=__fmul2_rn(__fmul2_rn(inv,sh),sh); }
      if (MODE==6){ es=__fadd2_rn(__ffma2_rn(r2u,f2(c*c),inv),f2(-2.f*c)); }
      if (MODE==7||MODE==17){ es=__fadd2_rn(__ffma2_rn(r2u,f2(c*c),inv),f2(-2.f*c)); es.x=ix?es.x:0.f; es.y=iy?es.y:0.f; }
      Q[p]=__ffma2_rn(es,f2(xq.w),Q[p]);
      float2 inv2=__fmul2_rn(inv,inv), inv3=__fmul2_rn(inv2,inv), inv6=__fmul2_rn(inv3,inv3);
      A[p]=__ffma2_rn(inv6,f2(pp.x),A[p]); B[p]=__ffma2_rn(inv3,f2(pp.y),B[p]);
    }
  }
  float s=0; for(int p=0;p<KP;p++) s+=Q[p].x+Q[p].y+A[p].x+A[p].y+B[p].x+B[p].y;
  out[blockIdx.x*blockDim.x+threadIdx.x]=s;
}
template<int KP,int MODE> void run(const char* name, int blocks_per_sm){
  float* d; cudaMalloc(&d, 148*64*128*4);
  int n=4000; int blocks=148*blocks_per_sm;
  k<KP,MODE><<<blocks,128>>>(d,100,0.01f,144.f,1.f/144); cudaDeviceSynchronize();
  cudaEvent_t a,b; cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a); k<KP,MODE><<<blocks,128>>>(d,n,0.01f,144.f,1.f/144); cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms,a,b);
  double pairs=(double)blocks*128*n*KP*2;
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("%-22s KP=%d warps/SM=%2d: %.3f Tpairs/s  = %.2f pairs/clk/SM @1.965GHz\n", name, KP, blocks_per_sm*4, pairs/ms/1e9, pairs/(ms*1e-3)/148/1.965e9);
  cudaFree(d);
}
int main(){
  run<4,17>("expanded r2, full cut",4); run<4,17>("expanded r2, full cut",3);
  run<4,1>("clamp only",4); run<4,5>("clamp+r2mask",4); run<4,6>("clamp+es(no mask)",4); run<4,7>("clamp+r2mask+es+esmask",4);
  run<4,2>("cut: es FFMA2+FADD2+FSEL",4); run<4,3>("cut: es inv_m*s*s",4);
  run<4,2>("cut: es FFMA2+FADD2+FSEL",3); run<4,3>("cut: es inv_m*s*s",3);
  run<6,3>("cut: es inv_m*s*s",3);
  return 0;
}
