// FP32 pipe probe for sm_100a: FFMA, FFMA2, MUFU.RSQ throughput (standalone, first-round measurement).
#include <cstdio>
#include <cuda_runtime.h>
#define CK(x) do{cudaError_t e=(x); if(e){printf("CUDA %s line %d\n", cudaGetErrorString(e), __LINE__); return 1;}}while(0)
constexpr int CH = 16;
__global__ void __launch_bounds__(256) k_ffma(float* out, float b, float c, int iters){
  float a[CH];
  #pragma unroll
  for(int i=0;i<CH;i++) a[i]=threadIdx.x*1e-3f+i;
  for(int it=0; it<iters; it++){
    #pragma unroll
    for(int i=0;i<CH;i++) a[i]=fmaf(a[i],b,c);
  }
  float s=0; for(int i=0;i<CH;i++) s+=a[i];
  if(s==1234.5f) out[threadIdx.x]=s;
}
__global__ void __launch_bounds__(256) k_ffma2(float* out, float b, float c, int iters){
  float2 a[CH];
  #pragma unroll
  for(int i=0;i<CH;i++) a[i]=make_float2(threadIdx.x*1e-3f+i, i*0.5f);
  float2 b2=make_float2(b,b*0.5f), c2=make_float2(c,c*0.5f);
  for(int it=0; it<iters; it++){
    #pragma unroll
    for(int i=0;i<CH;i++) a[i]=__ffma2_rn(a[i],b2,c2);
  }
  float s=0; for(int i=0;i<CH;i++) s+=a[i].x+a[i].y;
  if(s==1234.5f) out[threadIdx.x]=s;
}
__global__ void __launch_bounds__(256) k_rsq(float* out, float c, int iters){
  float a[CH];
  #pragma unroll
  for(int i=0;i<CH;i++) a[i]=threadIdx.x*1e-3f+i+1.f;
  for(int it=0; it<iters; it++){
    #pragma unroll
    for(int i=0;i<CH;i++) a[i]=rsqrtf(a[i]+c);
  }
  float s=0; for(int i=0;i<CH;i++) s+=a[i];
  if(s==1234.5f) out[threadIdx.x]=s;
}
// mixed: the pair law with one LDS.128 broadcast per source, 2 targets per thread, FFMA2.
__global__ void __launch_bounds__(256) k_pair2(float* out, const float4* src, int nsrc, int reps){
  __shared__ float4 s[1024];
  for(int i=threadIdx.x;i<1024;i+=blockDim.x) s[i]=src[i];
  __syncthreads();
  float2 nx=make_float2(-threadIdx.x*1e-3f,-threadIdx.x*2e-3f), ny=nx, nz=nx;
  float2 ax={0,0},ay={0,0},az={0,0},ph={0,0};
  const float2 e2=make_float2(1e-6f,1e-6f);
  for(int r=0;r<reps;r++){
    #pragma unroll 8
    for(int j=0;j<1024;j++){ float4 q=s[j];
      float2 dx=__fadd2_rn(make_float2(q.x,q.x),nx), dy=__fadd2_rn(make_float2(q.y,q.y),ny), dz=__fadd2_rn(make_float2(q.z,q.z),nz);
      float2 r2=__ffma2_rn(dx,dx,e2); r2=__ffma2_rn(dy,dy,r2); r2=__ffma2_rn(dz,dz,r2);
      float2 inv; inv.x=rsqrtf(r2.x); inv.y=rsqrtf(r2.y);
      float2 t=__fmul2_rn(make_float2(q.w,q.w),inv); ph=__fadd2_rn(ph,t); float2 i2=__fmul2_rn(inv,inv); float2 s2=__fmul2_rn(t,i2);
      ax=__ffma2_rn(s2,dx,ax); ay=__ffma2_rn(s2,dy,ay); az=__ffma2_rn(s2,dz,az);
    }
  }
  float v=ax.x+ax.y+ay.x+ay.y+az.x+az.y+ph.x+ph.y;
  if(v==1234.5f) out[threadIdx.x]=v;
}
// scalar variant: 1 target per thread
__global__ void __launch_bounds__(256) k_pair1(float* out, const float4* src, int nsrc, int reps){
  __shared__ float4 s[1024];
  for(int i=threadIdx.x;i<1024;i+=blockDim.x) s[i]=src[i];
  __syncthreads();
  float nx=-threadIdx.x*1e-3f, ny=nx, nz=nx;
  float ax=0,ay=0,az=0,ph=0;
  for(int r=0;r<reps;r++){
    #pragma unroll 8
    for(int j=0;j<1024;j++){ float4 q=s[j];
      float dx=q.x+nx, dy=q.y+ny, dz=q.z+nz;
      float r2=fmaf(dx,dx,1e-6f); r2=fmaf(dy,dy,r2); r2=fmaf(dz,dz,r2);
      float inv=rsqrtf(r2); float t=q.w*inv; ph+=t; float s2=t*(inv*inv);
      ax=fmaf(s2,dx,ax); ay=fmaf(s2,dy,ay); az=fmaf(s2,dz,az);
    }
  }
  float v=ax+ay+az+ph;
  if(v==1234.5f) out[threadIdx.x]=v;
}
int main(){
  int dev=0; cudaDeviceProp p; CK(cudaGetDeviceProperties(&p,dev));
  int clk=0; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, dev);
  printf("{\"gpu\":\"%s\",\"sms\":%d,\"clock_khz_attr\":%d}\n", p.name, p.multiProcessorCount, clk);
  float* out; CK(cudaMalloc(&out, 4096));
  float4* src; CK(cudaMalloc(&src, 1024*16));
  float4 h[1024]; for(int i=0;i<1024;i++) h[i]=make_float4(i*0.001f,i*0.002f,i*0.003f,1.0f/1024);
  CK(cudaMemcpy(src,h,sizeof(h),cudaMemcpyHostToDevice));
  cudaEvent_t a,b; cudaEventCreate(&a); cudaEventCreate(&b);
  int sms=p.multiProcessorCount;
  for(int occ: {4, 8}){
    int blocks=sms*occ, thr=256; int iters=4096;
    double thr_total=(double)blocks*thr;
    for(int rep=0;rep<2;rep++){
      float ms;
      cudaEventRecord(a); k_ffma<<<blocks,thr>>>(out,0.999f,1e-3f,iters); cudaEventRecord(b); CK(cudaEventSynchronize(b)); cudaEventElapsedTime(&ms,a,b);
      double f1=thr_total*iters*CH*2/(ms*1e-3);
      cudaEventRecord(a); k_ffma2<<<blocks,thr>>>(out,0.999f,1e-3f,iters); cudaEventRecord(b); CK(cudaEventSynchronize(b)); cudaEventElapsedTime(&ms,a,b);
      double f2=thr_total*iters*CH*4/(ms*1e-3);
      cudaEventRecord(a); k_rsq<<<blocks,thr>>>(out,1e-3f,iters/4); cudaEventRecord(b); CK(cudaEventSynchronize(b)); cudaEventElapsedTime(&ms,a,b);
      double r1=thr_total*(iters/4)*CH/(ms*1e-3);
      int reps=16;
      cudaEventRecord(a); k_pair2<<<blocks,thr>>>(out,src,1024,reps); cudaEventRecord(b); CK(cudaEventSynchronize(b)); cudaEventElapsedTime(&ms,a,b);
      double p2=thr_total*2*reps*1024/(ms*1e-3);
      cudaEventRecord(a); k_pair1<<<blocks,thr>>>(out,src,1024,reps); cudaEventRecord(b); CK(cudaEventSynchronize(b)); cudaEventElapsedTime(&ms,a,b);
      double p1=thr_total*reps*1024/(ms*1e-3);
      printf("{\"occ\":%d,\"rep\":%d,\"ffma_tflops\":%.2f,\"ffma2_tflops\":%.2f,\"rsqrt_gops\":%.1f,\"pair_ffma2_gint\":%.1f,\"pair_scalar_gint\":%.1f}\n",
        occ,rep,f1/1e12,f2/1e12,r1/1e9,p2/1e9,p1/1e9);
    }
  }
  CK(cudaGetLastError());
  return 0;
}
