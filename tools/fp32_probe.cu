// FP32 pipe probe for sm_100a: FFMA, FFMA2, MUFU.RSQ throughput (standalone, first-round measurement).
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ float rsq(float x){ float y; asm("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x)); return y; }
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
    for(int i=0;i<CH;i++) a[i]=rsq(a[i]+c);
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
      float2 inv; inv.x=rsq(r2.x); inv.y=rsq(r2.y);
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
      float inv=rsq(r2); float t=q.w*inv; ph+=t; float s2=t*(inv*inv);
      ax=fmaf(s2,dx,ax); ay=fmaf(s2,dy,ay); az=fmaf(s2,dz,az);
    }
  }
  float v=ax+ay+az+ph;
  if(v==1234.5f) out[threadIdx.x]=v;
}

// scalar, NT targets per thread (ILP), optional equal-mass (12 FP32 ops)
template<int NT, bool EQ>
__global__ void __launch_bounds__(256) k_pairS(float* out, const float4* src, int nsrc, int reps){
  __shared__ float4 s[1024];
  for(int i=threadIdx.x;i<1024;i+=blockDim.x) s[i]=src[i];
  __syncthreads();
  float nx[NT],ny[NT],nz[NT],ax[NT],ay[NT],az[NT],ph[NT];
  #pragma unroll
  for(int k=0;k<NT;k++){nx[k]=-threadIdx.x*1e-3f-k*1e-4f;ny[k]=nx[k]*0.5f;nz[k]=nx[k]*0.25f;ax[k]=ay[k]=az[k]=ph[k]=0;}
  for(int r=0;r<reps;r++){
    #pragma unroll 4
    for(int j=0;j<1024;j++){ float4 q=s[j];
      #pragma unroll
      for(int k=0;k<NT;k++){
        float dx=q.x+nx[k], dy=q.y+ny[k], dz=q.z+nz[k];
        float r2=fmaf(dx,dx,1e-6f); r2=fmaf(dy,dy,r2); r2=fmaf(dz,dz,r2);
        float inv=rsq(r2);
        if(EQ){ ph[k]+=inv; float s3=inv*inv*inv; ax[k]=fmaf(s3,dx,ax[k]); ay[k]=fmaf(s3,dy,ay[k]); az[k]=fmaf(s3,dz,az[k]); }
        else { float t=q.w*inv; ph[k]+=t; float s2=t*(inv*inv);
          ax[k]=fmaf(s2,dx,ax[k]); ay[k]=fmaf(s2,dy,ay[k]); az[k]=fmaf(s2,dz,az[k]); }
      }
    }
  }
  float v=0; for(int k=0;k<NT;k++) v+=ax[k]+ay[k]+az[k]+ph[k];
  if(v==1234.5f) out[threadIdx.x]=v;
}
// FFMA2, 2*NP targets per thread
template<int NP, bool EQ>
__global__ void __launch_bounds__(256) k_pairV(float* out, const float4* src, int nsrc, int reps){
  __shared__ float4 s[1024];
  for(int i=threadIdx.x;i<1024;i+=blockDim.x) s[i]=src[i];
  __syncthreads();
  float2 nx[NP],ny[NP],nz[NP],ax[NP],ay[NP],az[NP],ph[NP];
  #pragma unroll
  for(int k=0;k<NP;k++){nx[k]=make_float2(-threadIdx.x*1e-3f-k*1e-4f,-threadIdx.x*2e-3f); ny[k]=nx[k]; nz[k]=nx[k];
    ax[k]=ay[k]=az[k]=ph[k]=make_float2(0,0);}
  const float2 e2=make_float2(1e-6f,1e-6f);
  for(int r=0;r<reps;r++){
    #pragma unroll 4
    for(int j=0;j<1024;j++){ float4 q=s[j];
      #pragma unroll
      for(int k=0;k<NP;k++){
      float2 dx=__fadd2_rn(make_float2(q.x,q.x),nx[k]), dy=__fadd2_rn(make_float2(q.y,q.y),ny[k]), dz=__fadd2_rn(make_float2(q.z,q.z),nz[k]);
      float2 r2=__ffma2_rn(dx,dx,e2); r2=__ffma2_rn(dy,dy,r2); r2=__ffma2_rn(dz,dz,r2);
      float2 inv; inv.x=rsq(r2.x); inv.y=rsq(r2.y);
      if(EQ){ ph[k]=__fadd2_rn(ph[k],inv); float2 i2=__fmul2_rn(inv,inv); float2 s2=__fmul2_rn(inv,i2);
        ax[k]=__ffma2_rn(s2,dx,ax[k]); ay[k]=__ffma2_rn(s2,dy,ay[k]); az[k]=__ffma2_rn(s2,dz,az[k]); }
      else {
      float2 t=__fmul2_rn(make_float2(q.w,q.w),inv); ph[k]=__fadd2_rn(ph[k],t); float2 i2=__fmul2_rn(inv,inv); float2 s2=__fmul2_rn(t,i2);
      ax[k]=__ffma2_rn(s2,dx,ax[k]); ay[k]=__ffma2_rn(s2,dy,ay[k]); az[k]=__ffma2_rn(s2,dz,az[k]); }
      }
    }
  }
  float v=0; for(int k=0;k<NP;k++) v+=ax[k].x+ax[k].y+ay[k].x+ay[k].y+az[k].x+az[k].y+ph[k].x+ph[k].y;
  if(v==1234.5f) out[threadIdx.x]=v;
}
// pure 3-register FFMA: a = a*b + c with b,c per-thread registers
__global__ void __launch_bounds__(256) k_ffma3(float* out, float b0, float c0, int iters){
  float a[CH], b[4], c[4];
  for(int i=0;i<4;i++){b[i]=b0+threadIdx.x*1e-7f*i; c[i]=c0*(i+1)+threadIdx.x*1e-9f;}
  #pragma unroll
  for(int i=0;i<CH;i++) a[i]=threadIdx.x*1e-3f+i;
  for(int it=0; it<iters; it++){
    #pragma unroll
    for(int i=0;i<CH;i++) a[i]=fmaf(a[i],b[i&3],c[(i>>2)&3]);
  }
  float s=0; for(int i=0;i<CH;i++) s+=a[i];
  if(s==1234.5f) out[threadIdx.x]=s;
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

  {
    int blocks=sms*8, thr=256, reps=16; double tt=(double)blocks*thr; float ms;
    auto run=[&](const char* nm, void(*k)(float*,const float4*,int,int), int tpt){
      for(int w=0;w<2;w++){ k<<<blocks,thr>>>(out,src,1024,reps); }
      cudaEventRecord(a); k<<<blocks,thr>>>(out,src,1024,reps); cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms,a,b);
      printf("{\"kernel\":\"%s\",\"gint_per_s\":%.1f}\n", nm, tt*tpt*reps*1024/(ms*1e-3)/1e9);
    };
    run("S1",k_pairS<1,false>,1); run("S2",k_pairS<2,false>,2); run("S4",k_pairS<4,false>,4);
    run("S1eq",k_pairS<1,true>,1); run("S2eq",k_pairS<2,true>,2);
    run("V1",k_pairV<1,false>,2); run("V2",k_pairV<2,false>,4); run("V1eq",k_pairV<1,true>,2); run("V2eq",k_pairV<2,true>,4);
    cudaEventRecord(a); k_ffma3<<<blocks,thr>>>(out,0.999f,1e-3f,4096); cudaEventRecord(b); cudaEventSynchronize(b); cudaEventElapsedTime(&ms,a,b);
    printf("{\"kernel\":\"ffma3reg\",\"tflops\":%.2f}\n", tt*4096*CH*2/(ms*1e-3)/1e12);
  }
  CK(cudaGetLastError());
  return 0;
}
