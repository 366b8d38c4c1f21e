// loop_ceiling.cu -- how fast can the P2P inner loop run with no task / TMA /
// reduction overhead?  Each warp sweeps a shared-memory array of sources with
// the product's interact2 (4 targets per lane as two FFMA2 pairs), optionally
// folding into fp64 every 128 sources like the product.  Reports interactions/s
// and the fraction of the 13-op FP32 ceiling; used to split the product
// kernel's loss into "loop" and "everything else".
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/loop_ceiling tools/loop_ceiling.cu
#include <cstdio>
#include <cuda_runtime.h>

#include "../paper_conf_ipps_overmanpmm13_b200/csrc/p2p_kernel.cuh"

using namespace afmm;

constexpr int kSrc = 384;

__device__ __forceinline__ float rcp_ftz(float x) {
    float y;
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}
// Variant 1: 1/r^2 from MUFU.RCP instead of inv*inv (moves one FMUL2 to the XU pipe)
__device__ __forceinline__ void interact2_rcp(const float4 q, const float2 nx, const float2 ny, const float2 nz,
                                              const float2 e2, float2 &ax, float2 &ay, float2 &az, float2 &ph) {
    const float2 dx = __fadd2_rn(make_float2(q.x, q.x), nx);
    const float2 dy = __fadd2_rn(make_float2(q.y, q.y), ny);
    const float2 dz = __fadd2_rn(make_float2(q.z, q.z), nz);
    float2 r2 = __ffma2_rn(dx, dx, e2);
    r2 = __ffma2_rn(dy, dy, r2);
    r2 = __ffma2_rn(dz, dz, r2);
    float2 inv, i2;
    inv.x = rsqrt_ftz(r2.x);
    inv.y = rsqrt_ftz(r2.y);
    i2.x = rcp_ftz(r2.x);
    i2.y = rcp_ftz(r2.y);
    const float2 t = __fmul2_rn(make_float2(q.w, q.w), inv);
    ph = __fadd2_rn(ph, t);
    const float2 s = __fmul2_rn(t, i2);
    ax = __ffma2_rn(s, dx, ax);
    ay = __ffma2_rn(s, dy, ay);
    az = __ffma2_rn(s, dz, az);
}
// Variant 4: the three acceleration FFMA2s of one pair in one PTX block (so
// ptxas may issue them back to back with s in the same operand slot -> .reuse)
__device__ __forceinline__ unsigned long long f2u(float2 v) {
    unsigned long long r;
    asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(v.x), "f"(v.y));
    return r;
}
__device__ __forceinline__ float2 u2f(unsigned long long r) {
    float2 v;
    asm("mov.b64 {%0, %1}, %2;" : "=f"(v.x), "=f"(v.y) : "l"(r));
    return v;
}
__device__ __forceinline__ void interact2_blk(const float4 q, const float2 nx, const float2 ny, const float2 nz,
                                              const float2 e2, unsigned long long &ax, unsigned long long &ay,
                                              unsigned long long &az, float2 &ph) {
    const float2 dx = __fadd2_rn(make_float2(q.x, q.x), nx);
    const float2 dy = __fadd2_rn(make_float2(q.y, q.y), ny);
    const float2 dz = __fadd2_rn(make_float2(q.z, q.z), nz);
    float2 r2 = __ffma2_rn(dx, dx, e2);
    r2 = __ffma2_rn(dy, dy, r2);
    r2 = __ffma2_rn(dz, dz, r2);
    float2 inv;
    inv.x = rsqrt_ftz(r2.x);
    inv.y = rsqrt_ftz(r2.y);
    const float2 t = __fmul2_rn(make_float2(q.w, q.w), inv);
    ph = __fadd2_rn(ph, t);
    const float2 i2 = __fmul2_rn(inv, inv);
    const float2 s = __fmul2_rn(t, i2);
    asm volatile("{\n\tfma.rn.f32x2 %0, %3, %4, %0;\n\tfma.rn.f32x2 %1, %3, %5, %1;\n\tfma.rn.f32x2 %2, %3, %6, %2;\n}"
                 : "+l"(ax), "+l"(ay), "+l"(az) : "l"(f2u(s)), "l"(f2u(dx)), "l"(f2u(dy)), "l"(f2u(dz)));
}
// Variant 2: scalar FP32 ops (no FFMA2)
__device__ __forceinline__ void interact1(const float4 q, float nx, float ny, float nz, float e2, float &ax,
                                          float &ay, float &az, float &ph) {
    const float dx = q.x + nx, dy = q.y + ny, dz = q.z + nz;
    const float r2 = fmaf(dz, dz, fmaf(dy, dy, fmaf(dx, dx, e2)));
    const float inv = rsqrt_ftz(r2);
    const float t = q.w * inv;
    ph += t;
    const float s = t * (inv * inv);
    ax = fmaf(s, dx, ax);
    ay = fmaf(s, dy, ay);
    az = fmaf(s, dz, az);
}


// Variant 5/6: equal-mass loop (12 packed ops); 6 = the three a-updates as six scalar FFMAs
// (an FFMA2 reading three distinct register pairs costs 3 pipe cycles, two scalar FFMAs 2)
template <bool kScalarA>
__device__ __forceinline__ void interact2_eq(const float4 q, const float2 nx, const float2 ny, const float2 nz,
                                             const float2 e2, float2 &ax, float2 &ay, float2 &az, float2 &ph) {
    const float2 dx = __fadd2_rn(make_float2(q.x, q.x), nx);
    const float2 dy = __fadd2_rn(make_float2(q.y, q.y), ny);
    const float2 dz = __fadd2_rn(make_float2(q.z, q.z), nz);
    float2 r2 = __ffma2_rn(dx, dx, e2);
    r2 = __ffma2_rn(dy, dy, r2);
    r2 = __ffma2_rn(dz, dz, r2);
    float2 inv;
    inv.x = rsqrt_ftz(r2.x);
    inv.y = rsqrt_ftz(r2.y);
    ph = __fadd2_rn(ph, inv);
    const float2 i2 = __fmul2_rn(inv, inv);
    const float2 s = __fmul2_rn(inv, i2);
    if (kScalarA) {
        asm("fma.rn.f32 %0, %1, %2, %0;" : "+f"(ax.x) : "f"(s.x), "f"(dx.x));
        asm("fma.rn.f32 %0, %1, %2, %0;" : "+f"(ax.y) : "f"(s.y), "f"(dx.y));
        asm("fma.rn.f32 %0, %1, %2, %0;" : "+f"(ay.x) : "f"(s.x), "f"(dy.x));
        asm("fma.rn.f32 %0, %1, %2, %0;" : "+f"(ay.y) : "f"(s.y), "f"(dy.y));
        asm("fma.rn.f32 %0, %1, %2, %0;" : "+f"(az.x) : "f"(s.x), "f"(dz.x));
        asm("fma.rn.f32 %0, %1, %2, %0;" : "+f"(az.y) : "f"(s.y), "f"(dz.y));
    } else {
        ax = __ffma2_rn(s, dx, ax);
        ay = __ffma2_rn(s, dy, ay);
        az = __ffma2_rn(s, dz, az);
    }
}
// Variant 7: general masses, scalar a-updates
__device__ __forceinline__ void interact2_sa(const float4 q, const float2 nx, const float2 ny, const float2 nz,
                                             const float2 e2, float2 &ax, float2 &ay, float2 &az, float2 &ph) {
    const float2 dx = __fadd2_rn(make_float2(q.x, q.x), nx);
    const float2 dy = __fadd2_rn(make_float2(q.y, q.y), ny);
    const float2 dz = __fadd2_rn(make_float2(q.z, q.z), nz);
    float2 r2 = __ffma2_rn(dx, dx, e2);
    r2 = __ffma2_rn(dy, dy, r2);
    r2 = __ffma2_rn(dz, dz, r2);
    float2 inv;
    inv.x = rsqrt_ftz(r2.x);
    inv.y = rsqrt_ftz(r2.y);
    const float2 t = __fmul2_rn(make_float2(q.w, q.w), inv);
    ph = __fadd2_rn(ph, t);
    const float2 i2 = __fmul2_rn(inv, inv);
    const float2 s = __fmul2_rn(t, i2);
    asm("fma.rn.f32 %0, %1, %2, %0;" : "+f"(ax.x) : "f"(s.x), "f"(dx.x));
    asm("fma.rn.f32 %0, %1, %2, %0;" : "+f"(ax.y) : "f"(s.y), "f"(dx.y));
    asm("fma.rn.f32 %0, %1, %2, %0;" : "+f"(ay.x) : "f"(s.x), "f"(dy.x));
    asm("fma.rn.f32 %0, %1, %2, %0;" : "+f"(ay.y) : "f"(s.y), "f"(dy.y));
    asm("fma.rn.f32 %0, %1, %2, %0;" : "+f"(az.x) : "f"(s.x), "f"(dz.x));
    asm("fma.rn.f32 %0, %1, %2, %0;" : "+f"(az.y) : "f"(s.y), "f"(dz.y));
}

template <int kWarpsT, int kU, bool kFoldOn, int kVar>
__global__ void __launch_bounds__(32 * kWarpsT, 1) loop_kernel(const float4 *__restrict__ g, int reps, float eps2,
                                                              float *out) {
    __shared__ float4 src[kSrc];   // shared by the CTA's warps (a broadcast read either way)
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    for (int i = threadIdx.x; i < kSrc; i += 32 * kWarpsT) src[i] = g[(blockIdx.x * 7 + i) % 4096];
    __syncthreads();
    const float2 e2 = make_float2(eps2, eps2);
    float2 nx[2], ny[2], nz[2], ax[2], ay[2], az[2], ph[2];
    for (int q = 0; q < 2; ++q) {
        const float4 a = g[lane * 4 + 2 * q], b = g[lane * 4 + 2 * q + 1];
        nx[q] = make_float2(-a.x, -b.x);
        ny[q] = make_float2(-a.y, -b.y);
        nz[q] = make_float2(-a.z, -b.z);
        ax[q] = ay[q] = az[q] = ph[q] = make_float2(0.f, 0.f);
    }
    double acc[16] = {0};
    const float4 *s = src + 0 * warp;
    for (int r = 0; r < reps; ++r) {
        for (int k0 = 0; k0 < kSrc; k0 += 128) {
#pragma unroll kU
            for (int k = k0; k < k0 + 128; ++k) {
#pragma unroll
                for (int q = 0; q < 2; ++q) {
                    if (kVar == 0 || (kVar == 1 && q == 1))
                        interact2<false>(s[k], nx[q], ny[q], nz[q], e2, ax[q], ay[q], az[q], ph[q], false, false);
                    else if (kVar == 4) {
                        unsigned long long ux = f2u(ax[q]), uy = f2u(ay[q]), uz = f2u(az[q]);
                        interact2_blk(s[k], nx[q], ny[q], nz[q], e2, ux, uy, uz, ph[q]);
                        ax[q] = u2f(ux); ay[q] = u2f(uy); az[q] = u2f(uz);
                    }
                    else if (kVar == 5)
                        interact2_eq<false>(s[k], nx[q], ny[q], nz[q], e2, ax[q], ay[q], az[q], ph[q]);
                    else if (kVar == 6)
                        interact2_eq<true>(s[k], nx[q], ny[q], nz[q], e2, ax[q], ay[q], az[q], ph[q]);
                    else if (kVar == 7)
                        interact2_sa(s[k], nx[q], ny[q], nz[q], e2, ax[q], ay[q], az[q], ph[q]);
                    else if (kVar == 1 || kVar == 3)
                        interact2_rcp(s[k], nx[q], ny[q], nz[q], e2, ax[q], ay[q], az[q], ph[q]);
                    else {
                        const float4 v = s[k];
                        interact1(v, nx[q].x, ny[q].x, nz[q].x, e2.x, ax[q].x, ay[q].x, az[q].x, ph[q].x);
                        interact1(v, nx[q].y, ny[q].y, nz[q].y, e2.x, ax[q].y, ay[q].y, az[q].y, ph[q].y);
                    }
                }
            }
            if (kFoldOn) {
#pragma unroll
                for (int q = 0; q < 2; ++q) {
                    acc[8 * q + 0] += ax[q].x; acc[8 * q + 1] += ay[q].x; acc[8 * q + 2] += az[q].x;
                    acc[8 * q + 3] += ph[q].x; acc[8 * q + 4] += ax[q].y; acc[8 * q + 5] += ay[q].y;
                    acc[8 * q + 6] += az[q].y; acc[8 * q + 7] += ph[q].y;
                    ax[q] = ay[q] = az[q] = ph[q] = make_float2(0.f, 0.f);
                }
            }
        }
    }
    double t = 0;
    for (int q = 0; q < 2; ++q) t += ax[q].x + ay[q].y + az[q].x + ph[q].y;
    for (int i = 0; i < 16; ++i) t += acc[i];
    if (t == 1234.5) out[threadIdx.x] = (float)t;
}

template <int kWarpsT, int kU, bool kFoldOn, int kVar = 0>
void run(const float4 *g, float *out, int sms, const char *name) {
    const int reps = 200;
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    float best = 1e30f;
    for (int it = 0; it < 5; ++it) {
        cudaEventRecord(a);
        loop_kernel<kWarpsT, kU, kFoldOn, kVar><<<sms, 32 * kWarpsT>>>(g, reps, 1e-6f, out);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (ms < best) best = ms;
    }
    const double inter = (double)sms * kWarpsT * 32 * 4 * (double)kSrc * reps;
    const double ips = inter / (best * 1e-3);
    printf("%-28s warps=%2d unroll=%d fold=%d  %.4f ms  %.3e int/s  %.1f%% of 20-flop peak@1965\n", name, kWarpsT,
           kU, (int)kFoldOn, best, ips, 100.0 * ips * 20 / 74.44992e12);
    cudaEventDestroy(a);
    cudaEventDestroy(b);
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    float4 *g;
    float *out;
    cudaMalloc(&g, 4096 * sizeof(float4));
    cudaMalloc(&out, 4096 * 4);
    float4 h[4096];
    unsigned s = 12345;
    for (int i = 0; i < 4096; ++i) {
        auto u = [&] { s = s * 1664525u + 1013904223u; return (s >> 8) * (1.0f / 16777216.0f); };
        h[i] = make_float4(u(), u(), u(), 1e-6f);
    }
    cudaMemcpy(g, h, sizeof(h), cudaMemcpyHostToDevice);
    run<12, 4, true>(g, out, sms, "product-like");
    run<12, 4, true, 7>(g, out, sms, "scalar a-updates");
    run<12, 4, true, 5>(g, out, sms, "equal mass");
    run<12, 4, true, 6>(g, out, sms, "equal mass, scalar a");
    run<16, 4, true, 6>(g, out, sms, "equal mass, scalar a");
    run<12, 8, true, 6>(g, out, sms, "equal mass, scalar a");
    run<12, 4, false>(g, out, sms, "no fold");
    run<8, 4, true>(g, out, sms, "8 warps");
    run<16, 4, true>(g, out, sms, "16 warps");
    run<12, 2, true>(g, out, sms, "unroll 2");
    run<12, 8, true>(g, out, sms, "unroll 8");
    run<12, 4, true, 4>(g, out, sms, "a-update asm block");
    run<12, 4, true, 1>(g, out, sms, "rcp on one pair");
    run<12, 4, true, 3>(g, out, sms, "rcp on both pairs");
    run<12, 4, true, 2>(g, out, sms, "scalar FFMA");
    run<16, 4, true, 2>(g, out, sms, "scalar FFMA");
    printf("%s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
