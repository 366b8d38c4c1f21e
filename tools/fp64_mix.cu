// fp64_mix.cu -- can the FP64 pipe carry part of the P2P interactions while the
// FP32 (FFMA2) pipe runs the rest?  On B200 (sm_100a) DFMA runs at half the
// FP32 lane rate on its own pipe, and the product loop is FP32-pipe bound
// (13 packed ops per two interactions) with issue slots to spare.  Each lane
// holds 4 fp32 targets (two FFMA2 pairs, as in the product) plus K fp64
// targets; every source (float4 + double4 copy in shared memory) is applied to
// all of them.  Also: rsqrt.approx.ftz.f64 accuracy and raw pipe rates.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/fp64_mix tools/fp64_mix.cu
#include <cmath>
#include <cstdio>
#include <cuda_runtime.h>

#include "../paper_conf_ipps_overmanpmm13_b200/csrc/p2p_kernel.cuh"

using namespace afmm;

constexpr int kSrc = 384;

__device__ __forceinline__ double rsqrt64(double x) {
    double y;
    asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
    return y;
}
__device__ __forceinline__ double rsqrt64_via32(double x) {
    return (double)rsqrt_ftz((float)x);
}

// kMode: 0 = double4 source in smem; 1 = convert the float4 source (F2F); 2 = double source + fp32 rsqrt
template <int kMode>
__device__ __forceinline__ void interact64(const float4 q, const double4 qd, double nx, double ny, double nz,
                                           double e2, double &ax, double &ay, double &az, double &ph) {
    double xj, yj, zj, mj;
    if (kMode == 1) {
        xj = q.x; yj = q.y; zj = q.z; mj = q.w;
    } else {
        xj = qd.x; yj = qd.y; zj = qd.z; mj = qd.w;
    }
    const double dx = xj + nx, dy = yj + ny, dz = zj + nz;
    const double r2 = fma(dz, dz, fma(dy, dy, fma(dx, dx, e2)));
    const double inv = kMode == 2 ? rsqrt64_via32(r2) : rsqrt64(r2);
    const double t = mj * inv;
    ph += t;
    const double s = t * (inv * inv);
    ax = fma(s, dx, ax);
    ay = fma(s, dy, ay);
    az = fma(s, dz, az);
}

template <int kWarpsT, int kK, int kMode, int kU>
__global__ void __launch_bounds__(32 * kWarpsT, 1) mix_kernel(const float4 *__restrict__ g, int reps, float eps2,
                                                             float *out) {
    __shared__ float4 src[kSrc];
    __shared__ double4 srcd[kSrc];
    const int lane = threadIdx.x & 31;
    for (int i = threadIdx.x; i < kSrc; i += 32 * kWarpsT) {
        const float4 v = g[(blockIdx.x * 7 + i) % 4096];
        src[i] = v;
        srcd[i] = make_double4(v.x, v.y, v.z, v.w);
    }
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
    double dnx[kK > 0 ? kK : 1], dny[kK > 0 ? kK : 1], dnz[kK > 0 ? kK : 1];
    double dax[kK > 0 ? kK : 1], day[kK > 0 ? kK : 1], daz[kK > 0 ? kK : 1], dph[kK > 0 ? kK : 1];
    for (int q = 0; q < kK; ++q) {
        const float4 a = g[512 + lane * 4 + q];
        dnx[q] = -(double)a.x; dny[q] = -(double)a.y; dnz[q] = -(double)a.z;
        dax[q] = day[q] = daz[q] = dph[q] = 0.0;
    }
    double acc[16] = {0};
    for (int r = 0; r < reps; ++r) {
        for (int k0 = 0; k0 < kSrc; k0 += 128) {
#pragma unroll kU
            for (int k = k0; k < k0 + 128; ++k) {
                const float4 v = src[k];
#pragma unroll
                for (int q = 0; q < 2; ++q)
                    interact2<false>(v, nx[q], ny[q], nz[q], e2, ax[q], ay[q], az[q], ph[q], false, false);
                if (kK > 0) {
                    double4 vd = make_double4(0, 0, 0, 0);
                    if (kMode != 1) vd = srcd[k];
#pragma unroll
                    for (int q = 0; q < kK; ++q)
                        interact64<kMode>(v, vd, dnx[q], dny[q], dnz[q], (double)eps2, dax[q], day[q], daz[q],
                                          dph[q]);
                }
            }
#pragma unroll
            for (int q = 0; q < 2; ++q) {
                acc[8 * q + 0] += ax[q].x; acc[8 * q + 1] += ay[q].x; acc[8 * q + 2] += az[q].x;
                acc[8 * q + 3] += ph[q].x; acc[8 * q + 4] += ax[q].y; acc[8 * q + 5] += ay[q].y;
                acc[8 * q + 6] += az[q].y; acc[8 * q + 7] += ph[q].y;
                ax[q] = ay[q] = az[q] = ph[q] = make_float2(0.f, 0.f);
            }
        }
    }
    double t = 0;
    for (int i = 0; i < 16; ++i) t += acc[i];
    for (int q = 0; q < kK; ++q) t += dax[q] + day[q] + daz[q] + dph[q];
    if (t == 1234.5) out[threadIdx.x] = (float)t;
}

template <int kWarpsT, int kK, int kMode, int kU = 4>
void run(const float4 *g, float *out, int sms, const char *name) {
    const int reps = 100;
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    float best = 1e30f;
    for (int it = 0; it < 5; ++it) {
        cudaEventRecord(a);
        mix_kernel<kWarpsT, kK, kMode, kU><<<sms, 32 * kWarpsT>>>(g, reps, 1e-6f, out);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (ms < best) best = ms;
    }
    const double inter = (double)sms * kWarpsT * 32 * (4 + kK) * (double)kSrc * reps;
    const double ips = inter / (best * 1e-3);
    printf("%-34s warps=%2d K64=%d unroll=%d  %.4f ms  %.3e int/s  %.1f%% of 20-flop FP32 peak@1965\n", name,
           kWarpsT, kK, kU, best, ips, 100.0 * ips * 20 / 74.44992e12);
    cudaEventDestroy(a);
    cudaEventDestroy(b);
}

// raw rates: independent DFMA chains; MUFU.RSQ64H
template <int kOp>
__global__ void __launch_bounds__(512, 1) rate_kernel(int reps, double seed, float *out) {
    double v[8];
    for (int i = 0; i < 8; ++i) v[i] = seed + threadIdx.x + i;
    for (int r = 0; r < reps; ++r) {
#pragma unroll
        for (int u = 0; u < 16; ++u)
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                if (kOp == 0) v[i] = fma(v[i], 0.999999, 1e-9);
                else v[i] = rsqrt64(v[i] + 1.0);
            }
    }
    double t = 0;
    for (int i = 0; i < 8; ++i) t += v[i];
    if (t == 1234.5) out[threadIdx.x] = (float)t;
}
template <int kOp>
void rate(int sms, float *out, const char *name) {
    const int reps = 2000;
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    float best = 1e30f;
    for (int it = 0; it < 3; ++it) {
        cudaEventRecord(a);
        rate_kernel<kOp><<<sms, 512>>>(reps, 1.5, out);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (ms < best) best = ms;
    }
    const double ops = (double)sms * 512 * reps * 16 * 8;
    printf("%-20s %.3e ops/s = %.1f per SM per ns\n", name, ops / (best * 1e-3), ops / (best * 1e-3) / sms / 1e9);
}

__global__ void acc_kernel(const double *x, double *err, int n) {
    int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) {
        const double y = rsqrt64(x[i]);
        const double ref = 1.0 / sqrt(x[i]);
        err[i] = fabs(y - ref) / ref;
    }
}

int main() {
    int sms = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    float4 *g;
    float *out;
    cudaMalloc(&g, 4096 * sizeof(float4));
    cudaMalloc(&out, 4096 * 4);
    static float4 h[4096];
    unsigned s = 12345;
    for (int i = 0; i < 4096; ++i) {
        auto u = [&] { s = s * 1664525u + 1013904223u; return (s >> 8) * (1.0f / 16777216.0f); };
        h[i] = make_float4(u(), u(), u(), 1e-6f);
    }
    cudaMemcpy(g, h, sizeof(h), cudaMemcpyHostToDevice);
    // accuracy of rsqrt.approx.ftz.f64 over [1e-8, 1e4]
    const int n = 1 << 20;
    double *hx = new double[n], *he = new double[n];
    for (int i = 0; i < n; ++i) hx[i] = pow(10.0, -8.0 + 12.0 * (i + 0.37) / n);
    double *dx, *de;
    cudaMalloc(&dx, n * 8);
    cudaMalloc(&de, n * 8);
    cudaMemcpy(dx, hx, n * 8, cudaMemcpyHostToDevice);
    acc_kernel<<<(n + 255) / 256, 256>>>(dx, de, n);
    cudaMemcpy(he, de, n * 8, cudaMemcpyDeviceToHost);
    double mx = 0;
    for (int i = 0; i < n; ++i) mx = he[i] > mx ? he[i] : mx;
    printf("rsqrt.approx.ftz.f64 max rel err %.3e (2^%.1f)\n", mx, log2(mx));

    rate<0>(sms, out, "DFMA");
    rate<1>(sms, out, "rsqrt.approx.f64");
    run<12, 0, 0>(g, out, sms, "fp32 only (product loop)");
    run<12, 1, 0>(g, out, sms, "+1 fp64 target (double4 smem)");
    run<12, 2, 0>(g, out, sms, "+2 fp64 targets (double4 smem)");
    run<12, 3, 0>(g, out, sms, "+3 fp64 targets (double4 smem)");
    run<12, 2, 1>(g, out, sms, "+2 fp64 targets (F2F convert)");
    run<12, 2, 2>(g, out, sms, "+2 fp64 targets (fp32 rsqrt)");
    run<8, 2, 0>(g, out, sms, "+2 fp64 targets (double4 smem)");
    run<16, 2, 0>(g, out, sms, "+2 fp64 targets (double4 smem)");
    run<12, 2, 0, 2>(g, out, sms, "+2 fp64 targets (double4 smem)");
    printf("%s\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
