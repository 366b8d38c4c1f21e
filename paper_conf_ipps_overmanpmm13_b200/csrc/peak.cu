// peak.cu -- FP32 pipe peak microbenchmark.
// MEASURED_PEAKS.json has no FP32 entry; the roofline of the P2P kernel is the
// FP32 FMA pipe, so the library measures it on the box it runs on.
#include <cuda_runtime.h>

#include "../../include/afmm_p2p.h"

namespace {
constexpr int kChains = 16;
constexpr int kIters = 4096;

__global__ void __launch_bounds__(256) ffma_peak(float *out, float b, float c, long long *clk) {
    float a[kChains];
#pragma unroll
    for (int i = 0; i < kChains; ++i) a[i] = threadIdx.x * 1e-3f + i;
    const long long t0 = clock64();
    for (int it = 0; it < kIters; ++it) {
#pragma unroll
        for (int i = 0; i < kChains; ++i) a[i] = fmaf(a[i], b, c);
    }
    const long long t1 = clock64();
    float s = 0.f;
#pragma unroll
    for (int i = 0; i < kChains; ++i) s += a[i];
    if (s == 1234.5f) out[threadIdx.x] = s;
    if (threadIdx.x == 0 && blockIdx.x == 0) *clk = t1 - t0;
}

__global__ void __launch_bounds__(256) ffma2_peak(float *out, float b, float c) {
    float2 a[kChains];
#pragma unroll
    for (int i = 0; i < kChains; ++i) a[i] = make_float2(threadIdx.x * 1e-3f + i, 0.5f * i);
    const float2 b2 = make_float2(b, 0.5f * b), c2 = make_float2(c, 0.5f * c);
    for (int it = 0; it < kIters; ++it) {
#pragma unroll
        for (int i = 0; i < kChains; ++i) a[i] = __ffma2_rn(a[i], b2, c2);
    }
    float s = 0.f;
#pragma unroll
    for (int i = 0; i < kChains; ++i) s += a[i].x + a[i].y;
    if (s == 1234.5f) out[threadIdx.x] = s;
}
}  // namespace

extern "C" afmm_status afmm_fp32_peak(int device, double *tflops_ffma, double *tflops_ffma2,
                                      double *sm_mhz) {
    if (cudaSetDevice(device) != cudaSuccess) return AFMM_ECUDA;
    int sms = 0;
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device) != cudaSuccess) return AFMM_ECUDA;
    float *out = nullptr;
    long long *clk = nullptr;
    cudaEvent_t a = nullptr, b = nullptr;
    afmm_status st = AFMM_OK;
    if (cudaMalloc(&out, 4096) != cudaSuccess || cudaMalloc(&clk, sizeof(long long)) != cudaSuccess ||
        cudaEventCreate(&a) != cudaSuccess || cudaEventCreate(&b) != cudaSuccess) {
        st = AFMM_ECUDA;
    } else {
        const int blocks = sms * 8, threads = 256;
        const double lanes = (double)blocks * threads * kIters * kChains;
        float best1 = 1e30f, best2 = 1e30f, ms = 0.f;
        long long cyc = 0;
        for (int rep = 0; rep < 4; ++rep) {
            cudaEventRecord(a);
            ffma_peak<<<blocks, threads>>>(out, 0.999f, 1e-3f, clk);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            cudaEventElapsedTime(&ms, a, b);
            if (ms < best1) {
                best1 = ms;
                cudaMemcpy(&cyc, clk, sizeof(cyc), cudaMemcpyDeviceToHost);
            }
            cudaEventRecord(a);
            ffma2_peak<<<blocks, threads>>>(out, 0.999f, 1e-3f);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            cudaEventElapsedTime(&ms, a, b);
            if (ms < best2) best2 = ms;
        }
        if (cudaGetLastError() != cudaSuccess) st = AFMM_ECUDA;
        if (tflops_ffma) *tflops_ffma = lanes * 2.0 / (best1 * 1e-3) / 1e12;
        if (tflops_ffma2) *tflops_ffma2 = lanes * 4.0 / (best2 * 1e-3) / 1e12;
        // block 0's loop cycles over the launch duration: a lower bound on the SM clock
        if (sm_mhz) *sm_mhz = (double)cyc / (best1 * 1e-3) / 1e6;
    }
    cudaFree(out);
    cudaFree(clk);
    if (a) cudaEventDestroy(a);
    if (b) cudaEventDestroy(b);
    return st;
}
