// peak.cu -- FP32 pipe peak microbenchmark (north_star "the
// chip's measured FP32 FMA peak").  MEASURED_PEAKS.json has no FP32 entry; the
// roofline of the P2P kernel is the FP32 FMA pipe, so the library measures it on
// the box it runs on.
//
// Both probes run 4 CTAs x 256 threads per SM (32 warps: 8 per SMSP), each
// thread 16 independent accumulators (16 scalar chains, or 8 float2 chains for
// FFMA2) under a 64-register budget, so neither occupancy nor registers limit
// them (the round-1 probe ran 2048 threads per SM with 16 float2 chains and was
// register-bound).  The SM clock is block 0 / thread 0's %clock64 cycles over
// its %globaltimer nanoseconds across the same loop (the clock the probe itself
// ran at, not cycles over the launch's wall time).
#include <cuda_runtime.h>

#include "../../include/afmm_p2p.h"

namespace {
constexpr int kChains = 16;
constexpr int kIters = 8192;
constexpr int kThreadsPerBlock = 256, kBlocksPerSM = 4;

__device__ __forceinline__ unsigned long long gtimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

__global__ void __launch_bounds__(kThreadsPerBlock, kBlocksPerSM) ffma_peak(float *out, float b, float c,
                                                                            long long *clk) {
    float a[kChains];
#pragma unroll
    for (int i = 0; i < kChains; ++i) a[i] = threadIdx.x * 1e-3f + i;
    const unsigned long long g0 = gtimer();
    const long long t0 = clock64();
    for (int it = 0; it < kIters; ++it) {
#pragma unroll
        for (int i = 0; i < kChains; ++i) a[i] = fmaf(a[i], b, c);
    }
    const long long t1 = clock64();
    const unsigned long long g1 = gtimer();
    float s = 0.f;
#pragma unroll
    for (int i = 0; i < kChains; ++i) s += a[i];
    if (s == 1234.5f) out[threadIdx.x] = s;
    if (threadIdx.x == 0 && blockIdx.x == 0) {
        clk[0] = t1 - t0;
        clk[1] = (long long)(g1 - g0);
    }
}

__global__ void __launch_bounds__(kThreadsPerBlock, kBlocksPerSM) ffma2_peak(float *out, float b, float c) {
    float2 a[kChains / 2];
#pragma unroll
    for (int i = 0; i < kChains / 2; ++i) a[i] = make_float2(threadIdx.x * 1e-3f + i, 0.5f * i);
    const float2 b2 = make_float2(b, 0.5f * b), c2 = make_float2(c, 0.5f * c);
    for (int it = 0; it < kIters; ++it) {
#pragma unroll
        for (int i = 0; i < kChains / 2; ++i) a[i] = __ffma2_rn(a[i], b2, c2);
    }
    float s = 0.f;
#pragma unroll
    for (int i = 0; i < kChains / 2; ++i) s += a[i].x + a[i].y;
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
    if (cudaMalloc(&out, 4096) != cudaSuccess || cudaMalloc(&clk, 2 * sizeof(long long)) != cudaSuccess ||
        cudaEventCreate(&a) != cudaSuccess || cudaEventCreate(&b) != cudaSuccess) {
        st = AFMM_ECUDA;
    } else {
        const int blocks = sms * kBlocksPerSM, threads = kThreadsPerBlock;
        // flops per launch: every thread runs kIters x kChains FMAs (2 flop each)
        const double fmas = (double)blocks * threads * kIters * kChains;
        float best1 = 1e30f, best2 = 1e30f, ms = 0.f;
        long long cyc[2] = {0, 1};
        for (int rep = 0; rep < 5; ++rep) {
            cudaEventRecord(a);
            ffma_peak<<<blocks, threads>>>(out, 0.999f, 1e-3f, clk);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            cudaEventElapsedTime(&ms, a, b);
            if (ms < best1) {
                best1 = ms;
                cudaMemcpy(cyc, clk, sizeof(cyc), cudaMemcpyDeviceToHost);
            }
            cudaEventRecord(a);
            ffma2_peak<<<blocks, threads>>>(out, 0.999f, 1e-3f);
            cudaEventRecord(b);
            cudaEventSynchronize(b);
            cudaEventElapsedTime(&ms, a, b);
            if (ms < best2) best2 = ms;
        }
        if (cudaGetLastError() != cudaSuccess) st = AFMM_ECUDA;
        if (tflops_ffma) *tflops_ffma = fmas * 2.0 / (best1 * 1e-3) / 1e12;
        if (tflops_ffma2) *tflops_ffma2 = fmas * 2.0 / (best2 * 1e-3) / 1e12;
        // cycles per nanosecond of the same loop in one thread = GHz
        if (sm_mhz) *sm_mhz = cyc[1] > 0 ? (double)cyc[0] / (double)cyc[1] * 1e3 : 0.0;
    }
    cudaFree(out);
    cudaFree(clk);
    if (a) cudaEventDestroy(a);
    if (b) cudaEventDestroy(b);
    return st;
}
