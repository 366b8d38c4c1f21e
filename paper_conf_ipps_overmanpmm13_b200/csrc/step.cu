// step.cu -- leapfrog kick / drift kernels (include/afmm_step.h).
#include <algorithm>
#include <cmath>

#include <cuda_runtime.h>

#include "../../include/afmm_step.h"

namespace {

__global__ void axpy3_kernel(long long n, float *__restrict__ u, float *__restrict__ v, float *__restrict__ w,
                             const float *__restrict__ a, const float *__restrict__ b,
                             const float *__restrict__ c, float h) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n;
         i += (long long)gridDim.x * blockDim.x) {
        u[i] = __fmaf_rn(h, a[i], u[i]);
        v[i] = __fmaf_rn(h, b[i], v[i]);
        w[i] = __fmaf_rn(h, c[i], w[i]);
    }
}

__global__ void kick_drift_kernel(long long n, float *__restrict__ x, float *__restrict__ y, float *__restrict__ z,
                                  float *__restrict__ vx, float *__restrict__ vy, float *__restrict__ vz,
                                  const float *__restrict__ ax, const float *__restrict__ ay,
                                  const float *__restrict__ az, float h, float dt) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n;
         i += (long long)gridDim.x * blockDim.x) {
        const float ux = __fmaf_rn(h, ax[i], vx[i]), uy = __fmaf_rn(h, ay[i], vy[i]), uz = __fmaf_rn(h, az[i], vz[i]);
        vx[i] = ux;
        vy[i] = uy;
        vz[i] = uz;
        x[i] = __fmaf_rn(dt, ux, x[i]);
        y[i] = __fmaf_rn(dt, uy, y[i]);
        z[i] = __fmaf_rn(dt, uz, z[i]);
    }
}

afmm_status launch(long long n, float *u, float *v, float *w, const float *a, const float *b, const float *c,
                   float h, void *stream) {
    if (n < 0 || !std::isfinite(h)) return AFMM_EINVAL;
    if (n == 0) return AFMM_OK;
    if (!u || !v || !w || !a || !b || !c) return AFMM_EINVAL;
    const int threads = 256;
    const long long blocks = std::min<long long>((n + threads - 1) / threads, 148LL * 32);
    axpy3_kernel<<<(int)blocks, threads, 0, static_cast<cudaStream_t>(stream)>>>(n, u, v, w, a, b, c, h);
    return cudaGetLastError() == cudaSuccess ? AFMM_OK : AFMM_ECUDA;
}

}  // namespace

extern "C" afmm_status afmm_kick(long long n, float *vx, float *vy, float *vz, const float *ax, const float *ay,
                                 const float *az, float h, void *stream) {
    return launch(n, vx, vy, vz, ax, ay, az, h, stream);
}

extern "C" afmm_status afmm_drift(long long n, float *x, float *y, float *z, const float *vx, const float *vy,
                                  const float *vz, float dt, void *stream) {
    return launch(n, x, y, z, vx, vy, vz, dt, stream);
}

extern "C" afmm_status afmm_kick_drift(long long n, float *x, float *y, float *z, float *vx, float *vy, float *vz,
                                       const float *ax, const float *ay, const float *az, float h, float dt,
                                       void *stream) {
    if (n < 0 || !std::isfinite(h) || !std::isfinite(dt)) return AFMM_EINVAL;
    if (n == 0) return AFMM_OK;
    if (!x || !y || !z || !vx || !vy || !vz || !ax || !ay || !az) return AFMM_EINVAL;
    const int threads = 256;
    const long long blocks = std::min<long long>((n + threads - 1) / threads, 148LL * 32);
    kick_drift_kernel<<<(int)blocks, threads, 0, static_cast<cudaStream_t>(stream)>>>(n, x, y, z, vx, vy, vz, ax, ay,
                                                                                     az, h, dt);
    return cudaGetLastError() == cudaSuccess ? AFMM_OK : AFMM_ECUDA;
}
