/*
 * afmm_step.h -- C ABI of the time-step kernels of the dynamic workload
 * (BASELINE configs[4]: "200 leapfrog time steps").
 *
 * PAPER.md L16 SIII.D: "After the copies are done, the particle positions are
 * updated by the CPU"; the integrator is unnamed (reading R23: kick-drift-kick
 * leapfrog).  On B200 the update runs on the GPU on each rank's own slice.
 * All arrays are DEVICE pointers of n fp32 values; the call is asynchronous on
 * `stream` (cudaStream_t as void*, NULL = legacy default stream).
 * Arithmetic: one fused multiply-add per component (single RN rounding).
 * Errors: AFMM_EINVAL (n < 0, null pointer, non-finite step), AFMM_ECUDA.
 */
#ifndef AFMM_STEP_H
#define AFMM_STEP_H

#include "afmm_p2p.h"

#ifdef __cplusplus
extern "C" {
#endif

/* kick:  v <- v + h * a   (h = dt/2 in KDK) */
afmm_status afmm_kick(long long n, float *vx, float *vy, float *vz, const float *ax, const float *ay,
                      const float *az, float h, void *stream);

/* drift: x <- x + dt * v */
afmm_status afmm_drift(long long n, float *x, float *y, float *z, const float *vx, const float *vy,
                       const float *vz, float dt, void *stream);

/* kick then drift in one pass (the first two updates of a KDK step):
 * v <- v + h * a, then x <- x + dt * v with the kicked v -- the same two
 * roundings per component as afmm_kick followed by afmm_drift (bit-identical),
 * one read of a, v, x and one write of v, x instead of two launches. */
afmm_status afmm_kick_drift(long long n, float *x, float *y, float *z, float *vx, float *vy, float *vz,
                            const float *ax, const float *ay, const float *az, float h, float dt, void *stream);

#ifdef __cplusplus
}
#endif
#endif /* AFMM_STEP_H */
