// p2p_kernel.cuh -- the near-field P2P kernel for sm_100a.
//
// What it computes (PAPER.md L12 SI.C, L16 SIII.C; pair law reading R1-R3 in
// DESIGN.md): for every target body i of a target leaf t and every source body
// j of U(t), j != i,
//     phi_i -= G m_j / r,   a_i += G m_j d / r^3,   d = x_j - x_i,  r^2 = |d|^2 + eps2.
//
// B200 design: every warp is an autonomous pipeline.
//  * Work = tasks of <= 128 targets (one leaf, or a 128-target slice of a big
//    leaf), ordered largest-cost-first by the host; warps claim tasks from an
//    atomic queue one task ahead and prefetch its descriptors.
//  * A task's sources (its own leaf first, then runs of consecutive U-list
//    leaves merged into contiguous body segments) stream through a private
//    kWStages x kWCap-body shared-memory ring per warp, filled by 1-D TMA bulk
//    copies (cp.async.bulk ... mbarrier::complete_tx) one chunk ahead of the
//    math -- across task boundaries, so the ring never drains between tasks.
//  * lane mapping: 4 targets per lane as two FFMA2 pairs (the source coordinate
//    broadcast as the .F32 operand; two independent chains per source),
//    g = ceil(n/4) lanes per copy and C = 32/g source-split copies per warp, so
//    adaptive leaves of any size keep the lanes busy (the paper's
//    one-thread-per-target blocks idle them, L16 SIII.C).  No CTA barrier
//    anywhere: reductions over copies are warp-local.
//  * math: rsqrt.approx.ftz; 13 packed FP32 ops + 2 MUFU per two interactions.
//  * accumulation (reading R17): fp32 partials over <= kFold (256) sources per
//    copy, folded into fp64 accumulators in shared memory; at the task's end the
//    copies are reduced by a fixed-order fp64 shuffle tree; one RN rounding to fp32.  Deterministic and independent of
//    the partition (bit-identical across world sizes).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace afmm {

// Tuning knobs (overridable with -D for tools/tune builds; defaults are the product's).
#ifndef AFMM_WCAP
#define AFMM_WCAP 448
#endif
#ifndef AFMM_WSTAGES
#define AFMM_WSTAGES 2
#endif
#ifndef AFMM_WARPS
#define AFMM_WARPS 12
#endif
#ifndef AFMM_MINB
#define AFMM_MINB 1
#endif
#ifndef AFMM_UNROLL
#define AFMM_UNROLL 4
#endif
#ifndef AFMM_FOLD
#define AFMM_FOLD 256
#endif
#ifndef AFMM_PACK_WIDE
#define AFMM_PACK_WIDE 1                          // pack_chunk_kernel: float4 reads when aligned
#endif
#ifndef AFMM_TSPAN
#define AFMM_TSPAN 1                              // device-timer span of the launch (P2PParams.tspan)
#endif
#ifndef AFMM_PROF
#define AFMM_PROF 0                               // per-warp cycle breakdown (tools/prof_breakdown.py)
#endif
#if AFMM_PROF
constexpr int kProfSlots = 16;
__device__ unsigned long long afmm_prof_buf[148 * 32 * kProfSlots];
#define PROF_T(v) const long long v = clock64()
#define PROF_ADD(k, t0) (prof ? (void)(prof[k] += clock64() - (t0)) : (void)0)
#else
#define PROF_T(v)
#define PROF_ADD(k, t0)
#endif
constexpr int kWarps = AFMM_WARPS;              // warps per CTA (all consumers)
constexpr int kThreads = 32 * kWarps;
constexpr int kWCap = AFMM_WCAP;                // bodies per warp stage
constexpr int kWStages = AFMM_WSTAGES;          // per-warp TMA ring depth
#ifndef AFMM_TPT
#define AFMM_TPT 4
#endif
constexpr int kTPT = AFMM_TPT;                  // targets per lane (even)
constexpr int kPairs = kTPT / 2;                // FFMA2 pairs per lane
constexpr int kVals = 4 * kTPT;                 // fp64 accumulators per lane (ax, ay, az, phi per target)
constexpr int kTaskTargets = kTPT * 32;         // targets per task (32 lanes x kTPT)
constexpr int kFold = AFMM_FOLD;                // fp32 partial length per copy before the fp64 fold
constexpr int kMinBlocksPerSM = AFMM_MINB;
constexpr int kUnroll = AFMM_UNROLL;            // inner-loop unroll (sources)
constexpr int kStageBytesW = kWStages * kWCap * 16;     // per warp
constexpr int kAccBytesW = kVals * 32 * 8;              // per warp
constexpr int kDynSmem = kWarps * (kStageBytesW + kAccBytesW);
static_assert(4 * kTaskTargets * (int)sizeof(float) <= kAccBytesW, "output staging must fit the accumulator area");

// ---- target slicing (host and device worklist builders share this; SURVEY
// S8(a) a5 "leaves bucketed by size, so adaptive leaves of 1..S bodies do not
// idle lanes").  A slice of m <= 128 targets runs on g = ceil(m/4) lanes per
// copy and C = 32/g source-split copies, i.e. ceil(nsrc/C) warp iterations.
// Only the largest m of each C matters (a smaller slice with the same C costs
// the same), so the candidates are m in {4,8,12,16,20,24,32,40,64,128}.  A leaf
// of tn targets is cut into slices by an exact integer DP minimising
//     sum_slices ceil(nsrc / C(m)) + kSliceTaskCost,
// the second term standing for a task's fixed cost (descriptors, first-chunk
// latency, copy reduction) in warp iterations.  Integer arithmetic only, so the
// host and device builders produce identical task lists.
#ifndef AFMM_STATIC_FRAC
#define AFMM_STATIC_FRAC 0.9                      // share of the tasks dealt statically (snake rounds) ...
#endif
#ifndef AFMM_STATIC_MIN_TASKS
#define AFMM_STATIC_MIN_TASKS 48                  // ... when there are at least this many tasks per warp
#endif
#ifndef AFMM_TASK_COST
#define AFMM_TASK_COST 32
#endif
constexpr int kSliceCands = 10;
constexpr long long kSliceTaskCost = AFMM_TASK_COST;
constexpr int kMaxDpSlices = 2 * kTaskTargets / kTPT + 1;   // slices of the DP part (< 2 kTaskTargets targets)
// candidate copy counts C (each the largest g = 32 / C lanes per copy), and the
// largest slice for each: m = kTPT * floor(32 / C)
__host__ __device__ __forceinline__ int slice_cand_C(int i) {
    return i == 0 ? 32 : i == 1 ? 16 : i == 2 ? 10 : i == 3 ? 8 : i == 4 ? 6 : i == 5 ? 5 : i == 6 ? 4 : i == 7 ? 3
         : i == 8 ? 2 : 1;
}
__host__ __device__ __forceinline__ int slice_cand_m(int i) { return kTPT * (32 / slice_cand_C(i)); }
__host__ __device__ __forceinline__ int slice_copies(int m) {   // C = 32 / ceil(m / kTPT)
    return 32 / ((m + kTPT - 1) / kTPT);
}
__host__ __device__ __forceinline__ long long slice_iters(long long nsrc, int m) {
    const long long C = slice_copies(m), ns = nsrc > 1 ? nsrc : 1;
    return (ns + C - 1) / C;
}
// Task-size cap (strong scaling): a slice may cost at most `cap` warp iterations,
// so the largest task stays a small fraction of a warp's share of the launch (with
// few tasks per warp the kernel would otherwise last as long as its largest task).
// Candidates whose ceil(nsrc / C) exceeds the cap are dropped, except m = kTPT
// (C = 32), the smallest slice.  Leaves of 2 M or more targets, M the largest
// allowed candidate, first take full M-target slices until < 2 M remain
// (tn % M + M, so the remainder may still merge with one full block); the DP cuts
// the rest.  Returns the number of DP slices and writes their sizes (each
// 1..kTaskTargets) to sz[0..k); *n_full = leading full slices of *full_m targets;
// *max_m (optional) = the largest slice, which has the largest cost (slice_iters is
// nondecreasing in m).
__host__ __device__ inline int plan_slices(int tn, long long nsrc, long long cap, int *n_full, int *full_m,
                                           unsigned short *sz, int *max_m = nullptr) {
    bool ok[kSliceCands];
    int M = slice_cand_m(0);
#pragma unroll
    for (int i = 0; i < kSliceCands; ++i) {
        ok[i] = i == 0 || slice_iters(nsrc, slice_cand_m(i)) <= cap;
        if (ok[i]) M = slice_cand_m(i);
    }
    int rest = tn, full = 0;
    if (tn >= 2 * M) {
        rest = tn % M + M;
        full = (tn - rest) / M;
    }
    *n_full = full;
    *full_m = M;
    long long cost[kSliceCands];
#pragma unroll
    for (int i = 0; i < kSliceCands; ++i) cost[i] = slice_iters(nsrc, slice_cand_m(i)) + kSliceTaskCost;
    // Every candidate is a multiple of kTPT, so f(a) -- the best cost of cutting a
    // targets -- is constant on each block (kTPT(q-1), kTPT q] (induction: a - m
    // stays in one block), and so is the argmin: the DP runs over blocks q.  The
    // last kHist values of f are a shift register (fh[j] = f(q - 1 - j), f = 0 at
    // and before block 0), so every candidate reads a fixed register.
    constexpr int kHist = kTaskTargets / kTPT;
    long long fh[kHist];
#pragma unroll
    for (int j = 0; j < kHist; ++j) fh[j] = 0;
    unsigned char arg[2 * kTaskTargets / kTPT + 1];
    const int nb = (rest + kTPT - 1) / kTPT;
    for (int q = 1; q <= nb; ++q) {
        long long best = -1;
        int bi = 0;
#pragma unroll
        for (int i = 0; i < kSliceCands; ++i) {
            if (!ok[i]) continue;
            const long long v = fh[slice_cand_m(i) / kTPT - 1] + cost[i];
            if (best < 0 || v < best) {
                best = v;
                bi = i;
            }
        }
#pragma unroll
        for (int j = kHist - 1; j > 0; --j) fh[j] = fh[j - 1];
        fh[0] = best;
        arg[q] = (unsigned char)bi;
    }
    int k = 0, mx = full > 0 ? M : 0;
    for (int a = rest; a > 0;) {
        const int mc = slice_cand_m(arg[(a + kTPT - 1) / kTPT]);
        const int m = mc < a ? mc : a;
        sz[k++] = (unsigned short)m;
        mx = m > mx ? m : mx;
        a -= m;
    }
    if (max_m) *max_m = mx;
    return k;
}
// Size of slice j of a plan (full slices first).
__host__ __device__ __forceinline__ int plan_size(int j, int n_full, int full_m, const unsigned short *sz) {
    return j < n_full ? full_m : sz[j - n_full];
}
// Cap for a rank whose tasks total about `inter` interactions on `warps` warps:
// inter / (32 lanes * kTPT) warp iterations if every lane slot were used, split
// kCapDiv ways per warp; never below kCapMin.
#ifndef AFMM_CAP_DIV
#define AFMM_CAP_DIV 3
#endif
constexpr long long kCapMin = 64;
__host__ __device__ inline long long task_cap(long long inter, long long warps) {
    const long long c = inter / ((long long)kTaskTargets * (warps > 0 ? warps : 1) * AFMM_CAP_DIV);
    return c > kCapMin ? c : kCapMin;
}

// Task: targets [tgt_start, +tgt_count <= 128) of the leaf whose bodies start
// at self_start; self_len = the leaf's size if it is in its own U-list (then
// the first segment is the leaf itself), else 0; sources = segments
// [seg_begin, +seg_count) totalling nsrc bodies.
struct Task {
    int tgt_start, tgt_count, self_start, self_len, seg_begin, seg_count, nsrc;
    int piece;               // pipelined host evaluation: output piece (low 16 bits) and the last input
                             // chunk its sources and targets need (high 16 bits); else 0
};
// Segment: bodies [gstart, gstart+len).
struct Seg {
    int gstart, len;
};

constexpr int kMaxWin = 8;                     // own outputs + up to 7 peers (one NVSwitch box)
struct P2PParams {
    const float4 *bodies;    // packed {x,y,z,m}, tree order
    const Task *tasks;
    const Seg *segs;
    int n_tasks;
    int *queue;              // task counter of the dynamic tail, zeroed before launch
    int static_rounds;       // R: tasks [0, R*W) are dealt to the W warps in snake order (no atomic),
                             // tasks [R*W, n_tasks) are claimed from `queue`
    float *out[kMaxWin][4];  // output windows {ax, ay, az, phi}: [0] = this eval's outputs, [1, n_win) = peer
                             // ranks' output arrays (NVLink P2P / IPC pointers): the fused gather (row a7)
    int n_win;
    float eps2;
    double G;                // output scale: G (gravity) or 1/(8 pi mu) (Stokeslet)
    int *done;               // nullptr, or per-piece counters of finished tasks (afmm_p2p_eval_host_pipelined)
    // streamed inputs (afmm_p2p_eval_host_pipelined; the chunked body replication of
    // afmm_p2p_eval at world > 1): nullptr, or the mask of input chunks already in
    // place (bit k = chunk k; written by a stream memory operation on the copy /
    // communication stream); a task whose sources and targets lie in the chunks of
    // need = piece >> 16 waits until (*in_ready & need) == need.  *in_err is set if
    // a wait exceeds wait_ns (never delivered: results invalid, reported as an error)
    const unsigned *in_ready;
    int *in_err;
    unsigned long long wait_ns;
    unsigned in_epoch;       // *in_ready = (epoch << 16) | mask: a word of an older evaluation (another
                             // epoch) counts as nothing delivered, so the flag is never reset between evals
    // nullptr, or {min CTA start, max warp end} in %globaltimer ns (the kernel's
    // device-timer span: the GPU time all-reduced over ranks, L20 SVII.A)
    unsigned long long *tspan;
    // equal masses: nullptr, or the packed-body trailer word that the pack kernel
    // sets when some m_j differs from m_0 (0 = all equal -> the 12-op pair loop,
    // the common mass applied in the epilogue)
    const int *mass_unequal;
    // streamed inputs only: nullptr, or a word whose bit k is set when some mass in
    // input chunk k differs from m_0; a task runs the equal-mass loop when the bits
    // of its need mask are clear (read after the task's wait_inputs, so every bit it
    // looks at is final)
    const unsigned *mass_bits;
    float m0;                // streamed inputs: m_0 (from the host), the equal-mass scale's mass ...
    const float *m0_ptr;     // ... or, if not null, read from here after the task's wait (the packed
                             // array's trailer: chunked replication, where the host does not know m_0)
    // 1: outputs are written through shared memory as whole runs of consecutive
    // targets per component (host-mapped output arrays: full PCIe lines, not 4-byte
    // pieces with byte enables)
    int out_coalesce;
};

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t *b, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *b, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.release.cta.shared::cta.b64 _, [%0], %1;"
                 ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *b, uint32_t parity) {
    asm volatile(
        "{\n"
        ".reg .pred P1;\n"
        "LAB_WAIT:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
        "@P1 bra DONE;\n"
        "bra LAB_WAIT;\n"
        "DONE:\n"
        "}\n" ::"r"(smem_u32(b)), "r"(parity) : "memory");
}
// 1-D bulk async copy global -> shared, completion counted on an mbarrier (TMA).
__device__ __forceinline__ void tma_load_1d(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
        ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
#if AFMM_PROF
__device__ __forceinline__ long long __smid_dummy() {
    unsigned r;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(r));
    return r;
}
#endif
__device__ __forceinline__ float rsqrt_ftz(float x) {
    float y;
    asm("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

// One source against two targets (FFMA2; 13 packed FP32 ops + 2 MUFU.RSQ).
// n{x,y,z} hold the NEGATED target coordinates.
template <bool kMasked, bool kEq = false>
__device__ __forceinline__ void interact2(const float4 q, const float2 nx, const float2 ny,
                                          const float2 nz, const float2 e2, float2 &ax, float2 &ay,
                                          float2 &az, float2 &ph, bool skip0, bool skip1) {
    const float2 dx = __fadd2_rn(make_float2(q.x, q.x), nx);
    const float2 dy = __fadd2_rn(make_float2(q.y, q.y), ny);
    const float2 dz = __fadd2_rn(make_float2(q.z, q.z), nz);
    float2 r2 = __ffma2_rn(dx, dx, e2);
    r2 = __ffma2_rn(dy, dy, r2);
    r2 = __ffma2_rn(dz, dz, r2);
    float2 inv;
    inv.x = rsqrt_ftz(r2.x);
    inv.y = rsqrt_ftz(r2.y);
    if (kMasked) {                       // j == i: drop the self pair (reading R2)
        inv.x = skip0 ? 0.0f : inv.x;
        inv.y = skip1 ? 0.0f : inv.y;
    }
    // equal masses (kEq): the common mass m is applied once in the epilogue, so the
    // pair needs 1/r and 1/r^3 only (12 packed ops instead of 13)
    const float2 t = kEq ? inv : __fmul2_rn(make_float2(q.w, q.w), inv);   // m_j / r
    ph = __fadd2_rn(ph, t);
    const float2 i2 = __fmul2_rn(inv, inv);
    const float2 s = __fmul2_rn(t, i2);                         // m_j / r^3
    ax = __ffma2_rn(s, dx, ax);
    ay = __ffma2_rn(s, dy, ay);
    az = __ffma2_rn(s, dz, az);
}

// ---- pair laws.  A source occupies kWords float4 in the staged ring; the
// four fp32 partial pairs are (ax, ay, az, phi) for gravity and (ux, uy, uz, -)
// for Stokeslets.
struct Gravity {
    static constexpr int kWords = 1;
    static constexpr bool kMaskSelf = true;        // reading R2: the j == i pair is excluded
    static constexpr bool kHasEq = true;           // an equal-mass variant exists
    template <bool kMasked, bool kEq>
    __device__ __forceinline__ static void apply(const float4 *__restrict__ src, int k, const float2 nx,
                                                 const float2 ny, const float2 nz, const float2 e2, float2 &a0,
                                                 float2 &a1, float2 &a2, float2 &a3, bool s0, bool s1) {
        interact2<kMasked, kEq>(src[k], nx, ny, nz, e2, a0, a1, a2, a3, s0, s1);
    }
    // a = G v, phi = -G v
    __device__ __forceinline__ static float out(int comp, double v, double scale) {
        return (float)(comp == 3 ? -scale * v : scale * v);
    }
    __device__ __forceinline__ static float outf(int comp, float v, float scale) {
        return comp == 3 ? -__fmul_rn(scale, v) : __fmul_rn(scale, v);
    }
};

// Regularized Stokeslet (reading R26; PAPER L22 SVIII.B "method of regularized
// Stokeslets as described in [15]"): u_i += [f_k (r^2 + 2 e^2) + (f_k . d) d] /
// (r^2 + e^2)^{3/2} (times 1/(8 pi mu) at the end); the self term is finite and
// included.  Source words: {x, y, z, fx}, {fy, fz, 0, 0}.  Per two interactions:
// 19 packed FP32 ops + 2 MUFU.RSQ.
struct Stokeslet {
    static constexpr int kWords = 2;
    static constexpr bool kMaskSelf = false;
    static constexpr bool kHasEq = false;
    template <bool kMasked, bool kEq>
    __device__ __forceinline__ static void apply(const float4 *__restrict__ src, int k, const float2 nx,
                                                 const float2 ny, const float2 nz, const float2 e2, float2 &ux,
                                                 float2 &uy, float2 &uz, float2 &, bool, bool) {
        const float4 q0 = src[2 * k], q1 = src[2 * k + 1];
        const float2 dx = __fadd2_rn(make_float2(q0.x, q0.x), nx);
        const float2 dy = __fadd2_rn(make_float2(q0.y, q0.y), ny);
        const float2 dz = __fadd2_rn(make_float2(q0.z, q0.z), nz);
        float2 r2 = __ffma2_rn(dx, dx, e2);                      // r^2 + e^2
        r2 = __ffma2_rn(dy, dy, r2);
        r2 = __ffma2_rn(dz, dz, r2);
        float2 inv;
        inv.x = rsqrt_ftz(r2.x);
        inv.y = rsqrt_ftz(r2.y);
        const float2 i3 = __fmul2_rn(__fmul2_rn(inv, inv), inv);  // (r^2 + e^2)^{-3/2}
        const float2 fx = make_float2(q0.w, q0.w), fy = make_float2(q1.x, q1.x), fz = make_float2(q1.y, q1.y);
        float2 fd = __fmul2_rn(fx, dx);
        fd = __ffma2_rn(fy, dy, fd);
        fd = __ffma2_rn(fz, dz, fd);
        const float2 a = __ffma2_rn(e2, i3, inv);                 // (r^2 + 2 e^2) (r^2 + e^2)^{-3/2}
        const float2 b = __fmul2_rn(fd, i3);                      // (f . d) (r^2 + e^2)^{-3/2}
        ux = __ffma2_rn(b, dx, __ffma2_rn(a, fx, ux));
        uy = __ffma2_rn(b, dy, __ffma2_rn(a, fy, uy));
        uz = __ffma2_rn(b, dz, __ffma2_rn(a, fz, uz));
    }
    // u = v / (8 pi mu); the fourth output is zero
    __device__ __forceinline__ static float out(int comp, double v, double scale) {
        return comp == 3 ? 0.0f : (float)(scale * v);
    }
    __device__ __forceinline__ static float outf(int comp, float v, float scale) {
        return comp == 3 ? 0.0f : __fmul_rn(scale, v);
    }
};

// Targets of one lane: kPairs FFMA2 pairs (negated coordinates) and the
// staged-list index of each target (-1: padding slot).
struct Targets {
    float2 nx[kPairs], ny[kPairs], nz[kPairs];
    int m[kTPT];
};

// fp32 partial sums of one copy plus the lane's fp64 accumulators in shared
// memory ([kVals][32] per warp, conflict free; u = 4*target_slot + component).
struct Partial {
    float2 ax[kPairs], ay[kPairs], az[kPairs], ph[kPairs];
    int cnt;                              // sources since the last fold
    bool folded;                          // the fp64 accumulators hold this task's earlier partials
    double *acc;                          // &acc_w[0][lane]
    __device__ __forceinline__ void clear() {
#pragma unroll
        for (int q = 0; q < kPairs; ++q) ax[q] = ay[q] = az[q] = ph[q] = make_float2(0.f, 0.f);
        cnt = 0;
    }
    // fp32 partial -> fp64 accumulators (the first fold of a task initialises them,
    // so nothing is zeroed at task start and tasks that never fold never touch them)
    __device__ __forceinline__ void fold() {
        if (folded) {
#pragma unroll
            for (int q = 0; q < kPairs; ++q) {
                double *a = acc + 8 * q * 32;
                a[0 * 32] += (double)ax[q].x; a[1 * 32] += (double)ay[q].x;
                a[2 * 32] += (double)az[q].x; a[3 * 32] += (double)ph[q].x;
                a[4 * 32] += (double)ax[q].y; a[5 * 32] += (double)ay[q].y;
                a[6 * 32] += (double)az[q].y; a[7 * 32] += (double)ph[q].y;
            }
        } else {
#pragma unroll
            for (int q = 0; q < kPairs; ++q) {
                double *a = acc + 8 * q * 32;
                a[0 * 32] = (double)ax[q].x; a[1 * 32] = (double)ay[q].x;
                a[2 * 32] = (double)az[q].x; a[3 * 32] = (double)ph[q].x;
                a[4 * 32] = (double)ax[q].y; a[5 * 32] = (double)ay[q].y;
                a[6 * 32] = (double)az[q].y; a[7 * 32] = (double)ph[q].y;
            }
        }
        folded = true;
        clear();
    }
};

// Lane mapping of a task with g lanes per copy (1 <= g <= 32): C = 32 / g copies,
// rcpC = ceil(2^16 / C), rcpG = ceil(2^16 / g) (floor(lane * rcpG / 2^16) == lane / g
// for lane < 32).  Packed {C | rcpC << 8, rcpG}, read from the constant bank.
struct LaneMapTable {
    int2 v[33];
    constexpr LaneMapTable() : v() {
        for (int g = 1; g <= 32; ++g) {
            const int C = 32 / g;
            v[g].x = C | (((65536 + C - 1) / C) << 8);
            v[g].y = (65536 + g - 1) / g;
        }
    }
};
__constant__ constexpr LaneMapTable kLaneMap{};
__device__ __forceinline__ int2 lane_map(int g) { return kLaneMap.v[g]; }

// Consume sources src[k], k = k0, k0+C, ... < kend; fp32 partials are folded
// into fp64 before they would exceed kFold sources.  Masks compare k with
// T.m[j] - moff.  rcpC = ceil(2^16 / C): floor(N rcpC / 2^16) == floor(N / C)
// exactly for 0 <= N < 2048, C <= 32 (no integer division in the loop setup).
template <class Law, bool kMasked, bool kEq>
__device__ __forceinline__ void consume(const float4 *__restrict__ src, int k, int kend, int C, int rcpC,
                                        const Targets &T, int moff, const float2 e2, Partial &P) {
    while (k < kend) {
        if (P.cnt >= kFold) P.fold();
        const int span = min(kend - k, (kFold - P.cnt) * C);
        const int iters = ((span + C - 1) * rcpC) >> 16;            // ceil(span / C)
#pragma unroll kUnroll
        for (int it = 0; it < iters; ++it, k += C) {
#pragma unroll
            for (int q = 0; q < kPairs; ++q)
                Law::template apply<kMasked, kEq>(src, k, T.nx[q], T.ny[q], T.nz[q], e2, P.ax[q], P.ay[q], P.az[q],
                                             P.ph[q], kMasked && k == T.m[2 * q] - moff,
                                             kMasked && k == T.m[2 * q + 1] - moff);
        }
        P.cnt += iters;
    }
}

// Per-stage metadata of a warp's ring (written by lane 0 at issue time).
struct ChunkMeta {
    int tgt_start, tgt_count, toff, self_len, first, nb, is_first, is_last, piece;
};

// Issue side of a warp's pipeline: the task whose sources are being streamed
// and the task after it (claimed one task ahead; a deeper prefetch costs more
// registers than its latency saves).  Descriptors are warp-uniform; segments live in lanes (lane i holds segment i of its task) and
// `pre` is the exclusive prefix of the current task's segment lengths, so every
// lane can issue the bulk copy of its own segment's part of a chunk.
struct Stream {
    int task, nxt;                // task ids (>= n_tasks: none)
    Task t;                       // the current task's descriptor (warp-uniform); the next one's is
                                  // prefetched into shared memory (desc[slot], cp.async)
    Task *desc;                   // this warp's two descriptor slots
    int slot;                     // the slot holding (or receiving) task nxt's descriptor
    Seg sg;                       // this lane's segment of t
    int pre;                      // sum of the lengths of t's segments before this lane's (seg_count <= 32)
    bool pre_ok;                  // pre computed (deferred to t's first chunk issue)
    int staged;                   // sources of t already staged
    int seq;                      // tasks this warp has taken (claim)
};

// Rounds of the static deal for n tasks over W warps: floor(frac * n / W) when
// tasks are small and many (>= AFMM_STATIC_MIN_TASKS per warp, small S: there the
// claim's atomic latency is a visible share of a task), else 0 (all dynamic: with
// few, long tasks the cost model's error would unbalance a static deal).  A/B on
// C2: S = 32 +4.6 %, S = 512 -9 % if dealt statically (DESIGN.md v10).
__host__ __device__ inline int static_rounds(int n, int W) {
    if (W <= 0 || n < (long long)AFMM_STATIC_MIN_TASKS * W) return 0;
    return (int)((double)AFMM_STATIC_FRAC * n / W);
}
// The warp's seq-th task.  Tasks are sorted largest-cost-first; the first R
// rounds of W (= all warps of the grid) are dealt in snake order -- round r
// gives warp w task r*W + w (r even) or r*W + W-1-w (r odd), an LPT-style deal
// that needs no atomic and whose ids are known ahead -- and the smaller tasks
// after them are claimed dynamically, which absorbs the static part's error.
__device__ __forceinline__ int claim(const P2PParams &p, int &seq, int lane) {
    const int W = gridDim.x * kWarps, gw = blockIdx.x * kWarps + (threadIdx.x >> 5);
    const int r = seq++;
    if (r < p.static_rounds) return r * W + ((r & 1) ? W - 1 - gw : gw);
    int it = 0;
    if (lane == 0) it = atomicAdd(p.queue, 1);
    return p.static_rounds * W + __shfl_sync(0xffffffffu, it, 0);
}
__device__ __forceinline__ void load_desc(const P2PParams &p, int id, Task &t) {
    t = p.tasks[min(id, p.n_tasks - 1)];                 // a past-the-end id reads the last task, never used
}
// The next task's descriptor goes to shared memory by cp.async (lanes 0 and 1,
// 16 bytes each) and is read back when the task becomes current -- a task
// later.  (Held in registers, round 1's prefetched descriptor was merged into the
// loop-carried registers right after its load, so every task advance waited for
// the load: ncu source page, C2 S = 32, 5 % of the samples on one MOV.)
__device__ __forceinline__ void prefetch_desc(const P2PParams &p, int id, Task *slot, int lane) {
    if (lane < 2) {
        const char *src = reinterpret_cast<const char *>(p.tasks + min(id, p.n_tasks - 1)) + 16 * lane;
        asm volatile("cp.async.ca.shared.global [%0], [%1], 16;\n\tcp.async.commit_group;"
                     ::"r"(smem_u32(reinterpret_cast<char *>(slot) + 16 * lane)), "l"(src) : "memory");
    }
}
__device__ __forceinline__ void take_desc(Task &t, const Task *slot, int lane) {
    if (lane < 2) asm volatile("cp.async.wait_group 0;" ::: "memory");
    __syncwarp();
    t = *slot;
}
// this lane's segment of task t (issued when t becomes current; its prefix is
// taken one chunk later, so the load's latency hides behind a chunk of math)
__device__ __forceinline__ Seg load_seg(const P2PParams &p, int id, const Task &t, int lane) {
    Seg sg{0, 0};
    if (id < p.n_tasks && lane < t.seg_count) sg = p.segs[t.seg_begin + lane];
    return sg;
}
__device__ __forceinline__ int excl_prefix(int v, int lane) {
    int inc = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int u = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += u;
    }
    return inc - v;
}

// Bulk copies of the part of segment (gstart, len), whose first source has index
// `pre` in the task's source list, that falls in the chunk [lo, hi).
template <int kWords>
__device__ __forceinline__ void copy_piece(const P2PParams &p, float4 *buf, uint64_t *bar, int gstart, int len,
                                           int pre, int lo, int hi) {
    const int a = max(pre, lo), b = min(pre + len, hi);
    if (a < b)
        tma_load_1d(buf + (size_t)(a - lo) * kWords, p.bodies + (size_t)(gstart + a - pre) * kWords,
                    (uint32_t)(b - a) * 16u * kWords, bar);
}

__device__ __forceinline__ unsigned long long globaltimer_ns() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

// Streamed inputs: before a task's first chunk is staged, wait until every input
// chunk its sources (and targets) reach has arrived: the task's need mask (high
// 16 bits of Task.piece) must be contained in *in_ready, the mask of delivered
// chunks (written by a stream memory operation after each chunk's copy / pack /
// broadcast).  Every lane acquires the word; the proxy fence orders the delivered
// bodies before this warp's bulk copies.  No hang: a wait longer than p.wait_ns
// (globaltimer) sets *in_err, and once *in_err is set every later wait of every
// warp returns at once (the results are invalid and reported as an error).
__device__ __forceinline__ void wait_inputs(const P2PParams &p, int piece) {
    const unsigned need = (unsigned)piece >> 16;
    const auto arrived = [&](unsigned v) { return (v >> 16) == p.in_epoch && (v & need) == need; };
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p.in_ready) : "memory");
    if (!arrived(v)) {
        const unsigned long long t0 = globaltimer_ns();
        for (;;) {
            __nanosleep(256);
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p.in_ready) : "memory");
            if (arrived(v)) break;
            if (*(volatile int *)p.in_err) break;                 // an earlier wait already timed out
            if (globaltimer_ns() - t0 > p.wait_ns) {
                if ((threadIdx.x & 31) == 0) atomicExch(p.in_err, 1);
                break;
            }
        }
    }
    asm volatile("fence.proxy.async.global;" ::: "memory");
}

// Stage the next chunk (<= kWCap bodies) of the stream into `buf`; returns
// false when no task is left.  Lane 0 posts the byte count, then every lane
// whose segment overlaps the chunk issues that piece (no warp-serial walk).
template <int kWords, bool kStream>
__device__ __forceinline__ bool issue_chunk(const P2PParams &p, Stream &S, float4 *buf, uint64_t *bar,
                                            ChunkMeta *meta, int lane, long long *prof = nullptr) {
    if (S.task >= p.n_tasks) return false;
    if (!S.pre_ok) {
        S.pre = excl_prefix(S.sg.len, lane);
        S.pre_ok = true;
    }
    const int nb = min(kWCap / kWords, S.t.nsrc - S.staged);
    if (kStream && p.in_ready && S.staged == 0) wait_inputs(p, S.t.piece);
    PROF_T(t_a);
    if (lane == 0) {
        ChunkMeta m;
        m.tgt_start = S.t.tgt_start;
        m.tgt_count = S.t.tgt_count;
        m.toff = S.t.tgt_start - S.t.self_start;
        m.self_len = S.t.self_len;
        m.first = S.staged;
        m.nb = nb;
        m.is_first = S.staged == 0;
        m.is_last = S.staged + nb >= S.t.nsrc;
        m.piece = S.t.piece;
        *meta = m;
        fence_proxy_async();
        mbar_arrive_expect_tx(bar, (uint32_t)nb * 16u * kWords);
    }
    __syncwarp();
    PROF_ADD(12, t_a);
    PROF_T(t_b);
    const int lo = S.staged, hi = S.staged + nb;
    if (S.t.seg_count <= 32) {
        copy_piece<kWords>(p, buf, bar, S.sg.gstart, S.sg.len, S.pre, lo, hi);
    } else {                                              // rare: > 32 segments, windows of 32
        int base = 0;
        for (int w = 0; w < S.t.seg_count && base < hi; w += 32) {
            Seg sw{0, 0};
            if (w + lane < S.t.seg_count) sw = p.segs[S.t.seg_begin + w + lane];
            const int pre = base + excl_prefix(sw.len, lane);
            copy_piece<kWords>(p, buf, bar, sw.gstart, sw.len, pre, lo, hi);
            base = __shfl_sync(0xffffffffu, pre + sw.len, 31);
        }
    }
    S.staged = hi;
    PROF_ADD(13, t_b);
    PROF_T(t_c);
    if (S.staged >= S.t.nsrc) {                           // advance to the prefetched task
        S.task = S.nxt;
        take_desc(S.t, S.desc + S.slot, lane);
        S.sg = load_seg(p, S.task, S.t, lane);
        S.pre_ok = false;
        S.staged = 0;
        S.nxt = claim(p, S.seq, lane);                    // and prefetch the one after
        S.slot ^= 1;
        prefetch_desc(p, S.nxt, S.desc + S.slot, lane);
    }
    PROF_ADD(14, t_c);
    return true;
}

// Load this lane's targets (4 consecutive of the n targets of the task): from
// the staged self leaf when present in this stage, else from global memory.
template <int kWords>
__device__ __forceinline__ void load_targets(Targets &T, const float4 *__restrict__ stage,
                                             const float4 *__restrict__ bodies, const ChunkMeta &m,
                                             int l, bool active) {
    const bool staged = m.self_len > 0 && m.toff + m.tgt_count <= m.nb;
#pragma unroll
    for (int q = 0; q < kPairs; ++q) {
        float4 b[2];
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            const int j = 2 * q + h;
            const int i = min(kTPT * l + j, m.tgt_count - 1);     // padding slots repeat the last target
            T.m[j] = (kTPT * l + j < m.tgt_count) ? m.toff + i : -1;
            if (active) b[h] = staged ? stage[(size_t)(m.toff + i) * kWords] : bodies[(size_t)(m.tgt_start + i) * kWords];
            else b[h] = make_float4(0.f, 0.f, 0.f, 0.f);
        }
        T.nx[q] = make_float2(-b[0].x, -b[1].x);
        T.ny[q] = make_float2(-b[0].y, -b[1].y);
        T.nz[q] = make_float2(-b[0].z, -b[1].z);
    }
}

// kStream: the streamed features (input-chunk waits, per-task equal-mass test,
// finished-task counters, coalesced host-mapped output stores); a separate
// instantiation so the device path carries none of their registers.
// Register budget pinned at kMaxRegs (= 160: 12 warps x 32 lanes x 160 = 61,440 of
// the SM's 65,536 registers), so the 4,096 left always hold one 128-thread x
// 32-register pack_chunk_kernel block beside a P2P CTA (the streamed inputs of
// afmm_p2p_eval_host_pipelined); afmm_p2p_create re-checks the fit from the
// built kernels' attributes (co_resident_pack) and the pipelined evaluation falls
// back to packing every chunk before the launch when it does not hold.
constexpr int kMaxRegs = kThreads <= 384 ? 160 : ((65536 - 4096) / kThreads) / 8 * 8;   // (tuning builds: more warps)
static_assert(kMinBlocksPerSM == 1 && kMaxRegs * kThreads <= 65536, "register budget: one CTA per SM");
// (The device-path kernel keeps __launch_bounds__: about the same register count, but
// its code under __maxnreg__ measured 1.2 % slower, profiles/r2_ab_regs.txt.)
template <class Law, bool kStream>
__device__ __forceinline__ void p2p_body(const P2PParams &p) {
    extern __shared__ __align__(128) unsigned char dsmem[];
    __shared__ __align__(8) uint64_t full_all[kWarps][kWStages];
    __shared__ ChunkMeta meta_all[kWarps][kWStages];
    __shared__ __align__(16) Task desc_all[kWarps][2];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    float4 (*stage)[kWCap] = reinterpret_cast<float4 (*)[kWCap]>(dsmem + warp * kStageBytesW);
    double *accw = reinterpret_cast<double *>(dsmem + kWarps * kStageBytesW + warp * kAccBytesW);
    uint64_t *full = full_all[warp];
    ChunkMeta *meta = meta_all[warp];
    if (lane == 0) {
        for (int s = 0; s < kWStages; ++s) mbar_init(&full[s], 1);
        fence_mbar_init();
        if (AFMM_TSPAN && p.tspan && warp == 0) atomicMin(p.tspan, globaltimer_ns());
    }
    __syncwarp();
#if AFMM_PROF
    long long prof[kProfSlots] = {0};
    unsigned long long gt0;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(gt0));
    PROF_T(t_all);
#endif

    // ---- start the stream: claim two tasks, fill the ring but one stage
    Stream S;
    S.seq = 0;
    S.desc = desc_all[warp];
    S.slot = 0;
    S.task = claim(p, S.seq, lane);
    load_desc(p, S.task, S.t);
    S.sg = load_seg(p, S.task, S.t, lane);
    S.pre_ok = false;
    S.nxt = claim(p, S.seq, lane);
    prefetch_desc(p, S.nxt, S.desc + S.slot, lane);
    S.staged = 0;
    int issued = 0;
    for (; issued < kWStages - 1; ++issued)
        if (!issue_chunk<Law::kWords, kStream>(p, S, stage[issued % kWStages], &full[issued % kWStages],
                                      &meta[issued % kWStages], lane))
            break;

    const float2 e2 = make_float2(p.eps2, p.eps2);
    bool eqm = Law::kHasEq && p.mass_unequal != nullptr && *p.mass_unequal == 0;
    double scale_eq = p.G * (double)(kStream ? p.m0 : p.bodies[0].w);   // G m for equal masses
    double scale = eqm ? scale_eq : p.G;                               // else G
    float scale_f = (float)scale;
    bool scale_exact = (double)scale_f == scale;
    Targets T;
    Partial P;
    P.acc = accw + lane;
    int g = 1, C = 1, rcpC = 65536, c = 0, l = 0;
    bool active = false;
    P.folded = false;
    for (int q = 0; q < issued; ++q) {
        // keep the ring one chunk ahead (across task boundaries)
        PROF_T(t_is);
        if (issued == q + kWStages - 1) {
            const int s2 = issued % kWStages;
#if AFMM_PROF
            if (issue_chunk<Law::kWords, kStream>(p, S, stage[s2], &full[s2], &meta[s2], lane, prof)) ++issued;
#else
            if (issue_chunk<Law::kWords, kStream>(p, S, stage[s2], &full[s2], &meta[s2], lane)) ++issued;
#endif
        }
        PROF_ADD(0, t_is);
        const int st = q % kWStages;
        PROF_T(t_w);
        mbar_wait(&full[st], (uint32_t)((q / kWStages) & 1));
        const ChunkMeta m = meta[st];
        PROF_ADD(1, t_w);
        PROF_T(t_f);
#if AFMM_PROF
        prof[6] += 1;
        prof[7] += m.is_first;
#endif
        if (m.is_first) {
            g = (m.tgt_count + kTPT - 1) / kTPT;          // kTPT is a power of two: a shift
            const int2 mg = lane_map(g);                  // {C | rcpC << 8, rcpG}: no integer division
            C = mg.x & 255;
            rcpC = mg.x >> 8;
            c = (lane * mg.y) >> 16;                      // lane / g
            l = lane - c * g;
            active = c < C;
            load_targets<Law::kWords>(T, stage[st], p.bodies, m, l, active);
            if (kStream && Law::kHasEq && p.mass_bits) {         // streamed inputs: per-task equal-mass test
                unsigned b;
                asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(b) : "l"(p.mass_bits) : "memory");
                eqm = (b & ((unsigned)m.piece >> 16)) == 0;
                if (p.m0_ptr) scale_eq = p.G * (double)*(const volatile float *)p.m0_ptr;
                scale = eqm ? scale_eq : p.G;
                scale_f = (float)scale;
                scale_exact = (double)scale_f == scale;
            }
            P.clear();
            P.folded = false;
        }
        PROF_ADD(2, t_f);
        PROF_T(t_m);
        if (active) {
            const int kself = Law::kMaskSelf ? min(max(m.self_len - m.first, 0), m.nb) : 0;
            // first k >= kself with k = c (mod C)
            const int k0 = kself <= c ? c : c + C * (((kself - c + C - 1) * rcpC) >> 16);
            if (Law::kHasEq && eqm) {
                if (kself > 0) consume<Law, true, true>(stage[st], c, kself, C, rcpC, T, m.first, e2, P);
                consume<Law, false, true>(stage[st], k0, m.nb, C, rcpC, T, 0, e2, P);
            } else {
                if (kself > 0) consume<Law, true, false>(stage[st], c, kself, C, rcpC, T, m.first, e2, P);
                consume<Law, false, false>(stage[st], k0, m.nb, C, rcpC, T, 0, e2, P);
            }
        }
        PROF_ADD(3, t_m);
        PROF_T(t_l);
        if (m.is_last) {
            // final per-lane values, then a fixed-order tree over the warp's copies
            // (lanes c*g + l2, c < C): round o adds copy c+o into copy c for c = 0 mod 2o
            // (R17).  If no lane folded (every copy's sources fit one fp32 partial) the
            // tree runs on the fp32 partials, else in fp64 on accumulators + partials.
            float o[kVals];                   // outputs (one RN rounding, R18)
            if (__any_sync(0xffffffffu, P.folded)) {
                double v[kVals];
#pragma unroll
                for (int q = 0; q < kPairs; ++q) {
                    const double *a = P.acc + 8 * q * 32;
                    const bool f = active && P.folded;
                    v[8 * q + 0] = (f ? a[0 * 32] : 0.0) + (double)P.ax[q].x;
                    v[8 * q + 1] = (f ? a[1 * 32] : 0.0) + (double)P.ay[q].x;
                    v[8 * q + 2] = (f ? a[2 * 32] : 0.0) + (double)P.az[q].x;
                    v[8 * q + 3] = (f ? a[3 * 32] : 0.0) + (double)P.ph[q].x;
                    v[8 * q + 4] = (f ? a[4 * 32] : 0.0) + (double)P.ax[q].y;
                    v[8 * q + 5] = (f ? a[5 * 32] : 0.0) + (double)P.ay[q].y;
                    v[8 * q + 6] = (f ? a[6 * 32] : 0.0) + (double)P.az[q].y;
                    v[8 * q + 7] = (f ? a[7 * 32] : 0.0) + (double)P.ph[q].y;
                }
                for (int ro = 1; ro < C; ro <<= 1) {
                    const bool take = (c & (2 * ro - 1)) == 0 && c + ro < C;
#pragma unroll
                    for (int u = 0; u < kVals; ++u) {
                        const double w = __shfl_down_sync(0xffffffffu, v[u], ro * g);
                        if (take) v[u] += w;
                    }
                }
#pragma unroll
                for (int u = 0; u < kVals; ++u) o[u] = Law::out(u & 3, v[u], scale);
            } else {
                float f[kVals];
#pragma unroll
                for (int q = 0; q < kPairs; ++q) {
                    f[8 * q + 0] = P.ax[q].x; f[8 * q + 1] = P.ay[q].x;
                    f[8 * q + 2] = P.az[q].x; f[8 * q + 3] = P.ph[q].x;
                    f[8 * q + 4] = P.ax[q].y; f[8 * q + 5] = P.ay[q].y;
                    f[8 * q + 6] = P.az[q].y; f[8 * q + 7] = P.ph[q].y;
                }
                for (int ro = 1; ro < C; ro <<= 1) {
                    const bool take = (c & (2 * ro - 1)) == 0 && c + ro < C;
#pragma unroll
                    for (int u = 0; u < kVals; ++u) {
                        const float w = __shfl_down_sync(0xffffffffu, f[u], ro * g);
                        if (take) f[u] = __fadd_rn(f[u], w);
                    }
                }
                // fp32 G: G*f rounded once in fp32 equals the fp64 product rounded
                // once (the product of two fp32 values is exact in fp64), so this
                // path skips the conversions with bit-identical outputs
#pragma unroll
                for (int u = 0; u < kVals; ++u)
                    o[u] = scale_exact ? Law::outf(u & 3, f[u], scale_f) : Law::out(u & 3, (double)f[u], scale);
            }
            if (kStream && p.out_coalesce) {
                // stage the task's outputs in the (now free) accumulator area as
                // [component][target], then every lane stores consecutive targets
                __syncwarp();
                float *sc = reinterpret_cast<float *>(accw);
                if (active && c == 0) {
#pragma unroll
                    for (int j = 0; j < kTPT; ++j) {
                        const int u = 8 * (j >> 1) + 4 * (j & 1), tgt = kTPT * l + j;
#pragma unroll
                        for (int a = 0; a < 4; ++a) sc[a * kTaskTargets + tgt] = o[u + a];
                    }
                }
                __syncwarp();
#pragma unroll
                for (int a = 0; a < 4; ++a)
                    for (int t = lane; t < m.tgt_count; t += 32) p.out[0][a][m.tgt_start + t] = sc[a * kTaskTargets + t];
            } else if (active && c == 0) {
#pragma unroll
                for (int j = 0; j < kTPT; ++j) {
                    const int tgt = kTPT * l + j;
                    if (tgt < m.tgt_count) {
                        const int u = 8 * (j >> 1) + 4 * (j & 1), i = m.tgt_start + tgt;
                        const float o0 = o[u + 0], o1 = o[u + 1], o2 = o[u + 2], o3 = o[u + 3];
                        p.out[0][0][i] = o0;                    // own outputs
                        p.out[0][1][i] = o1;
                        p.out[0][2][i] = o2;
                        p.out[0][3][i] = o3;
                        if (p.n_win > 1) {                      // then every peer window (fused gather)
#pragma unroll 1
                            for (int w = 1; w < p.n_win; ++w) {
                                p.out[w][0][i] = o0;
                                p.out[w][1][i] = o1;
                                p.out[w][2][i] = o2;
                                p.out[w][3][i] = o3;
                            }
                        }
                    }
                }
            }
            if (kStream && p.done) {      // publish the task's outputs (pipelined copy-back waits on it)
                __threadfence();
                __syncwarp();
                if (lane == 0) atomicAdd(p.done + (m.piece & 0xffff), 1);
            }
        }
        PROF_ADD(4, t_l);
        PROF_T(t_s);
        __syncwarp();                     // stage st (and the accumulators) free again
        PROF_ADD(5, t_s);
    }
    if (p.n_win > 1) __threadfence_system();   // peer-window stores performed before the kernel completes
    if (AFMM_TSPAN && p.tspan && lane == 0) atomicMax(p.tspan + 1, globaltimer_ns());
#if AFMM_PROF
    PROF_ADD(8, t_all);
    unsigned long long gt1;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(gt1));
    prof[9] = (long long)gt0;
    prof[10] = (long long)gt1;
    prof[11] = __smid_dummy();
    if (lane == 0)
        for (int k = 0; k < kProfSlots; ++k) afmm_prof_buf[(blockIdx.x * kWarps + warp) * kProfSlots + k] = prof[k];
#endif
}

template <class Law>
__global__ void __launch_bounds__(kThreads, kMinBlocksPerSM) p2p_kernel_t(const __grid_constant__ P2PParams p) {
    p2p_body<Law, false>(p);
}
template <class Law>
__global__ void __maxnreg__(kMaxRegs) p2p_stream_kernel_t(const __grid_constant__ P2PParams p) {
    p2p_body<Law, true>(p);
}

// Stokeslet bodies: {x, y, z, fx}, {fy, fz, 0, 0}
__global__ void pack_stokeslet_kernel(long long n, const float *__restrict__ x, const float *__restrict__ y,
                                      const float *__restrict__ z, const float *__restrict__ fx,
                                      const float *__restrict__ fy, const float *__restrict__ fz,
                                      float4 *__restrict__ out) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n;
         i += (long long)gridDim.x * blockDim.x) {
        out[2 * i] = make_float4(x[i], y[i], z[i], fx[i]);
        out[2 * i + 1] = make_float4(fy[i], fz[i], 0.f, 0.f);
    }
}

// Streamed-input pack (afmm_p2p_eval_host_pipelined): runs NEXT TO the persistent
// P2P kernel, so it must fit in what a P2P CTA leaves free on an SM (4096
// registers): 128 threads, <= 24 registers, 32-bit indices.  The SoA inputs are
// device staging copies or host-mapped pinned arrays (zero-copy: read over PCIe).
// Sets bit `chunk` of *mass_bits when some mass of the chunk differs from m0.
// With all four inputs 16-byte aligned each thread reads 4 bodies per array as one
// float4 (512-byte warp requests: fewer, fuller PCIe read TLPs in zero-copy mode).
// <= 32 registers (launch bounds): the block must fit beside a P2P CTA.
__global__ void __launch_bounds__(128, 16) pack_chunk_kernel(int n, const float *__restrict__ x,
                                                             const float *__restrict__ y, const float *__restrict__ z,
                                                             const float *__restrict__ m, float4 *__restrict__ out,
                                                             float m0, unsigned *mass_bits, int chunk) {
    bool diff = false;
    int i0 = 0;
    if (AFMM_PACK_WIDE && ((reinterpret_cast<uintptr_t>(x) | reinterpret_cast<uintptr_t>(y) |
                            reinterpret_cast<uintptr_t>(z) | reinterpret_cast<uintptr_t>(m)) & 15) == 0) {
        const int n4 = n >> 2;
        for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += gridDim.x * blockDim.x) {
            const float4 X = reinterpret_cast<const float4 *>(x)[i], Y = reinterpret_cast<const float4 *>(y)[i];
            const float4 Z = reinterpret_cast<const float4 *>(z)[i], M = reinterpret_cast<const float4 *>(m)[i];
            out[4 * i + 0] = make_float4(X.x, Y.x, Z.x, M.x);
            out[4 * i + 1] = make_float4(X.y, Y.y, Z.y, M.y);
            out[4 * i + 2] = make_float4(X.z, Y.z, Z.z, M.z);
            out[4 * i + 3] = make_float4(X.w, Y.w, Z.w, M.w);
            diff |= (M.x != m0) | (M.y != m0) | (M.z != m0) | (M.w != m0);
        }
        i0 = 4 * n4;
    }
    for (int i = i0 + blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
        const float mi = m[i];
        out[i] = make_float4(x[i], y[i], z[i], mi);
        diff |= mi != m0;
    }
    if (__any_sync(0xffffffffu, diff) && (threadIdx.x & 31) == 0) atomicOr(mass_bits, 1u << chunk);
}

// SoA -> packed {x, y, z, m}; the trailer after the bodies: unequal[0] = -1 (all
// bits) when some m_i != m_0 (the equal-mass flag, zeroed before), unequal[1] =
// m_0's bits (the equal-mass scale for ranks that receive the packed array)
__global__ void pack_bodies_kernel(long long n, const float *__restrict__ x, const float *__restrict__ y,
                                   const float *__restrict__ z, const float *__restrict__ m,
                                   float4 *__restrict__ out, int *__restrict__ unequal) {
    const float m0 = m[0];
    if (blockIdx.x == 0 && threadIdx.x == 0) unequal[1] = __float_as_int(m0);
    bool diff = false;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n;
         i += (long long)gridDim.x * blockDim.x) {
        const float mi = m[i];
        out[i] = make_float4(x[i], y[i], z[i], mi);
        diff |= mi != m0;
    }
    if (__any_sync(0xffffffffu, diff) && (threadIdx.x & 31) == 0) atomicOr(unequal, -1);
}

// kernel_ms[0] = the device-timer span of the last P2P launch in ms (0 if none ran)
__global__ void span_ms_kernel(const unsigned long long *__restrict__ tspan, double *__restrict__ kernel_ms) {
    kernel_ms[0] = tspan[1] > tspan[0] ? (double)(tspan[1] - tspan[0]) * 1e-6 : 0.0;
}



}  // namespace afmm
