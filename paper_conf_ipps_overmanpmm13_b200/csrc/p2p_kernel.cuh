// p2p_kernel.cuh -- the near-field P2P kernel for sm_100a.
//
// What it computes (PAPER.md L12 SI.C, L16 SIII.C; pair law reading R1-R3 in
// DESIGN.md): for every target body i of a work item (a chunk of <= 512 bodies
// of one target leaf t) and every source body j of U(t), j != i,
//     phi_i -= G m_j / r,   a_i += G m_j d / r^3,   d = x_j - x_i,  r^2 = |d|^2 + eps2.
//
// B200 design:
//  * persistent, warp-specialised CTAs: 8 consumer warps + 1 producer warp.
//    The producer pulls work items from an atomic queue (ordered largest-cost-
//    first by the host), loads the chunk/segment descriptors lane-parallel and
//    stages each chunk's source segments (the self leaf first, then merged runs
//    of consecutive U-list leaves) into a kStages-deep shared-memory ring with
//    1-D TMA bulk copies (cp.async.bulk ... mbarrier::complete_tx).  Full/empty
//    mbarriers per stage; consumers never wait on the producer's metadata
//    latency unless the ring runs dry.
//  * lane mapping: 2 targets per consumer thread (FFMA2 packed math, the source
//    coordinate broadcast as the .F32 operand), g = ceil(n_t/2) lanes per
//    "copy", C = min(256/g, kMaxCopies) copies; copy c consumes sources c, c+C,
//    ... so leaves of any size keep the lanes busy (the paper's one-thread-per-
//    target blocks idle the rest, L16 SIII.C).
//  * accumulation: fp32 partials over <= kFold sources per copy, folded into
//    fp64 accumulators in shared memory; copies reduced in fixed order in fp64
//    (one consumer-only named barrier per item); one RN rounding to fp32.
//    Deterministic and independent of the partition (bit-identical across
//    world sizes).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace afmm {

constexpr int kConsumers = 256;                 // consumer threads (8 warps)
constexpr int kThreads = kConsumers + 32;       // + 1 producer warp
constexpr int kCap = 1024;                      // bodies per shared-memory stage (16 KiB)
constexpr int kStages = 3;                      // TMA ring depth
constexpr int kMaxTargets = 512;                // targets per work item (2 per thread)
constexpr int kMaxCopies = 64;                  // source-split copies per item
constexpr int kFold = 64;                       // fp32 partial length per copy before the fp64 fold
constexpr int kMinBlocksPerSM = 3;
constexpr int kStageBytes = kStages * kCap * 16;
constexpr int kDynSmem = kStageBytes + 8 * kConsumers * 8;    // + fp64 accumulators

// Work item: targets [tgt_start, tgt_start+tgt_count) of the leaf starting at
// self_start; its sources are chunks [chunk_begin, chunk_begin+chunk_count).
struct Item {
    int tgt_start, tgt_count, self_start, self_len, chunk_begin, chunk_count, pad0, pad1;
};
// Chunk: segments [seg_begin, seg_begin+seg_count) totalling nbodies (<= kCap).
struct Chunk {
    int seg_begin, seg_count, nbodies, pad;
};
// Segment: bodies [gstart, gstart+len) staged at shared-memory body offset soff.
struct Seg {
    int gstart, len, soff, pad;
};

struct P2PParams {
    const float4 *bodies;    // packed {x,y,z,m}, tree order
    const Item *items;
    const Chunk *chunks;
    const Seg *segs;
    int n_items;
    int *queue;              // work counter, zeroed before launch
    float *ax, *ay, *az, *phi;
    float eps2;
    double G;
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
__device__ __forceinline__ void mbar_arrive(uint64_t *b) {
    asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
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
// named barrier among the consumer warps only (the producer never joins)
__device__ __forceinline__ void consumer_sync() {
    asm volatile("bar.sync 1, %0;" ::"n"(kConsumers) : "memory");
}
// 1-D bulk async copy global -> shared, completion counted on an mbarrier (TMA).
__device__ __forceinline__ void tma_load_1d(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
        ::"r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ float rsqrt_ftz(float x) {
    float y;
    asm("rsqrt.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}

// One source against two targets (FFMA2; 13 packed FP32 ops + 2 MUFU.RSQ).
// n{x,y,z} hold the NEGATED target coordinates.
template <bool kMasked>
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
    const float2 t = __fmul2_rn(make_float2(q.w, q.w), inv);   // m_j / r
    ph = __fadd2_rn(ph, t);
    const float2 i2 = __fmul2_rn(inv, inv);
    const float2 s = __fmul2_rn(t, i2);                         // m_j / r^3
    ax = __ffma2_rn(s, dx, ax);
    ay = __ffma2_rn(s, dy, ay);
    az = __ffma2_rn(s, dz, az);
}

// fp64 accumulators live in shared memory, [8][kConsumers] (conflict free), so
// the fp32 inner loop keeps its registers; folded every kFold sources.
struct Acc64 {
    double *p;   // &acc[0][tid]
    __device__ __forceinline__ void add(int u, float v) { p[u * kConsumers] += (double)v; }
};

// Consume sources k = k0, k0+C, ... < kend of one staged chunk.
template <bool kMasked>
__device__ __forceinline__ void consume(const float4 *__restrict__ src, int &k, int kend, int C,
                                        const float2 nx, const float2 ny, const float2 nz,
                                        const float2 e2, int m0, int m1, Acc64 &A) {
    while (k < kend) {
        float2 ax = make_float2(0.f, 0.f), ay = ax, az = ax, ph = ax;
        const int kstop = min(kend, k + kFold * C);
#pragma unroll 4
        for (; k < kstop; k += C) {
            const float4 q = src[k];
            interact2<kMasked>(q, nx, ny, nz, e2, ax, ay, az, ph, k == m0, k == m1);
        }
        A.add(0, ax.x); A.add(1, ay.x); A.add(2, az.x); A.add(3, ph.x);
        A.add(4, ax.y); A.add(5, ay.y); A.add(6, az.y); A.add(7, ph.y);
    }
}

struct StageMeta {
    int item, chunk;
};

// Producer warp: walk the queue, stage every chunk of every claimed item.
__device__ __forceinline__ void producer_loop(const P2PParams &p, float4 (*stage)[kCap],
                                              uint64_t *full, uint64_t *empty, StageMeta *meta,
                                              int lane) {
    int st = 0;
    uint32_t phase = 0;
    int item = -1, chunk = 0, nchunks = 0, chunk_begin = 0;
    for (;;) {
        if (chunk >= nchunks) {                    // claim the next item
            int it = 0;
            if (lane == 0) it = atomicAdd(p.queue, 1);
            it = __shfl_sync(0xffffffffu, it, 0);
            if (it >= p.n_items) {
                item = -1;
            } else {
                item = it;
                const Item w = p.items[it];
                nchunks = w.chunk_count;
                chunk_begin = w.chunk_begin;
                chunk = 0;
            }
        }
        mbar_wait(&empty[st], phase ^ 1u);         // slot free (passes at once on the first lap)
        if (item < 0) {
            if (lane == 0) {
                meta[st].item = -1;
                mbar_arrive(&full[st]);
            }
            return;
        }
        const Chunk ch = p.chunks[chunk_begin + chunk];
        // lane-parallel descriptor loads (one L2 round trip for up to 32 segments)
        Seg sg = {0, 0, 0, 0};
        if (lane < ch.seg_count) sg = p.segs[ch.seg_begin + lane];
        if (lane == 0) {
            meta[st].item = item;
            meta[st].chunk = chunk;
            fence_proxy_async();
            mbar_arrive_expect_tx(&full[st], (uint32_t)ch.nbodies * 16u);
        }
        __syncwarp();
        if (lane < ch.seg_count)
            tma_load_1d(&stage[st][sg.soff], p.bodies + sg.gstart, (uint32_t)sg.len * 16u, &full[st]);
        for (int base = 32; base < ch.seg_count; base += 32) {      // rare: > 32 segments
            if (base + lane < ch.seg_count) {
                const Seg s2 = p.segs[ch.seg_begin + base + lane];
                tma_load_1d(&stage[st][s2.soff], p.bodies + s2.gstart, (uint32_t)s2.len * 16u, &full[st]);
            }
        }
        ++chunk;
        if (++st == kStages) {
            st = 0;
            phase ^= 1u;
        }
    }
}

__global__ void __launch_bounds__(kThreads, kMinBlocksPerSM) p2p_kernel(const P2PParams p) {
    extern __shared__ __align__(128) unsigned char dsmem[];
    float4 (*stage)[kCap] = reinterpret_cast<float4 (*)[kCap]>(dsmem);                      // [kStages][kCap]
    double (*acc)[kConsumers] = reinterpret_cast<double (*)[kConsumers]>(dsmem + kStageBytes); // [8][kConsumers]
    __shared__ __align__(8) uint64_t full[kStages], empty[kStages];
    __shared__ StageMeta meta[kStages];

    const int tid = threadIdx.x;
    if (tid == 0) {
        for (int s = 0; s < kStages; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], kConsumers / 32);       // one arrive per consumer warp
        }
        fence_mbar_init();
    }
    __syncthreads();
    if (tid >= kConsumers) {                             // ---- producer warp
        producer_loop(p, stage, full, empty, meta, tid & 31);
        return;
    }

    // ---- consumer warps
    const float2 e2 = make_float2(p.eps2, p.eps2);
    float2 nx = make_float2(0.f, 0.f), ny = nx, nz = nx;
    Acc64 A{&acc[0][tid]};
    int g = 1, C = 1, c = 0, m0 = -1, m1 = -1;
    bool active = false;
    int st = 0;
    uint32_t phase = 0;
    for (;;) {
        mbar_wait(&full[st], phase);
        const StageMeta sm = meta[st];
        if (sm.item < 0) break;
        const Item it = p.items[sm.item];
        if (sm.chunk == 0) {
            g = (it.tgt_count + 1) >> 1;
            C = min(kConsumers / g, kMaxCopies);
            c = tid / g;
            const int l = tid - c * g;
            active = c < C;
            const int i0 = 2 * l;
            const int i1 = min(2 * l + 1, it.tgt_count - 1);
            const int toff = it.tgt_start - it.self_start;
            m0 = toff + i0;
            m1 = (2 * l + 1 < it.tgt_count) ? toff + i1 : m0;
            if (active) {
                const float4 b0 = p.bodies[it.tgt_start + i0];
                const float4 b1 = p.bodies[it.tgt_start + i1];
                nx = make_float2(-b0.x, -b1.x);
                ny = make_float2(-b0.y, -b1.y);
                nz = make_float2(-b0.z, -b1.z);
            }
#pragma unroll
            for (int u = 0; u < 8; ++u) acc[u][tid] = 0.0;
        }
        if (active) {
            const int nb = p.chunks[it.chunk_begin + sm.chunk].nbodies;
            const int kself = (sm.chunk == 0) ? it.self_len : 0;
            int k = c;
            consume<true>(stage[st], k, kself, C, nx, ny, nz, e2, m0, m1, A);
            consume<false>(stage[st], k, nb, C, nx, ny, nz, e2, m0, m1, A);
        }
        __syncwarp();
        if ((tid & 31) == 0) mbar_arrive(&empty[st]);     // this warp is done with the stage
        if (sm.chunk == it.chunk_count - 1) {
            // fixed-order fp64 reduction across copies: thread j < 8g reduces
            // component u = j / g of lane l = j % g over the C copies
            consumer_sync();
            for (int j = tid; j < 8 * g; j += kConsumers) {
                const int u = j / g, l = j - u * g;
                double v0 = 0.0, v1 = 0.0;
                int cc = 0;
                for (; cc + 1 < C; cc += 2) {
                    v0 += acc[u][cc * g + l];
                    v1 += acc[u][(cc + 1) * g + l];
                }
                if (cc < C) v0 += acc[u][cc * g + l];
                const double v = v0 + v1;
                const int tgt = 2 * l + (u >> 2);
                if (tgt < it.tgt_count) {
                    const int comp = u & 3;
                    float *dst = comp == 0 ? p.ax : comp == 1 ? p.ay : comp == 2 ? p.az : p.phi;
                    dst[it.tgt_start + tgt] = (float)(comp == 3 ? -p.G * v : p.G * v);
                }
            }
            consumer_sync();                              // acc free for the next item
        }
        if (++st == kStages) {
            st = 0;
            phase ^= 1u;
        }
    }
}

__global__ void pack_bodies_kernel(long long n, const float *__restrict__ x, const float *__restrict__ y,
                                   const float *__restrict__ z, const float *__restrict__ m,
                                   float4 *__restrict__ out) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n;
         i += (long long)gridDim.x * blockDim.x)
        out[i] = make_float4(x[i], y[i], z[i], m[i]);
}

}  // namespace afmm
