// p2p_kernel.cuh -- the near-field P2P kernel for sm_100a.
//
// What it computes (PAPER.md L12 SI.C, L16 SIII.C; pair law reading R1-R3 in
// DESIGN.md): for every target body i of a work item (a chunk of <= 512 bodies
// of one target leaf t) and every source body j of U(t), j != i,
//     phi_i -= G m_j / r,   a_i += G m_j d / r^3,   d = x_j - x_i,  r^2 = |d|^2 + eps2.
//
// B200 design:
//  * persistent CTAs (256 threads) pull work items from an atomic queue that
//    the host ordered largest-cost-first;
//  * the item's sources -- a handful of contiguous body segments, the self leaf
//    first -- are staged into shared memory with 1-D TMA bulk copies
//    (cp.async.bulk ... mbarrier::complete_tx), double-buffered so the next
//    chunk lands while this one is consumed;
//  * lane mapping: 2 targets per thread (FFMA2 packed math with the source
//    coordinate broadcast as the .F32 operand), g = ceil(n_t/2) lanes per
//    "copy", C = 256/g copies per CTA; copy c consumes sources c, c+C, ...
//    so leaves of any size 1..512 keep >= 95% of the lanes busy (the paper's
//    one-thread-per-target blocks idle the rest, L16 SIII.C);
//  * accumulation: fp32 partials over <= FOLD sources per copy, folded into fp64;
//    copies reduced in fixed order in fp64 through shared memory; one RN
//    rounding to fp32 at the end.  Deterministic and independent of the
//    partition (bit-identical across world sizes).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace afmm {

constexpr int kThreads = 256;        // threads per CTA
constexpr int kCap = 1024;           // bodies per shared-memory stage (16 KiB)
constexpr int kMaxTargets = 512;     // targets per work item (2 per thread)
constexpr int kFold = 32;            // fp32 partial length per copy before the fp64 fold
constexpr int kMinBlocksPerSM = 4;
constexpr int kStageBytes = 2 * kCap * 16;                   // two TMA stages
constexpr int kDynSmem = kStageBytes + 8 * kThreads * 8;     // + fp64 accumulators

// Work item: targets [tgt_start, tgt_start+tgt_count) of leaf starting at
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

// fp64 accumulators live in shared memory, [8][kThreads] (bank-conflict free),
// so the fp32 inner loop keeps its registers; folded every kFold sources.
struct Acc64 {
    double *p;   // &acc[0][tid]
    __device__ __forceinline__ void add(int u, float v) { p[u * kThreads] += (double)v; }
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

__device__ __forceinline__ void produce(int s, const P2PParams &p, float4 (*stage)[kCap],
                                        uint64_t *full, int *meta_item, int *meta_chunk,
                                        int &p_item, int &p_chunk, int &p_nchunks, int lane) {
    int item = -1, chunk = 0;
    if (lane == 0) {
        if (p_item < p.n_items && p_chunk >= p_nchunks) {
            p_item = atomicAdd(p.queue, 1);
            p_chunk = 0;
            p_nchunks = (p_item < p.n_items) ? p.items[p_item].chunk_count : 0;
            if (p_item > p.n_items) p_item = p.n_items;
        }
        if (p_item < p.n_items) {
            item = p_item;
            chunk = p_chunk++;
        }
    }
    item = __shfl_sync(0xffffffffu, item, 0);
    chunk = __shfl_sync(0xffffffffu, chunk, 0);
    if (item < 0) {
        if (lane == 0) {
            meta_item[s] = -1;
            mbar_arrive(&full[s]);
        }
        return;
    }
    const Chunk ch = p.chunks[p.items[item].chunk_begin + chunk];
    if (lane == 0) {
        meta_item[s] = item;
        meta_chunk[s] = chunk;
        mbar_arrive_expect_tx(&full[s], (uint32_t)ch.nbodies * 16u);
    }
    if (lane == 0) {
        // one elected thread issues the bulk copies (UBLKCP takes uniform operands)
        for (int sg = 0; sg < ch.seg_count; ++sg) {
            const Seg g = p.segs[ch.seg_begin + sg];
            tma_load_1d(&stage[s][g.soff], p.bodies + g.gstart, (uint32_t)g.len * 16u, &full[s]);
        }
    }
}

__global__ void __launch_bounds__(kThreads, kMinBlocksPerSM) p2p_kernel(const P2PParams p) {
    extern __shared__ __align__(128) unsigned char dsmem[];
    float4 (*stage)[kCap] = reinterpret_cast<float4 (*)[kCap]>(dsmem);                 // [2][kCap]
    double (*acc)[kThreads] = reinterpret_cast<double (*)[kThreads]>(dsmem + kStageBytes); // [8][kThreads]
    __shared__ __align__(8) uint64_t full[2];
    __shared__ int meta_item[2], meta_chunk[2];

    const int tid = threadIdx.x;
    const int lane = tid & 31;
    const bool producer = tid < 32;
    int p_item = -1, p_chunk = 0, p_nchunks = 0;   // producer cursor (lane 0 of warp 0)

    if (tid == 0) {
        mbar_init(&full[0], 1);
        mbar_init(&full[1], 1);
        fence_mbar_init();
    }
    __syncthreads();
    if (producer) {
        produce(0, p, stage, full, meta_item, meta_chunk, p_item, p_chunk, p_nchunks, lane);
        produce(1, p, stage, full, meta_item, meta_chunk, p_item, p_chunk, p_nchunks, lane);
    }

    const float2 e2 = make_float2(p.eps2, p.eps2);
    float2 nx = make_float2(0.f, 0.f), ny = nx, nz = nx;
    Acc64 A{&acc[0][threadIdx.x]};
    int g = 1, C = 1, c = 0, l = 0, m0 = -1, m1 = -1;
    bool active = false;

    for (int q = 0;; ++q) {
        const int s = q & 1;
        mbar_wait(&full[s], (uint32_t)((q >> 1) & 1));
        const int item = meta_item[s];
        if (item < 0) break;
        const int chunk = meta_chunk[s];
        const Item it = p.items[item];
        if (chunk == 0) {
            g = (it.tgt_count + 1) >> 1;
            C = kThreads / g;
            c = tid / g;
            l = tid - c * g;
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
            const int nb = p.chunks[it.chunk_begin + chunk].nbodies;
            const int kself = (chunk == 0) ? it.self_len : 0;
            int k = c;
            consume<true>(stage[s], k, kself, C, nx, ny, nz, e2, m0, m1, A);
            consume<false>(stage[s], k, nb, C, nx, ny, nz, e2, m0, m1, A);
        }
        if (chunk == it.chunk_count - 1) {
            // fixed-order fp64 reduction across copies (shared-memory accumulators)
            __syncthreads();
            if (tid < g) {
                double v[8];
#pragma unroll
                for (int u = 0; u < 8; ++u) v[u] = acc[u][tid];
                for (int cc = 1; cc < C; ++cc) {
#pragma unroll
                    for (int u = 0; u < 8; ++u) v[u] += acc[u][cc * g + tid];
                }
                const int i0 = it.tgt_start + 2 * tid;
                p.ax[i0] = (float)(p.G * v[0]);
                p.ay[i0] = (float)(p.G * v[1]);
                p.az[i0] = (float)(p.G * v[2]);
                p.phi[i0] = (float)(-p.G * v[3]);
                if (2 * tid + 1 < it.tgt_count) {
                    p.ax[i0 + 1] = (float)(p.G * v[4]);
                    p.ay[i0 + 1] = (float)(p.G * v[5]);
                    p.az[i0 + 1] = (float)(p.G * v[6]);
                    p.phi[i0 + 1] = (float)(-p.G * v[7]);
                }
            }
        }
        __syncthreads();               // stage s fully consumed
        if (producer) {
            fence_proxy_async();
            produce(s, p, stage, full, meta_item, meta_chunk, p_item, p_chunk, p_nchunks, lane);
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
