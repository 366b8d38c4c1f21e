// tree_build.cu -- GPU adaptive octree + U-list builder (include/afmm_tree.h).
//
// PAPER.md L10 SI.B: "a node is subdivided into eight children if it holds more
// than [S] bodies"; L16 SIII.B builds the tree by "recursive parallel partition
// of the body locations into the child trees on the way down".  The B200 form
// of that partition: fp64 quantisation + 63-bit Morton keys (one kernel), a
// stable radix sort (CUB), then a level-synchronous split where each open node
// finds its octant ranges by binary search in the sorted keys and children are
// placed by an exclusive scan (deterministic, no atomics).  Leaves are numbered
// by a scan over their first-body flags, which is Morton (DFS) order.  U-lists
// come from a per-leaf descent over the node arrays (count, scan, fill).
#include <algorithm>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <string>
#include <vector>

#include <cub/cub.cuh>
#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>

#include "../../include/afmm_tree.h"

namespace {

constexpr int kMaxLevel = 21;

__device__ __forceinline__ unsigned long long spread3(unsigned long long v) {
    v &= 0x1fffffull;
    v = (v | (v << 32)) & 0x1f00000000ffffull;
    v = (v | (v << 16)) & 0x1f0000ff0000ffull;
    v = (v | (v << 8)) & 0x100f00f00f00f00full;
    v = (v | (v << 4)) & 0x10c30c30c30c30c3ull;
    v = (v | (v << 2)) & 0x1249249249249249ull;
    return v;
}
__device__ __forceinline__ unsigned long long compact3(unsigned long long v) {
    v &= 0x1249249249249249ull;
    v = (v ^ (v >> 2)) & 0x10c30c30c30c30c3ull;
    v = (v ^ (v >> 4)) & 0x100f00f00f00f00full;
    v = (v ^ (v >> 8)) & 0x1f0000ff0000ffull;
    v = (v ^ (v >> 16)) & 0x1f00000000ffffull;
    v = (v ^ (v >> 32)) & 0x1fffffull;
    return v;
}

// q = clamp(floor((v - lo) * 2^(21-k)), 0, 2^21 - 1); fp64, explicit RN ops (no FMA)
__device__ __forceinline__ unsigned long long quantize(float v, double lo, double scale) {
    const double t = __dmul_rn(__dsub_rn((double)v, lo), scale);
    const double f = floor(t);
    if (!(f >= 0.0)) return 0ull;
    if (f > 2097151.0) return 2097151ull;
    return (unsigned long long)f;
}

__global__ void minmax_kernel(long long n, const float *__restrict__ x, const float *__restrict__ y,
                              const float *__restrict__ z, float *__restrict__ part) {
    float mn[3] = {INFINITY, INFINITY, INFINITY}, mx[3] = {-INFINITY, -INFINITY, -INFINITY};
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n;
         i += (long long)gridDim.x * blockDim.x) {
        const float v[3] = {x[i], y[i], z[i]};
#pragma unroll
        for (int a = 0; a < 3; ++a) {
            mn[a] = fminf(mn[a], v[a]);
            mx[a] = fmaxf(mx[a], v[a]);
        }
    }
    __shared__ float s[6][256];
#pragma unroll
    for (int a = 0; a < 3; ++a) {
        s[a][threadIdx.x] = mn[a];
        s[3 + a][threadIdx.x] = mx[a];
    }
    __syncthreads();
    for (int w = blockDim.x / 2; w > 0; w >>= 1) {
        if (threadIdx.x < w) {
#pragma unroll
            for (int a = 0; a < 3; ++a) {
                s[a][threadIdx.x] = fminf(s[a][threadIdx.x], s[a][threadIdx.x + w]);
                s[3 + a][threadIdx.x] = fmaxf(s[3 + a][threadIdx.x], s[3 + a][threadIdx.x + w]);
            }
        }
        __syncthreads();
    }
    if (threadIdx.x < 6) part[blockIdx.x * 6 + threadIdx.x] = s[threadIdx.x][0];
}

__global__ void keys_kernel(long long n, const float *__restrict__ x, const float *__restrict__ y,
                            const float *__restrict__ z, double lx, double ly, double lz,
                            double scale, unsigned long long *__restrict__ keys,
                            int *__restrict__ idx) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n;
         i += (long long)gridDim.x * blockDim.x) {
        const unsigned long long qx = quantize(x[i], lx, scale);
        const unsigned long long qy = quantize(y[i], ly, scale);
        const unsigned long long qz = quantize(z[i], lz, scale);
        keys[i] = spread3(qx) | (spread3(qy) << 1) | (spread3(qz) << 2);
        idx[i] = (int)i;
    }
}

struct Nodes {
    int *b, *e, *first_child, *nchild, *level;
    unsigned long long *prefix;
};

// ---- bucket sort of the keys by the previous build's leaf cells (rebuilds in the
// same domain: Enforce_S every C5 step).  The previous leaves are disjoint cells
// in Morton order, so bucket 2j+1 = the keys inside leaf j's cell, bucket 2j+2 =
// the keys between leaf j's cell and leaf j+1's (emptied space), bucket 0 = before
// leaf 0: the buckets' key ranges are disjoint and increasing, so sorting every
// bucket by (key, input index) and concatenating them in bucket order IS the
// stable sort by (key, index) (round 1: CUB's 8-pass 63-bit radix sort).  Most
// bodies stay in their leaf's cell between steps (≈ 74 % on C5), the buckets hold
// about a leaf each, and a warp sorts one (bitonic, <= kBucketCap keys); the few
// larger buckets (a KEEP rebuild lets leaves grow past S) go to a list that one CTA
// each sorts in shared memory (<= kBigCap keys); beyond that a full sort.
constexpr int kBucketCap = 512;
constexpr int kBigCap = 8192, kBigList = 128, kBigThreads = 1024;
constexpr size_t kBigSmem = (size_t)kBigCap * (sizeof(unsigned long long) + sizeof(int));
__global__ void cell_range_kernel(const int *__restrict__ Ldev, const int *__restrict__ ll,
                                  const unsigned long long *__restrict__ lp, unsigned long long *__restrict__ clo,
                                  unsigned long long *__restrict__ chi) {
    const int L = *Ldev;                          // the previous build's leaf count (device word: graph-stable)
    const int j = blockIdx.x * blockDim.x + threadIdx.x;
    if (j >= L) return;
    const int sh = 3 * (kMaxLevel - ll[j]);
    clo[j] = lp[j] << sh;
    chi[j] = (lp[j] + 1ull) << sh;
}
// keys (as keys_kernel) + the bucket of each key: the first previous leaf whose cell
// starts above the key, by a binary search over every kSampleStride-th cell start
// staged in shared memory, then over the <= stride leaves it leaves open; the
// bucket's counter is bumped once per warp and bucket (bodies arrive nearly in
// key order, so a warp's keys mostly share one bucket)
constexpr int kMaxSamples = 1024, kKeysThreads = 512;
__global__ void __launch_bounds__(kKeysThreads) keys_bucket_kernel(
    long long n, const float *__restrict__ x, const float *__restrict__ y, const float *__restrict__ z, double lx,
    double ly, double lz, double scale, unsigned long long *__restrict__ keys, const int *__restrict__ Ldev,
    const unsigned long long *__restrict__ clo, const unsigned long long *__restrict__ chi, int *__restrict__ bucket,
    int *__restrict__ slot, int *__restrict__ bcount) {
    __shared__ unsigned long long smp[kMaxSamples];
    const int L = *Ldev, stride = (L + kMaxSamples - 1) / kMaxSamples;
    const int ns = (L + stride - 1) / stride;
    for (int s = threadIdx.x; s < ns; s += blockDim.x) smp[s] = clo[(long long)s * stride];
    __syncthreads();
    const int lane = threadIdx.x & 31;
    for (long long base = (long long)blockIdx.x * blockDim.x; base < n; base += (long long)gridDim.x * blockDim.x) {
        const long long i = base + threadIdx.x;
        const bool act = i < n;
        const unsigned am = __ballot_sync(0xffffffffu, act);
        if (!act) continue;
        const unsigned long long k = spread3(quantize(x[i], lx, scale)) | (spread3(quantize(y[i], ly, scale)) << 1) |
                                     (spread3(quantize(z[i], lz, scale)) << 2);
        keys[i] = k;
        int a = 0, b = ns;                                    // first sample above k
        while (a < b) {
            const int mid = (a + b) >> 1;
            if (smp[mid] <= k) a = mid + 1;
            else b = mid;
        }
        int lo = a == 0 ? 0 : (a - 1) * stride + 1, hi = a == ns ? L : a * stride;
        while (lo < hi) {                                     // first leaf above k
            const int mid = (lo + hi) >> 1;
            if (clo[mid] <= k) lo = mid + 1;
            else hi = mid;
        }
        const int j = lo - 1;
        const int bk = j < 0 ? 0 : (k < chi[j] ? 2 * j + 1 : 2 * j + 2);
        bucket[i] = bk;
        const unsigned same = __match_any_sync(am, bk);
        const int leader = __ffs(same) - 1;
        int first = 0;
        if (lane == leader) first = atomicAdd(&bcount[bk], __popc(same));
        first = __shfl_sync(same, first, leader);
        slot[i] = first + __popc(same & ((1u << lane) - 1u));  // order inside a bucket: fixed by its sort
    }
}
__global__ void bucket_scatter_kernel(long long n, const unsigned long long *__restrict__ keys,
                                      const int *__restrict__ bucket, const int *__restrict__ slot,
                                      const int *__restrict__ boff, unsigned long long *__restrict__ bkeys,
                                      int *__restrict__ bidx) {
    const long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i >= n) return;
    const int pos = boff[bucket[i]] + slot[i];
    bkeys[pos] = keys[i];
    bidx[pos] = (int)i;
}
// one warp sorts one bucket of <= 32 R keys by (key, input index): a bitonic
// network on registers, element e = r * 32 + lane; partners 32 or more apart are
// in the same lane (register swap), nearer ones one shuffle away
__device__ __forceinline__ bool pair_gt(unsigned long long ka, int ia, unsigned long long kb, int ib) {
    return ka > kb || (ka == kb && ia > ib);
}
template <int R, int k, int j>
__device__ __forceinline__ void bitonic_stage(unsigned long long (&K)[R], int (&I)[R], int lane) {
    if constexpr (j >= 32) {                                  // same lane, registers r and r ^ (j / 32)
        constexpr int jr = j >> 5;
#pragma unroll
        for (int r = 0; r < R; ++r)
            if ((r & jr) == 0) {
                const int rp = r | jr;
                const bool up = ((r * 32 + lane) & k) == 0;
                const bool sw = pair_gt(K[r], I[r], K[rp], I[rp]) == up;
                const unsigned long long ka = K[r], kb = K[rp];
                const int ia = I[r], ib = I[rp];
                K[r] = sw ? kb : ka;
                K[rp] = sw ? ka : kb;
                I[r] = sw ? ib : ia;
                I[rp] = sw ? ia : ib;
            }
    } else {                                                  // lanes lane and lane ^ j
#pragma unroll
        for (int r = 0; r < R; ++r) {
            const unsigned long long ok = __shfl_xor_sync(0xffffffffu, K[r], j);
            const int oi = __shfl_xor_sync(0xffffffffu, I[r], j);
            const bool up = ((r * 32 + lane) & k) == 0;
            const bool keep_min = ((lane & j) == 0) == up;
            const bool take = pair_gt(K[r], I[r], ok, oi) == keep_min;
            K[r] = take ? ok : K[r];
            I[r] = take ? oi : I[r];
        }
    }
    if constexpr (j > 1) bitonic_stage<R, k, j / 2>(K, I, lane);
}
template <int R, int k>
__device__ __forceinline__ void bitonic_merge_all(unsigned long long (&K)[R], int (&I)[R], int lane) {
    bitonic_stage<R, k, k / 2>(K, I, lane);
    if constexpr (k < 32 * R) bitonic_merge_all<R, 2 * k>(K, I, lane);
}
template <int R>
__device__ __forceinline__ void warp_bitonic(int o, int cnt, const unsigned long long *__restrict__ bkeys,
                                             const int *__restrict__ bidx, unsigned long long *__restrict__ okeys,
                                             int *__restrict__ oidx, int lane) {
    unsigned long long K[R];
    int I[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const int e = r * 32 + lane;
        K[r] = e < cnt ? bkeys[o + e] : ~0ull;
        I[r] = e < cnt ? bidx[o + e] : 0x7fffffff;
    }
    bitonic_merge_all<R, 2>(K, I, lane);
#pragma unroll
    for (int r = 0; r < R; ++r) {
        const int e = r * 32 + lane;
        if (e < cnt) {
            okeys[o + e] = K[r];
            oidx[o + e] = I[r];
        }
    }
}
constexpr int kBucketWarps = 4;
__global__ void __launch_bounds__(32 * kBucketWarps) bucket_sort_kernel(const int *__restrict__ Ldev,
                                                                        const int *__restrict__ boff,
                                                                        const unsigned long long *__restrict__ bkeys,
                                                                        const int *__restrict__ bidx,
                                                                        unsigned long long *__restrict__ okeys,
                                                                        int *__restrict__ oidx,
                                                                        int *__restrict__ overflow,
                                                                        int *__restrict__ big,
                                                                        int *__restrict__ mid) {
    // buckets of <= 64 keys here (register-light: full occupancy), 65..512 keys listed
    // for bucket_mid_kernel, larger ones for bucket_big_kernel
    const int lane = threadIdx.x & 31;
    const int nb = 2 * *Ldev + 1;
    const int b = blockIdx.x * kBucketWarps + (threadIdx.x >> 5);
    if (b >= nb) return;                                      // whole warps
    const int o = boff[b], cnt = boff[b + 1] - o;
    if (cnt <= 1) {
        if (cnt == 1 && lane == 0) {
            okeys[o] = bkeys[o];
            oidx[o] = bidx[o];
        }
        return;
    }
    if (cnt > kBucketCap) {                                   // to the CTA sort; rarer still: a full sort
        if (lane == 0) {
            const int q = atomicAdd(big, 1);
            if (q < kBigList && cnt <= kBigCap) big[1 + q] = b;
            else atomicExch(overflow, 1);
        }
        return;
    }
    if (cnt <= 32) warp_bitonic<1>(o, cnt, bkeys, bidx, okeys, oidx, lane);
    else if (cnt <= 64) warp_bitonic<2>(o, cnt, bkeys, bidx, okeys, oidx, lane);
    else if (lane == 0) mid[1 + atomicAdd(mid, 1)] = b;       // the list holds every bucket if need be
}
// The listed buckets of 65..kBucketCap keys, a warp each (a fixed grid striding
// over the list, its length read on the device).
__global__ void __launch_bounds__(32 * kBucketWarps) bucket_mid_kernel(const int *__restrict__ mid,
                                                                       const int *__restrict__ boff,
                                                                       const unsigned long long *__restrict__ bkeys,
                                                                       const int *__restrict__ bidx,
                                                                       unsigned long long *__restrict__ okeys,
                                                                       int *__restrict__ oidx) {
    const int lane = threadIdx.x & 31, nmid = *mid;
    for (int q = blockIdx.x * kBucketWarps + (threadIdx.x >> 5); q < nmid; q += gridDim.x * kBucketWarps) {
        const int b = mid[1 + q], o = boff[b], cnt = boff[b + 1] - o;
        if (cnt <= 128) warp_bitonic<4>(o, cnt, bkeys, bidx, okeys, oidx, lane);
        else if (cnt <= 256) warp_bitonic<8>(o, cnt, bkeys, bidx, okeys, oidx, lane);
        else warp_bitonic<16>(o, cnt, bkeys, bidx, okeys, oidx, lane);
    }
}

// The listed buckets of kBucketCap < count <= kBigCap keys: one CTA per bucket, a
// bitonic network over (key, input index) in shared memory, padded to a power of
// two with keys above every 63-bit key.  A fixed grid that reads the list length
// on the device (graph-stable).
__global__ void __launch_bounds__(kBigThreads) bucket_big_kernel(const int *__restrict__ big,
                                                                 const int *__restrict__ boff,
                                                                 const unsigned long long *__restrict__ bkeys,
                                                                 const int *__restrict__ bidx,
                                                                 unsigned long long *__restrict__ okeys,
                                                                 int *__restrict__ oidx) {
    extern __shared__ unsigned long long sk[];
    int *si = reinterpret_cast<int *>(sk + kBigCap);
    const int nbig = min(big[0], kBigList);
    for (int q = blockIdx.x; q < nbig; q += gridDim.x) {
        const int b = big[1 + q], o = boff[b], cnt = boff[b + 1] - o;
        if (cnt > kBigCap) continue;                          // flagged: the caller sorts in full
        int P = 1;
        while (P < cnt) P <<= 1;
        for (int e = threadIdx.x; e < P; e += blockDim.x) {
            sk[e] = e < cnt ? bkeys[o + e] : ~0ull;
            si[e] = e < cnt ? bidx[o + e] : 0x7fffffff;
        }
        __syncthreads();
        for (int k = 2; k <= P; k <<= 1)
            for (int j = k >> 1; j > 0; j >>= 1) {
                for (int e = threadIdx.x; e < P; e += blockDim.x) {
                    const int pe = e ^ j;
                    if (pe > e) {
                        const bool up = (e & k) == 0;
                        const unsigned long long ka = sk[e], kb = sk[pe];
                        const int ia = si[e], ib = si[pe];
                        if (pair_gt(ka, ia, kb, ib) == up) {
                            sk[e] = kb;
                            sk[pe] = ka;
                            si[e] = ib;
                            si[pe] = ia;
                        }
                    }
                }
                __syncthreads();
            }
        for (int e = threadIdx.x; e < cnt; e += blockDim.x) {
            okeys[o + e] = sk[e];
            oidx[o + e] = si[e];
        }
        __syncthreads();
    }
}

// Internal nodes of the previous build, for Enforce_S: per level, node prefixes
// in ascending order ([base[l], base[l+1])) and their child counts.
struct PrevTree {
    const unsigned long long *prefix;
    const int *nchild;
    const long long *base;      // device, levels + 1 entries
    int levels;                 // 0: no previous tree (fresh build)
};

__device__ __forceinline__ bool prev_internal(const PrevTree &pv, int lev, unsigned long long prefix) {
    if (lev >= pv.levels) return false;
    long long lo = pv.base[lev], hi = pv.base[lev + 1];
    while (lo < hi) {
        const long long mid = lo + ((hi - lo) >> 1);
        if (pv.prefix[mid] < prefix) lo = mid + 1;
        else hi = mid;
    }
    return lo < pv.base[lev + 1] && pv.prefix[lo] == prefix && pv.nchild[lo] > 0;
}

// Per-node edits of FineGrainedOptimize (L20 SVI.B): per level, ascending
// prefixes with an action (1 = Collapse: stay a leaf, 2 = PushDown: split).
struct Edits {
    const unsigned long long *prefix;
    const int *action;
    const long long *base;      // device, kMaxLevel + 2 entries
    int n;                      // 0: none
};

__device__ __forceinline__ int edit_of(const Edits &ed, int lev, unsigned long long prefix) {
    long long lo = ed.base[lev], hi = ed.base[lev + 1];
    const long long end = hi;
    while (lo < hi) {
        const long long mid = lo + ((hi - lo) >> 1);
        if (ed.prefix[mid] < prefix) lo = mid + 1;
        else hi = mid;
    }
    return (lo < end && ed.prefix[lo] == prefix) ? ed.action[lo] : 0;
}

enum { kModeFresh = 0, kModeEnforce = 1, kModeKeep = 2 };

// For each node of the current level: split if > S bodies and level < 21
// (L10 SI.B).  Enforce_S (L20 SVI.A; pv.levels > 0) additionally keeps a node
// with exactly S bodies split when it was a parent before: Collapse applies only
// to parents with FEWER than S bodies, PushDown only to leaves with MORE than S.
// Child ranges by binary search on the octant digit inside [b, e): eight lanes
// per node, lane o finds the first position with digit >= o (independent
// searches, so a level costs one search's latency, not seven in a row).
// Does node id split (the rule above, edits applied)?  b, e, lev: its body range and level.
__device__ __forceinline__ bool node_splits(long long id, const Nodes &nd, int S, int mode, const PrevTree &pv,
                                            const Edits &ed, int &b, int &e, int &lev) {
    b = nd.b[id];
    e = nd.e[id];
    lev = nd.level[id];
    bool split;
    if (mode == kModeKeep)            // structure kept: split iff it was a parent (Collapse/PushDown edits below)
        split = pv.levels > 0 && prev_internal(pv, lev, nd.prefix[id]);
    else
        split = e - b > S || (mode == kModeEnforce && e - b == S && pv.levels > 0 && prev_internal(pv, lev, nd.prefix[id]));
    if (ed.n > 0) {
        const int a = edit_of(ed, lev, nd.prefix[id]);
        if (a == 1) split = false;
        else if (a == 2) split = true;
    }
    return split && lev < kMaxLevel;
}

// First position in [b, e) whose octant digit (key bits shift..shift+2) is >= o,
// searched by the W lanes of a group together (lane k of the group = kk): every
// round each lane reads one of W evenly spaced positions and a ballot (mask gmask,
// group bits at gshift) narrows the range W-fold -- log_W(e - b) rounds of one
// load instead of log_2 dependent loads.  All 32 lanes of the warp call it.
__device__ __forceinline__ int kary_bound(const unsigned long long *__restrict__ keys, int b, int e, int o, int shift,
                                          int W, int kk, int gshift, bool live) {
    int lo = b, hi = e;                                       // the answer lies in [lo, hi]
    while (__any_sync(0xffffffffu, live && hi > lo)) {
        const bool act = live && hi > lo;
        const int span = hi - lo;
        const int pk = lo + (int)(((long long)kk * span) / W);
        const bool ge = act && (int)((keys[pk] >> shift) & 7ull) >= o;
        const unsigned bal = (__ballot_sync(0xffffffffu, ge) >> gshift) & (W == 32 ? 0xffffffffu : ((1u << W) - 1u));
        if (act) {
            const int kf = bal ? __ffs(bal) - 1 : W;          // first sample with digit >= o
            if (kf == 0) {
                hi = lo;                                       // p_0 = lo qualifies
            } else {
                const int pprev = lo + (int)(((long long)(kf - 1) * span) / W);
                if (kf < W) hi = lo + (int)(((long long)kf * span) / W);
                lo = pprev + 1;
            }
        }
    }
    return lo;
}

// one lane of the 8 of node i = gt >> 3 (lane o = gt & 7); all 32 lanes of the
// warp call it together (shuffles / ballot), with gt >= 8m for padding lanes
__device__ __forceinline__ void split_count_lane(long long gt, int m, long long base, const Nodes &nd,
                                                 const unsigned long long *__restrict__ keys, int S, int mode,
                                                 const PrevTree &pv, const Edits &ed, int *__restrict__ cb,
                                                 int *__restrict__ nc) {
    const int o = (int)(gt & 7);
    const int i = (int)(gt >> 3);
    const bool live = i < m;
    int b = 0, e = 0, lev = 0;
    bool split = false;
    if (live) {
        const long long id = base + i;
        b = nd.b[id];
        e = nd.e[id];
        lev = nd.level[id];
        if (mode == kModeKeep)        // structure kept: split iff it was a parent (Collapse/PushDown edits below)
            split = pv.levels > 0 && prev_internal(pv, lev, nd.prefix[id]);
        else
            split = e - b > S || (mode == kModeEnforce && e - b == S && pv.levels > 0 &&
                                  prev_internal(pv, lev, nd.prefix[id]));
        if (ed.n > 0) {
            const int a = edit_of(ed, lev, nd.prefix[id]);
            if (a == 1) split = false;
            else if (a == 2) split = true;
        }
        split = split && lev < kMaxLevel;
    }
    int bound = b;                                   // lane o: first position in [b, e) with digit >= o
    if (split && o > 0) {
        const int shift = 3 * (kMaxLevel - 1 - lev);
        int lo = b, hi = e;
        while (lo < hi) {
            const int mid = lo + ((hi - lo) >> 1);
            if ((int)((keys[mid] >> shift) & 7ull) < o) lo = mid + 1;
            else hi = mid;
        }
        bound = lo;
    }
    // next boundary (lane o+1's, or e for o = 7) -> is child o non-empty?
    int nxt = __shfl_down_sync(0xffffffffu, bound, 1, 8);
    if (o == 7) nxt = e;
    const unsigned nonempty = __ballot_sync(0xffffffffu, split && nxt > bound);
    if (!live) return;
    if (split) {
        cb[(size_t)i * 9 + o] = bound;
        if (o == 7) cb[(size_t)i * 9 + 8] = e;
    }
    if (o == 0) nc[i] = __popc((nonempty >> (threadIdx.x & 24)) & 0xffu);
}

__global__ void split_count_kernel(int m, int base, Nodes nd, const unsigned long long *__restrict__ keys,
                                   int S, int mode, PrevTree pv, Edits ed, int *__restrict__ cb,
                                   int *__restrict__ nc) {
    split_count_lane((long long)blockIdx.x * blockDim.x + threadIdx.x, m, base, nd, keys, S, mode, pv, ed, cb, nc);
}

__device__ __forceinline__ void split_write_node(int i, long long base, long long next_base, const Nodes &nd,
                                                 const int *__restrict__ cb, int cnt, int off) {
    const long long id = base + i;
    nd.nchild[id] = cnt;
    nd.first_child[id] = cnt ? (int)(next_base + off) : -1;
    if (!cnt) return;
    long long w = next_base + off;
    const unsigned long long pre = nd.prefix[id];
    const int lev = nd.level[id];
    for (int o = 0; o < 8; ++o) {
        const int b = cb[(size_t)i * 9 + o], e = cb[(size_t)i * 9 + o + 1];
        if (e > b) {
            nd.b[w] = b;
            nd.e[w] = e;
            nd.level[w] = lev + 1;
            nd.prefix[w] = (pre << 3) | (unsigned long long)o;
            nd.first_child[w] = -1;
            nd.nchild[w] = 0;
            ++w;
        }
    }
}

__global__ void split_write_kernel(int m, int base, int next_base, Nodes nd, const int *__restrict__ cb,
                                   const int *__restrict__ nc, const int *__restrict__ off) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= m) return;
    split_write_node(i, base, next_base, nd, cb, nc[i], off[i]);
}

// The whole level loop in ONE cooperative launch (no host round trip per level),
// ONE grid barrier per level: block b owns the tile [t0, t1) of the level's nodes;
// it (1) computes their split counts (8 lanes per node), (2) scans its tile's child
// counts, (3) publishes its tile's total in a status word tagged with the launch
// epoch and the level (so nothing is reset between levels or builds) and sums the
// totals of all earlier tiles in ONE parallel round (thread k waits for tile k's
// word; a block reduction -- the grid has <= 256 blocks), (4) writes its nodes'
// children, then the grid barrier; the level's total is written by the last tile.
// (A chained decoupled look-back walked the predecessors one L2 round trip at a
// time: the kernel issued on 2 % of its cycles, ncu.)
// Level starts go to ctl->base[]; a level that would exceed the node capacity sets
// ctl->overflow (each block checks its own writes) and every block stops after the
// barrier (the host grows the arrays and reruns).  (Round 1 had three barriers per
// level: counts, tile sums, writes.)
struct LevelCtl {
    long long base[kMaxLevel + 3];  // level starts, base[levels] = total nodes
    int count[kMaxLevel + 3];       // nodes of level l + 1 (the last tile's inclusive prefix of level l): a
                                    // slot per level, so no block reads a word the next level overwrites
    int levels;
    int overflow;
    unsigned bar_count, bar_gen;
    int sort_overflow;              // the bucket sort's flag, copied in before the launch (not the kernel's)
};

__device__ __forceinline__ void grid_barrier(LevelCtl *c) {
    __syncthreads();
    if (threadIdx.x == 0) {
        volatile unsigned *gen = &c->bar_gen;
        const unsigned g = *gen;
        __threadfence();
        if (atomicAdd(&c->bar_count, 1u) == gridDim.x - 1) {
            c->bar_count = 0;
            __threadfence();
            atomicAdd(&c->bar_gen, 1u);
        } else {
            while (*gen == g) __nanosleep(32);
        }
        __threadfence();
    }
    __syncthreads();
}

// status word of a tile: high 32 bits = epoch << 8 | level << 2 | flag (1 = aggregate,
// 2 = inclusive prefix), low 32 bits = the value
__device__ __forceinline__ unsigned long long tile_status(unsigned epoch, int lev, unsigned flag, unsigned v) {
    return ((unsigned long long)((epoch << 8) | ((unsigned)lev << 2) | flag) << 32) | v;
}

constexpr int kLvlThreads = 256;
__global__ void __launch_bounds__(kLvlThreads) levels_kernel(Nodes nd, const unsigned long long *__restrict__ keys,
                                                             int S, int mode, PrevTree pv, Edits ed,
                                                             int *__restrict__ cb, int *__restrict__ nc,
                                                             int *__restrict__ off,
                                                             unsigned long long *__restrict__ tstat, unsigned epoch,
                                                             LevelCtl *ctl, long long cap) {
    __shared__ int wsum[kLvlThreads / 32];
    __shared__ int carry, s_excl;
    __shared__ int sbound[9];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int G = (int)gridDim.x, bid = (int)blockIdx.x;
    long long base = 0;
    int m = 1;
    int lev = 0;
    if (bid == 0 && threadIdx.x == 0) {
        ctl->base[0] = 0;
        ctl->overflow = 0;
    }
    while (m > 0) {
        const int tile = (m + G - 1) / G;
        const int t0 = min(bid * tile, m), t1 = min(t0 + tile, m);
        // (1) split counts of the tile's nodes.  The few huge nodes of the top levels
        //     are every level's critical path (all blocks wait for them), so small
        //     tiles search wide: one node -> the whole block (warp o-1 finds octant
        //     boundary o, 33-ary), up to 8 nodes -> a warp per node (4 lanes per
        //     boundary, 5-ary); else 8 lanes per node (binary, split_count_lane).
        const int ntile = t1 - t0;
        if (ntile <= 1) {
            int b = 0, e = 0, nlev = 0;
            const bool split = ntile == 1 && node_splits(base + t0, nd, S, mode, pv, ed, b, e, nlev);
            const int shift = 3 * (kMaxLevel - 1 - nlev);
            if (wid < 7) {
                const int bound = kary_bound(keys, b, e, wid + 1, shift, 32, lane, 0, split);
                if (lane == 0) sbound[wid + 1] = bound;
            }
            __syncthreads();
            if (threadIdx.x == 0 && ntile == 1) {
                int cnt = 0;
                if (split) {
                    sbound[0] = b;
                    sbound[8] = e;
                    for (int o = 0; o < 8; ++o) {
                        cb[(size_t)t0 * 9 + o] = sbound[o];
                        cnt += sbound[o + 1] > sbound[o];
                    }
                    cb[(size_t)t0 * 9 + 8] = e;
                }
                nc[t0] = cnt;
            }
        } else if (ntile <= kLvlThreads / 32) {
            const int i = t0 + wid;
            int b = 0, e = 0, nlev = 0;
            const bool split = wid < ntile && node_splits(base + i, nd, S, mode, pv, ed, b, e, nlev);
            const int shift = 3 * (kMaxLevel - 1 - nlev);
            const int o = lane / 4 + 1, kk = lane & 3;
            const int bound = kary_bound(keys, b, e, o, shift, 4, kk, 4 * (o - 1) & 31, split && lane < 28);
            int bo[9];
            bo[0] = b;
            bo[8] = e;
#pragma unroll
            for (int oo = 1; oo < 8; ++oo) bo[oo] = __shfl_sync(0xffffffffu, bound, 4 * (oo - 1));
            if (lane == 0 && wid < ntile) {
                int cnt = 0;
                if (split) {
#pragma unroll
                    for (int oo = 0; oo < 9; ++oo) cb[(size_t)i * 9 + oo] = bo[oo];
#pragma unroll
                    for (int oo = 0; oo < 8; ++oo) cnt += bo[oo + 1] > bo[oo];
                }
                nc[i] = cnt;
            }
        } else {
            for (int w0 = threadIdx.x & ~31; 8 * t0 + w0 < 8 * t1; w0 += kLvlThreads)
                split_count_lane(8LL * t0 + w0 + lane, t1, base, nd, keys, S, mode, pv, ed, cb, nc);
        }
        __syncthreads();
        // (2) tile scan of the child counts -> off[i] (exclusive, tile-local), carry = tile sum
        if (threadIdx.x == 0) carry = 0;
        __syncthreads();
        for (int c0 = t0; c0 < t1; c0 += kLvlThreads) {
            const int i = c0 + threadIdx.x;
            const int v = i < t1 ? nc[i] : 0;
            int inc = v;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int u = __shfl_up_sync(0xffffffffu, inc, o);
                if (lane >= o) inc += u;
            }
            if (lane == 31) wsum[wid] = inc;
            __syncthreads();
            int wpre = 0;
            for (int k = 0; k < wid; ++k) wpre += wsum[k];
            int ctot = 0;
            for (int k = 0; k < kLvlThreads / 32; ++k) ctot += wsum[k];
            if (i < t1) off[i] = carry + wpre + inc - v;
            __syncthreads();
            if (threadIdx.x == 0) carry += ctot;
            __syncthreads();
        }
        // (3) publish this tile's total; sum the earlier tiles' totals in one parallel round
        if (threadIdx.x == 0) atomicExch(&tstat[bid], tile_status(epoch, lev, 1u, (unsigned)carry));
        unsigned part = 0;
        for (int k = threadIdx.x; k < bid; k += kLvlThreads) {
            unsigned long long sw;
            for (;;) {
                sw = *(volatile unsigned long long *)&tstat[k];
                if ((unsigned)(sw >> 34) == ((epoch << 6) | (unsigned)lev)) break;     // this level's word
                __nanosleep(20);
            }
            part += (unsigned)sw;
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) part += __shfl_xor_sync(0xffffffffu, part, o);
        __syncthreads();                                          // wsum reuse after the tile scan
        if (lane == 0) wsum[wid] = (int)part;
        __syncthreads();
        if (threadIdx.x == 0) {
            int e = 0;
            for (int k = 0; k < kLvlThreads / 32; ++k) e += wsum[k];
            s_excl = e;
            if (bid == G - 1) ctl->count[lev] = e + carry;       // read by every block after the barrier
        }
        __syncthreads();
        const int excl = s_excl;
        const long long next_base = base + m;
        // (4) children of the tile's nodes (the block's own writes checked against the capacity)
        if (next_base + excl + carry > cap) {
            if (threadIdx.x == 0) ctl->overflow = 1;
        } else {
            for (int i = t0 + threadIdx.x; i < t1; i += kLvlThreads)
                split_write_node(i, base, next_base, nd, cb, nc[i], excl + off[i]);
        }
        grid_barrier(ctl);
        if (*(volatile int *)&ctl->overflow) return;
        const int total = *(volatile int *)&ctl->count[lev];
        ++lev;
        if (bid == 0 && threadIdx.x == 0) {
            ctl->base[lev] = next_base;
            ctl->levels = lev;
        }
        base = next_base;
        m = total;
    }
}

// ---- Direct construction from the sorted keys (fresh builds and Enforce_S
// without edits; the level loop above stays for KEEP / FineGrainedOptimize edits).
// The split rule of R7 / R22 restated on the sorted keys: the node at level l that
// holds body i has MORE than S bodies iff some window of S + 1 consecutive sorted
// keys containing i shares its first l octal digits (such a window lies inside the
// node; conversely a node of >= S + 1 bodies holds such a window around i).  With
// w_j = lcp(key_j, key_{j+S}) in digits and M_i = max w_j over the windows that
// contain i, body i's leaf is at level min(M_i + 1, 21) (M_i = -1: the root); Enforce_S
// then descends further while the node holds exactly S bodies (M'_i, windows of S)
// and was a parent before.  Leaves start where lcp(key_{i-1}, key_i) < that level.
// The internal nodes are the leaves' ancestors: the level-l ancestor of leaf j
// starts at leaf j iff lcp with the previous leaf's first key < l, so every node is
// (leaf j, level l) with lo_j <= l <= level_j; its rank inside its level is a prefix
// count over the leaves, its children are the level l+1 nodes starting at leaves
// [j, j_end).  Output: the same level-major Nodes arrays as levels_kernel, plus
// the leaf arrays (bit-identical; tests compare both paths).
__device__ __forceinline__ int lcp_digits(unsigned long long a, unsigned long long b) {
    return a == b ? kMaxLevel : (__clzll((long long)(a ^ b)) - 1) / 3;
}
#ifndef AFMM_DIR_TILE
#define AFMM_DIR_TILE 1024
#endif
constexpr int kDirTile = AFMM_DIR_TILE;     // positions per block of leaf_level_kernel
constexpr int kDirThreads = 256;
constexpr int kDirMaxS = 2048;              // larger S: the level loop
constexpr int kDirLevels = kMaxLevel + 1;   // levels 0..21
struct DirCtl {
    long long base[kDirLevels + 1];         // level starts; base[levels] = nodes
    long long nn;
    long long nnz;                          // U-list entries (u_off[L])
    int levels;
    int L;
    int sort_overflow;                      // the bucket sort's flag, copied in before the readback
    int cap_overflow;                       // nodes > node capacity or leaves > leaf capacity: nothing written
    int ulist_overflow;                     // a warp-descent row / frontier overflowed: per-thread DFS fallback
    int nnz_overflow;                       // U-list entries > their capacity: u_idx not written
};
__device__ __forceinline__ bool dir_bad(const DirCtl *c) {
    return c->sort_overflow | c->cap_overflow | c->ulist_overflow | c->nnz_overflow;
}

// Range maxima over the window arrays: per 32-position block a prefix and a suffix
// maximum (warp scans) and a sparse table over the block maxima, so a window is
// max(suffix of its first block, prefix of its last, table lookup of the full
// blocks between) -- 2 warp scans per array instead of log2(S) doubling passes.
constexpr int kDirLen = kDirTile + kDirMaxS, kDirNB = kDirLen / 32, kDirST = 7;   // 2^6 = 64 < 96 blocks
static_assert(kDirLen % 32 == 0 && (1 << (kDirST - 1)) * 2 > kDirNB, "window table sizes");
__device__ __forceinline__ int dir_rmq(const signed char *X, const signed char *P, const signed char *Q,
                                       const signed char (*ST)[kDirNB], int lo, int hi) {
    const int bl = lo >> 5, bh = hi >> 5;
    if (bl == bh) {
        int m = -1;
        for (int a = lo; a <= hi; ++a) m = max(m, (int)X[a]);
        return m;
    }
    int m = max((int)Q[lo], (int)P[hi]);
    const int nbt = bh - bl - 1;
    if (nbt > 0) {
        const int k = 31 - __clz(nbt);
        m = max(m, max((int)ST[k][bl + 1], (int)ST[k][bh - (1 << k)]));
    }
    return m;
}

__global__ void __launch_bounds__(kDirThreads) leaf_level_kernel(long long n, const unsigned long long *__restrict__ keys,
                                                                 int S, int mode, PrevTree pv,
                                                                 const int *__restrict__ pv_levels, Edits ed,
                                                                 const int *__restrict__ hint_bucket,
                                                                 const int *__restrict__ hint_perm,
                                                                 const int *__restrict__ hint_ll,
                                                                 unsigned char *__restrict__ lvl, int *__restrict__ flag) {
    if (pv_levels) pv.levels = mode != kModeFresh ? *pv_levels : 0;    // the previous build's (device word)
    // array 0 = windows of S + 1 (w), 1 = windows of S (v, Enforce_S only); position a <->
    // window start j = t0 - S + a; -1 = no such window.  KEEP needs no counts: no windows.
    __shared__ signed char X[2][kDirLen], P[2][kDirLen], Q[2][kDirLen];
    __shared__ signed char ST[2][kDirST][kDirNB];
    const bool keep = mode == kModeKeep;
    const bool enf = mode == kModeEnforce && pv.levels > 0;
    const int na = keep ? 0 : enf ? 2 : 1;
    const long long t0 = (long long)blockIdx.x * kDirTile;
    const int len = keep ? 0 : kDirTile + S, nb = (len + 31) >> 5;
    for (int a = threadIdx.x; a < nb * 32; a += blockDim.x) {
        const long long j = t0 - S + a;
        signed char w = -1, v = -1;
        if (a < len && j >= 0) {
            const unsigned long long kj = j < n ? keys[j] : 0ull;
            if (j + S < n) w = (signed char)lcp_digits(kj, keys[j + S]);
            if (enf && j + S - 1 < n) v = (signed char)lcp_digits(kj, keys[j + S - 1]);
        }
        X[0][a] = w;
        X[1][a] = v;
    }
    __syncthreads();
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    for (int bk = wid; bk < nb; bk += kDirThreads / 32)
        for (int ar = 0; ar < na; ++ar) {
            const int x = X[ar][32 * bk + lane];
            int pre = x, suf = x;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int u = __shfl_up_sync(0xffffffffu, pre, o), d = __shfl_down_sync(0xffffffffu, suf, o);
                if (lane >= o) pre = max(pre, u);
                if (lane + o < 32) suf = max(suf, d);
            }
            P[ar][32 * bk + lane] = (signed char)pre;
            Q[ar][32 * bk + lane] = (signed char)suf;
            if (lane == 31) ST[ar][0][bk] = (signed char)pre;
        }
    const int kmax = 31 - __clz(max(1, (S >> 5) + 2));          // full blocks inside a window: < S / 32 + 2
    for (int k = 1; k <= kmax && k < kDirST; ++k) {
        __syncthreads();
        for (int t = threadIdx.x; t < na * nb; t += blockDim.x) {
            const int ar = t / nb, bk = t - ar * nb, o = 1 << (k - 1);
            const signed char x = ST[ar][k - 1][bk], y = bk + o < nb ? ST[ar][k - 1][bk + o] : (signed char)-1;
            ST[ar][k][bk] = x > y ? x : y;
        }
    }
    __syncthreads();
    for (int a0 = threadIdx.x; a0 < kDirTile; a0 += blockDim.x) {
        const long long i = t0 + a0;
        if (i >= n) break;
        // windows of S + 1 containing i: j in [i - S, i] -> a in [a0, a0 + S]
        const unsigned long long ki = keys[i];
        int l;
        if (keep && hint_bucket && (hint_bucket[hint_perm[i]] & 1)) {
            // KEEP, body still inside previous leaf j's cell (bucket 2j + 1 of the sort):
            // its path's nodes above that leaf were parents, the leaf was not
            l = hint_ll[hint_bucket[hint_perm[i]] >> 1];
        } else if (keep) {
            // KEEP: the node on i's path at level l splits iff it was a parent before -- true
            // down to some level and false below (a parent's parent is a parent): bisect for
            // the first level that was not
            int lo = 0, hi = min(pv.levels, kMaxLevel);
            while (lo < hi) {
                const int mid = (lo + hi) >> 1;
                if (prev_internal(pv, mid, ki >> (3 * (kMaxLevel - mid)))) lo = mid + 1;
                else hi = mid;
            }
            l = lo;
        } else {
            const int m1 = dir_rmq(X[0], P[0], Q[0], ST[0], a0, a0 + S);
            l = m1 < 0 ? 0 : min(m1 + 1, kMaxLevel);
            if (enf && l < kMaxLevel) {
                // windows of S containing i: j in [i - S + 1, i] -> a in [a0 + 1, a0 + S]
                const int m2 = dir_rmq(X[1], P[1], Q[1], ST[1], a0 + 1, a0 + S);
                while (l < kMaxLevel && l <= m2 && prev_internal(pv, l, ki >> (3 * (kMaxLevel - l)))) ++l;
            }
        }
        if (ed.n > 0) {
            // FineGrainedOptimize's edits on top (node_splits' override): above the rule's
            // leaf level l0 a Collapse stops the path, from l0 on a PushDown continues it
            const int l0 = l;
            for (l = 0; l < kMaxLevel; ++l) {
                const int a = edit_of(ed, l, ki >> (3 * (kMaxLevel - l)));
                if (a == 1 || (l >= l0 && a != 2)) break;
            }
        }
        lvl[i] = (unsigned char)l;
        flag[i] = (i == 0 || lcp_digits(keys[i - 1], ki) < l) ? 1 : 0;
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) flag[n] = 0;
}

// Leaf j (first body i): start, level, prefix, first key, and lo_j = the first level
// whose node starts at this leaf (lcp with the previous body + 1; 0 for leaf 0).
__global__ void leaf_info_kernel(long long n, const unsigned long long *__restrict__ keys,
                                 const unsigned char *__restrict__ lvl, const int *__restrict__ flag,
                                 const int *__restrict__ leaf_at, int *__restrict__ ls, int *__restrict__ ll,
                                 unsigned long long *__restrict__ lp, unsigned long long *__restrict__ fk,
                                 unsigned char *__restrict__ llo) {
    const long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i >= n || !flag[i]) return;
    const int id = leaf_at[i], l = lvl[i];
    const unsigned long long k = keys[i];
    ls[id] = (int)i;
    ll[id] = l;
    lp[id] = k >> (3 * (kMaxLevel - l));
    fk[id] = k;
    llo[id] = (unsigned char)(i == 0 ? 0 : lcp_digits(keys[i - 1], k) + 1);
}

// Per block of 256 leaves: how many nodes of each level start at its leaves (and
// the leaf counts).  Grid over an upper bound of L; L = leaf_at[n] on the device.
constexpr int kDirLeafBlock = 256;
__global__ void __launch_bounds__(kDirLeafBlock) node_count_kernel(long long n, const int *__restrict__ leaf_at,
                                                                   const int *__restrict__ ls,
                                                                   const int *__restrict__ ll,
                                                                   const unsigned char *__restrict__ llo,
                                                                   int *__restrict__ lc, int *__restrict__ chunk_cnt) {
    __shared__ int cnt[kDirLevels];
    const int L = leaf_at[n];
    if ((long long)blockIdx.x * kDirLeafBlock >= L) return;
    if (threadIdx.x < kDirLevels) cnt[threadIdx.x] = 0;
    __syncthreads();
    const int j = blockIdx.x * kDirLeafBlock + threadIdx.x;
    int lo = 1, hi = 0;
    if (j < L) {
        lo = llo[j];
        hi = ll[j];
        lc[j] = (j + 1 < L ? ls[j + 1] : (int)n) - ls[j];
    }
    for (int l = 0; l < kDirLevels; ++l) {
        const unsigned m = __ballot_sync(0xffffffffu, lo <= l && l <= hi);
        if ((threadIdx.x & 31) == 0 && m) atomicAdd(&cnt[l], __popc(m));
    }
    __syncthreads();
    if (threadIdx.x < kDirLevels) chunk_cnt[(size_t)blockIdx.x * kDirLevels + threadIdx.x] = cnt[threadIdx.x];
}

// One block, a warp per level: exclusive scan of the chunk counts over the chunks
// (chunk_base), level totals -> level starts, node total, levels; L.
__global__ void __launch_bounds__(32 * kDirLevels) node_scan_kernel(long long n, const int *__restrict__ leaf_at,
                                                                    const int *__restrict__ chunk_cnt,
                                                                    int *__restrict__ chunk_base,
                                                                    int *__restrict__ level_cnt, DirCtl *ctl) {
    __shared__ long long tot[kDirLevels];
    const int L = leaf_at[n];
    const int nchunk = (L + kDirLeafBlock - 1) / kDirLeafBlock;
    const int l = threadIdx.x >> 5, lane = threadIdx.x & 31;
    int carry = 0;
    for (int c0 = 0; c0 < nchunk; c0 += 32) {
        const int c = c0 + lane;
        const int v = c < nchunk ? chunk_cnt[(size_t)c * kDirLevels + l] : 0;
        int inc = v;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int u = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= o) inc += u;
        }
        if (c < nchunk) chunk_base[(size_t)c * kDirLevels + l] = carry + inc - v;
        carry += __shfl_sync(0xffffffffu, inc, 31);
    }
    if (lane == 0) {
        tot[l] = carry;
        level_cnt[l] = carry;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        long long b = 0;
        int levels = 0;
        for (int k = 0; k < kDirLevels; ++k) {
            ctl->base[k] = b;
            b += tot[k];
            if (tot[k] > 0) levels = k + 1;
        }
        ctl->base[kDirLevels] = b;
        ctl->nn = b;
        ctl->levels = levels;
        ctl->L = L;
    }
}

// Per leaf: its rank among the nodes of every level (rank[l][j] = nodes of level l
// starting at leaves < j; row length L + 1, rank[l][L] = the level's node count) and
// the nodes that start at it: b, level, prefix; for the leaf itself also e, no
// children, and the leaf <-> node maps.
__global__ void __launch_bounds__(kDirLeafBlock) node_rank_kernel(DirCtl *__restrict__ ctl,
                                                                  const int *__restrict__ chunk_base,
                                                                  const int *__restrict__ level_cnt,
                                                                  const int *__restrict__ ls,
                                                                  const int *__restrict__ lc,
                                                                  const int *__restrict__ ll,
                                                                  const unsigned char *__restrict__ llo,
                                                                  const unsigned long long *__restrict__ fk,
                                                                  int *__restrict__ rank, Nodes nd,
                                                                  int *__restrict__ node_leaf,
                                                                  int *__restrict__ leaf_node,
                                                                  long long node_cap, int leaf_cap) {
    __shared__ int wcnt[kDirLeafBlock / 32][kDirLevels];
    const int L = ctl->L;
    if (ctl->nn > node_cap || L > leaf_cap) {                  // every block returns; the host grows and reruns
        if (blockIdx.x == 0 && threadIdx.x == 0) ctl->cap_overflow = 1;
        return;
    }
    if ((long long)blockIdx.x * kDirLeafBlock >= L) return;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const int j = blockIdx.x * kDirLeafBlock + threadIdx.x;
    int lo = 1, hi = 0;
    if (j < L) {
        lo = llo[j];
        hi = ll[j];
    }
    unsigned below[kDirLevels];
#pragma unroll
    for (int l = 0; l < kDirLevels; ++l) {
        const unsigned m = __ballot_sync(0xffffffffu, lo <= l && l <= hi);
        below[l] = __popc(m & ((1u << lane) - 1u));
        if (lane == 0) wcnt[wid][l] = __popc(m);
    }
    __syncthreads();
    if (j < L) {
        const size_t row = (size_t)L + 1;
        const int bj = ls[j];
        const unsigned long long k = fk[j];
        int r[kDirLevels];
#pragma unroll
        for (int l = 0; l < kDirLevels; ++l) {
            r[l] = chunk_base[(size_t)blockIdx.x * kDirLevels + l] + (int)below[l];
            for (int w = 0; w < wid; ++w) r[l] += wcnt[w][l];
            rank[l * row + j] = r[l];
        }
#pragma unroll
        for (int l = 0; l < kDirLevels; ++l) {
            if (lo <= l && l <= hi) {
                const long long id = ctl->base[l] + r[l];
                nd.b[id] = bj;
                nd.level[id] = l;
                nd.prefix[id] = k >> (3 * (kMaxLevel - l));
                if (l == hi) {
                    nd.e[id] = bj + lc[j];
                    nd.nchild[id] = 0;
                    nd.first_child[id] = -1;
                    node_leaf[id] = j;
                    leaf_node[j] = (int)id;
                } else {                          // internal: its first child starts at this leaf too
                    nd.first_child[id] = (int)(ctl->base[l + 1] + r[l < kDirLevels - 1 ? l + 1 : l]);
                    node_leaf[id] = -1;
                }
            }
        }
        if (j == L - 1) {
#pragma unroll
            for (int l = 0; l < kDirLevels; ++l) rank[l * row + L] = level_cnt[l];
        }
    }
}

// Internal nodes, from the side where they end: the level-l ancestors of leaf
// j' - 1 that do not hold leaf j' (llo[j'] <= l < level of leaf j' - 1; every level
// for j' = L) end at leaf j': e = its first body (n), and the children are the level
// l + 1 nodes up to there (first_child was written by node_rank_kernel).  O(1) per node.
__global__ void node_links_kernel(long long n, const DirCtl *__restrict__ ctl, const int *__restrict__ ls,
                                  const int *__restrict__ ll, const unsigned char *__restrict__ llo,
                                  const int *__restrict__ rank, Nodes nd, long long node_cap, int leaf_cap) {
    if (ctl->nn > node_cap || ctl->L > leaf_cap) return;
    const int L = ctl->L;
    for (int j = blockIdx.x * blockDim.x + threadIdx.x + 1; j <= L; j += gridDim.x * blockDim.x) {   // j' in [1, L]
    const int lo = j < L ? llo[j] : 0, hi = ll[j - 1];
    const size_t row = (size_t)L + 1;
    const int e = j < L ? ls[j] : (int)n;
    for (int l = lo; l < hi; ++l) {
        const long long id = ctl->base[l] + rank[l * row + j] - 1;
        nd.e[id] = e;
        nd.nchild[id] = (int)(ctl->base[l + 1] + rank[(l + 1) * row + j] - nd.first_child[id]);
    }
    }
}

// The direct build's tail, after the U-lists: unless something overflowed, keep
// the node arrays as the next Enforce_S's previous tree (prefix, nchild, level
// starts) and the U-list total -- on the device, no host round trip.
__global__ void dir_finish_kernel(DirCtl *ctl, Nodes nd, const long long *__restrict__ u_off,
                                  unsigned long long *__restrict__ pv_prefix, int *__restrict__ pv_nchild,
                                  long long *__restrict__ pv_base, int *__restrict__ dstate) {
    if (dir_bad(ctl)) return;                     // (a failed attempt leaves the previous tree for the rerun)
    const long long nn = ctl->nn;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < nn; i += (long long)gridDim.x * blockDim.x) {
        pv_prefix[i] = nd.prefix[i];
        pv_nchild[i] = nd.nchild[i];
    }
    if (blockIdx.x == 0 && threadIdx.x <= kDirLevels) {
        const int l = threadIdx.x;
        if (l <= ctl->levels) pv_base[l] = l < ctl->levels ? ctl->base[l] : nn;
        if (l == 0) {
            ctl->nnz = u_off[ctl->L];
            dstate[0] = ctl->L;                   // read by the next build's bucket sort / Enforce_S
            dstate[1] = ctl->levels;
        }
    }
}

__global__ void leaf_flag_kernel(int nn, Nodes nd, int *__restrict__ flag) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= nn) return;
    if (nd.nchild[i] == 0) flag[nd.b[i]] = 1;
}

__global__ void leaf_write_kernel(int nn, Nodes nd, const int *__restrict__ leaf_at,
                                  int *__restrict__ node_leaf, int *__restrict__ ls,
                                  int *__restrict__ lc, int *__restrict__ ll,
                                  unsigned long long *__restrict__ lp) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= nn) return;
    if (nd.nchild[i] != 0) {
        node_leaf[i] = -1;
        return;
    }
    const int id = leaf_at[nd.b[i]];
    node_leaf[i] = id;
    ls[id] = nd.b[i];
    lc[id] = nd.e[i] - nd.b[i];
    ll[id] = nd.level[i];
    lp[id] = nd.prefix[i];
}

__device__ __forceinline__ void box_of(int level, unsigned long long prefix, long long A[3], long long &w) {
    const int sh = kMaxLevel - level;
    A[0] = (long long)compact3(prefix) << sh;
    A[1] = (long long)compact3(prefix >> 1) << sh;
    A[2] = (long long)compact3(prefix >> 2) << sh;
    w = 1LL << sh;
}

// Per-leaf descent: count (out == nullptr) or fill the U-list row.
__global__ void ulist_kernel(int L, Nodes nd, const int *__restrict__ node_leaf,
                             const int *__restrict__ leaf_node, const long long *__restrict__ u_off,
                             int *__restrict__ u_idx, long long *__restrict__ counts) {
    const int t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= L) return;
    const int tn = leaf_node[t];
    long long At[3], wt;
    box_of(nd.level[tn], nd.prefix[tn], At, wt);
    int stack[8 * (kMaxLevel + 2)];
    int sp = 0;
    stack[sp++] = 0;
    long long cnt = 0;
    long long w0 = u_idx ? u_off[t] : 0;
    while (sp > 0) {
        const int ni = stack[--sp];
        long long As[3], ws;
        box_of(nd.level[ni], nd.prefix[ni], As, ws);
        bool touch = true;
#pragma unroll
        for (int a = 0; a < 3; ++a) touch &= (At[a] <= As[a] + ws) && (As[a] <= At[a] + wt);
        if (!touch) continue;
        const int nc = nd.nchild[ni];
        if (nc == 0) {
            if (u_idx) u_idx[w0 + cnt] = node_leaf[ni];
            ++cnt;
        } else {
            const int fc = nd.first_child[ni];
            for (int c = nc - 1; c >= 0; --c) stack[sp++] = fc + c;
        }
    }
    if (counts) counts[t] = cnt;
}

// U-lists by a warp-cooperative level-order descent (one warp per target leaf):
// the frontier of nodes whose closed box touches the leaf's box is expanded 32
// nodes at a time, touching leaves are collected, and the row is put in
// ascending leaf order (= the per-thread DFS order above) by a rank sort.  Rows
// go to a fixed-capacity scratch row (kURow); counts[t] = row length.  A leaf
// whose frontier or row exceeds the capacity raises *overflow and the caller
// falls back to ulist_kernel for the whole tree (same result).
// Every node's box anchor packed as ax | ay << 21 | az << 42 (level-21 units),
// computed once per build so the descent below tests a node with one 8-byte load
// and a few shifts instead of three Morton compactions per node (the descent was
// instruction-bound, ncu: 69 % issue active).
// One 16-byte record per node for the descent: {anchor, level | nchild << 8, first
// child (internal) or leaf id (leaf)} -- one LDG.128 per visited node instead of
// five loads from the separate node arrays.
struct __align__(16) NodeRec {
    unsigned long long anc;
    int meta;
    int link;
};
__global__ void anchors_kernel(int nn, Nodes nd, const int *__restrict__ node_leaf, NodeRec *__restrict__ rec,
                               const DirCtl *__restrict__ ctl = nullptr) {
    if (ctl) {                                   // direct build: the node count is on the device
        if (dir_bad(ctl)) return;
        nn = (int)ctl->nn;
    }
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= nn) return;
    long long A[3], w;
    const int lev = nd.level[i], nc = nd.nchild[i];
    box_of(lev, nd.prefix[i], A, w);
    NodeRec r;
    r.anc = (unsigned long long)A[0] | ((unsigned long long)A[1] << 21) | ((unsigned long long)A[2] << 42);
    r.meta = lev | (nc << 8);
    r.link = nc ? nd.first_child[i] : node_leaf[i];
    rec[i] = r;
}

constexpr int kURow = 256;                  // max row length kept by the warp path
constexpr int kUFront = 512;                // max frontier length
constexpr int kUWarps = 4;                  // warps per block
__global__ void __launch_bounds__(32 * kUWarps) ulist_warp_kernel(int L, Nodes nd, const int *__restrict__ node_leaf,
                                                                  const int *__restrict__ leaf_node,
                                                                  const NodeRec *__restrict__ rec,
                                                                  int *__restrict__ rows, long long *__restrict__ counts,
                                                                  int *__restrict__ overflow,
                                                                  DirCtl *ctl = nullptr, int leaf_cap = 0) {
    __shared__ int front[kUWarps][2][kUFront];
    __shared__ int res[kUWarps][kURow];
    const int lane = threadIdx.x & 31, wi = threadIdx.x >> 5;
    const int nwarps = gridDim.x * kUWarps;
    if (ctl) {                                   // direct build: L on the device; counts past L zeroed (the scan
        if (dir_bad(ctl)) return;                // runs over the leaf capacity)
        L = ctl->L;
        overflow = &ctl->ulist_overflow;
        for (int j = L + 1 + blockIdx.x * blockDim.x + threadIdx.x; j <= leaf_cap; j += gridDim.x * blockDim.x)
            counts[j] = 0;
    }
    for (int t = blockIdx.x * kUWarps + wi; t < L; t += nwarps) {
        const int tn = leaf_node[t];
        long long At[3], wt;
        box_of(nd.level[tn], nd.prefix[tn], At, wt);
        int cur = 0, ncur = 1, nres = 0;
        bool ovf = false;
        if (lane == 0) front[wi][0][0] = 0;          // the root
        __syncwarp();
        while (ncur > 0 && !ovf) {
            int nnext = 0;
            for (int j0 = 0; j0 < ncur; j0 += 32) {
                const int j = j0 + lane;
                bool leaf = false;
                int nch = 0, fc = 0, lid = 0;
                if (j < ncur) {
                    const int ni = front[wi][cur][j];
                    const NodeRec r = rec[ni];
                    const int ws = 1 << (kMaxLevel - (r.meta & 255));
                    bool touch = true;
#pragma unroll
                    for (int a = 0; a < 3; ++a) {
                        const int As = (int)((r.anc >> (21 * a)) & 0x1fffffull);
                        touch &= (At[a] <= As + ws) && (As <= At[a] + wt);
                    }
                    if (touch) {
                        const int c = r.meta >> 8;
                        if (c == 0) {
                            leaf = true;
                            lid = r.link;
                        } else {
                            nch = c;
                            fc = r.link;
                        }
                    }
                }
                const unsigned lm = __ballot_sync(0xffffffffu, leaf);
                const int lpos = nres + __popc(lm & ((1u << lane) - 1));
                if (leaf && lpos < kURow) res[wi][lpos] = lid;
                nres += __popc(lm);
                int inc = nch;                        // exclusive prefix of child counts
#pragma unroll
                for (int o = 1; o < 32; o <<= 1) {
                    const int u = __shfl_up_sync(0xffffffffu, inc, o);
                    if (lane >= o) inc += u;
                }
                const int cpos = nnext + inc - nch;
                for (int c = 0; c < nch; ++c)
                    if (cpos + c < kUFront) front[wi][cur ^ 1][cpos + c] = fc + c;
                nnext += __shfl_sync(0xffffffffu, inc, 31);
            }
            __syncwarp();
            ovf = nres > kURow || nnext > kUFront;
            cur ^= 1;
            ncur = nnext;
        }
        if (ovf) {
            if (lane == 0) *overflow = 1;
            continue;
        }
        // rank sort (leaf ids are distinct): ascending leaf order
        int *row = rows + (size_t)t * kURow;
        for (int j = lane; j < nres; j += 32) {
            const int v = res[wi][j];
            int rk = 0;
            for (int k = 0; k < nres; ++k) rk += res[wi][k] < v;
            row[rk] = v;
        }
        if (lane == 0) counts[t] = nres;
        __syncwarp();
    }
}

__global__ void ulist_copy_kernel(int L, const int *__restrict__ rows, const long long *__restrict__ u_off,
                                  int *__restrict__ u_idx, DirCtl *ctl = nullptr, long long nnz_cap = 0) {
    if (ctl) {                                   // direct build: L and the entry total on the device
        if (dir_bad(ctl)) return;
        L = ctl->L;
        if (u_off[L] > nnz_cap) {
            if (blockIdx.x == 0 && threadIdx.x == 0) {
                ctl->nnz = u_off[L];                  // the size to grow to
                ctl->nnz_overflow = 1;
            }
            return;
        }
    }
    const int t = (int)((blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5);   // one warp per leaf
    if (t >= L) return;
    const long long o = u_off[t];
    const int n = (int)(u_off[t + 1] - o);
    for (int j = threadIdx.x & 31; j < n; j += 32) u_idx[o + j] = rows[(size_t)t * kURow + j];
}

__global__ void leaf_node_kernel(int nn, const int *__restrict__ node_leaf, int *__restrict__ leaf_node) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= nn) return;
    const int l = node_leaf[i];
    if (l >= 0) leaf_node[l] = i;
}

// index of (lev, prefix) among the previous build's nodes, or -1
__device__ __forceinline__ long long find_node(const PrevTree &pv, int lev, unsigned long long prefix) {
    if (lev >= pv.levels || lev < 0) return -1;
    long long lo = pv.base[lev], hi = pv.base[lev + 1];
    while (lo < hi) {
        const long long mid = lo + ((hi - lo) >> 1);
        if (pv.prefix[mid] < prefix) lo = mid + 1;
        else hi = mid;
    }
    return (lo < pv.base[lev + 1] && pv.prefix[lo] == prefix) ? lo : -1;
}

// M2L count (L18 SIV.D M(Op); reading R27): for node b (level >= 2), the
// children of the colleagues of parent(b) -- same-level nodes in the 3x3x3
// cells around it, parent included -- whose boxes do not touch b.  Counted as
// C(parent(b)) - N(b): C = the children the parent's colleagues have (their
// child counts), N = the nodes of b's level in b's own 3x3x3 cells, which are
// exactly the touching ones among those children (a same-level neighbour's parent
// is a colleague of b's parent) -- 54 lookups per node instead of up to 27 + 216.
__device__ __forceinline__ int neighbour_nodes(const PrevTree &pv, int lev, unsigned long long pre, bool children) {
    const long long c[3] = {(long long)compact3(pre), (long long)compact3(pre >> 1), (long long)compact3(pre >> 2)};
    const long long M = 1LL << lev;
    int cnt = 0;
    for (int dz = -1; dz <= 1; ++dz)
        for (int dy = -1; dy <= 1; ++dy)
            for (int dx = -1; dx <= 1; ++dx) {
                const long long qx = c[0] + dx, qy = c[1] + dy, qz = c[2] + dz;
                if (qx < 0 || qy < 0 || qz < 0 || qx >= M || qy >= M || qz >= M) continue;
                const long long q = find_node(pv, lev, spread3(qx) | (spread3(qy) << 1) | (spread3(qz) << 2));
                if (q >= 0) cnt += children ? pv.nchild[q] : 1;
            }
    return cnt;
}
__global__ void vlist_count_kernel(long long nn, PrevTree pv, unsigned long long *__restrict__ out) {
    const long long b = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    unsigned long long cnt = 0;
    if (b < nn) {
        int lev = 0;
        while (lev + 1 < pv.levels && pv.base[lev + 1] <= b) ++lev;
        if (lev >= 2) {
            const unsigned long long pre = pv.prefix[b];
            cnt = (unsigned long long)(neighbour_nodes(pv, lev - 1, pre >> 3, true) -
                                       neighbour_nodes(pv, lev, pre, false));
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
    if ((threadIdx.x & 31) == 0 && cnt) atomicAdd(out, cnt);
}

// sum_t n_t * sum_{s in U(t)} n_s
__global__ void p2p_count_kernel(int L, const int *__restrict__ lc, const long long *__restrict__ uo,
                                 const int *__restrict__ ui, unsigned long long *__restrict__ out) {
    const int t = blockIdx.x * blockDim.x + threadIdx.x;
    unsigned long long v = 0;
    if (t < L) {
        unsigned long long src = 0;
        for (long long u = uo[t]; u < uo[t + 1]; ++u) src += (unsigned long long)lc[ui[u]];
        v = src * (unsigned long long)lc[t];
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if ((threadIdx.x & 31) == 0 && v) atomicAdd(out, v);
}

__global__ void gather_kernel(long long n, const int *__restrict__ perm, const float *__restrict__ in,
                              float *__restrict__ out) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n;
         i += (long long)gridDim.x * blockDim.x)
        out[i] = in[perm[i]];
}
__global__ void gather_rows_kernel(long long n, int rows, const int *__restrict__ perm, const float *__restrict__ in,
                                   float *__restrict__ out) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n;
         i += (long long)gridDim.x * blockDim.x) {
        const long long src = perm[i];
        for (int r = 0; r < rows; ++r) out[r * n + i] = in[r * n + src];
    }
}
__global__ void scatter_kernel(long long n, const int *__restrict__ perm, const float *__restrict__ in,
                               float *__restrict__ out) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n;
         i += (long long)gridDim.x * blockDim.x)
        out[perm[i]] = in[i];
}

int grid_for(long long n, int threads) {
    long long g = (n + threads - 1) / threads;
    return (int)std::max<long long>(1, std::min<long long>(g, 1 << 20));
}

}  // namespace

// What a captured direct build depends on besides device-side state: the inputs,
// S, the mode, the domain and every buffer (ws_gen changes whenever one moves).
struct GraphKey {
    const float *x, *y, *z;
    long long n;
    int S, mode;
    unsigned long long gen;
    size_t cap;
    long long lcap, nnz_cap;
    double lo[3];
    int k;
    bool operator==(const GraphKey &o) const {
        return x == o.x && y == o.y && z == o.z && n == o.n && S == o.S && mode == o.mode && gen == o.gen &&
               cap == o.cap && lcap == o.lcap && nnz_cap == o.nnz_cap && lo[0] == o.lo[0] && lo[1] == o.lo[1] &&
               lo[2] == o.lo[2] && k == o.k;
    }
};

struct afmm_tree {
    int device = 0;
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    bool poisoned = false;
    bool built = false;
    std::string err;
    long long n = 0;
    int L = 0;
    long long nnz = 0, n_nodes = 0;
    double lo[3] = {0, 0, 0};
    int k = 0, max_level = 0;
    // device arrays
    int *perm = nullptr;
    unsigned long long *keys_sorted = nullptr;
    int *ls = nullptr, *lc = nullptr, *ll = nullptr;
    unsigned long long *lp = nullptr;
    long long *u_off = nullptr;
    int *u_idx = nullptr;
    std::vector<void *> owned;
    // node arrays of the last build (level-major, prefixes ascending per level):
    // the "previous tree" of the next afmm_tree_enforce
    unsigned long long *pv_prefix = nullptr;
    int *pv_nchild = nullptr;
    long long *pv_base = nullptr;
    size_t pv_cap = 0;
    int pv_levels = 0;
    // workspace arena: one grow-only device buffer per call site (no cudaMalloc
    // in steady state -- the tree is rebuilt every time step in C5)
    std::vector<void *> ws_ptr;
    std::vector<size_t> ws_cap;
    size_t node_cap = 1024;
    bool coop_ok = true;             // cooperative launch of levels_kernel available
    unsigned lvl_epoch = 0;          // launches of levels_kernel (tags its tile status words)
    long long sort_fallbacks = 0;    // bucket sorts that overflowed into the full radix sort
    // device words read by the next build: [0] = leaf count, [1] = levels of the last build (the
    // bucket sort and Enforce_S read them on the device, so a captured graph stays valid)
    int *d_state = nullptr;
    DirCtl *h_ctl = nullptr;         // pinned readback of the direct build
    unsigned long long ws_gen = 0;   // bumped whenever a workspace buffer is reallocated (graph key)
    static constexpr int kSlots = 4;                   // captured direct builds (the C5 loop alternates two input
    cudaGraphExec_t tg_exec[kSlots] = {};              // sets; the LB loop also alternates modes)
    GraphKey tg_key[kSlots] = {};
    long long tg_used[kSlots] = {};                    // last use (LRU replacement)
    GraphKey tg_seen[kSlots] = {};                     // keys of recent uncaptured builds: capture on a key's 2nd use
    int tg_seen_next = 0;
    long long tg_clock = 0;
    bool graph_broken = false;
    long long graph_launches = 0;
    long long dir_leaf_cap = 0;      // direct build: leaf / U-list entry capacities (grow-only, checked on the
    long long dir_nnz_cap = 0;       // device; an overflow grows them and reruns)
};

namespace {

afmm_status tfail(afmm_tree *t, afmm_status st, const char *fmt, ...) {
    if (t) {
        char buf[512];
        va_list ap;
        va_start(ap, fmt);
        vsnprintf(buf, sizeof(buf), fmt, ap);
        va_end(ap);
        t->err = buf;
        if (st == AFMM_ECUDA || st == AFMM_ENOMEM) t->poisoned = true;
    }
    return st;
}

#define TCU(t, call)                                                                          \
    do {                                                                                      \
        cudaError_t e_ = (call);                                                              \
        if (e_ != cudaSuccess)                                                                \
            return tfail((t), e_ == cudaErrorMemoryAllocation ? AFMM_ENOMEM : AFMM_ECUDA,      \
                         "%s failed: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__,     \
                         __LINE__);                                                           \
    } while (0)

void free_all(afmm_tree *t) {
    for (void *p : t->ws_ptr) cudaFree(p);
    t->ws_ptr.clear();
    t->ws_cap.clear();
    t->perm = nullptr;
    t->keys_sorted = nullptr;
    t->ls = t->lc = t->ll = nullptr;
    t->lp = nullptr;
    t->u_off = nullptr;
    t->u_idx = nullptr;
}

// grow-only workspace buffer for call site `slot` (contents not preserved on growth)
template <typename T>
afmm_status wsalloc(afmm_tree *t, int slot, T **p, size_t count) {
    const size_t bytes = std::max<size_t>(count, 1) * sizeof(T);
    if ((size_t)slot >= t->ws_ptr.size()) {
        t->ws_ptr.resize(slot + 1, nullptr);
        t->ws_cap.resize(slot + 1, 0);
    }
    if (t->ws_cap[slot] < bytes) {
        cudaFree(t->ws_ptr[slot]);
        t->ws_ptr[slot] = nullptr;
        t->ws_cap[slot] = 0;
        const size_t want = bytes + bytes / 2;
        ++t->ws_gen;
        TCU(t, cudaMalloc(&t->ws_ptr[slot], want));
        t->ws_cap[slot] = want;
    }
    *p = static_cast<T *>(t->ws_ptr[slot]);
    return AFMM_OK;
}

enum Slot {
    kPart, kKeys, kIdx, kKeysSorted, kPerm, kSortTmp, kNodeA, kNodeB = kNodeA + 6, kCb = kNodeB + 6, kNc, kOff,
    kScanTmp, kFlag, kLeafAt, kNodeLeaf, kScan2, kLs, kLc, kLl, kLp, kLeafNode, kCounts, kUoff, kScan3, kUidx,
    kFarfield, kEditPrefix, kEditAction, kEditBase, kURows, kUOvf, kLvlCtl, kTsum, kAnc,
    kCellLo, kCellHi, kBucket, kSlot, kBCount, kBOff, kBKeys, kBIdx, kBScan, kBOvf,
    kDirLvl, kDirFk, kDirLlo, kDirChunkCnt, kDirChunkBase, kDirLevelCnt, kDirCtl, kDirRank, kBBig, kBMid
};

__global__ void root_kernel(Nodes nd, int n) {
    nd.b[0] = 0;
    nd.e[0] = n;
    nd.first_child[0] = -1;
    nd.nchild[0] = 0;
    nd.level[0] = 0;
    nd.prefix[0] = 0ull;
}

}  // namespace

extern "C" afmm_status afmm_tree_create(int device, void *stream, afmm_tree **out) {
    if (!out) return AFMM_EINVAL;
    *out = nullptr;
    if (device < 0) return AFMM_EINVAL;
    afmm_tree *t = new (std::nothrow) afmm_tree();
    if (!t) return AFMM_ENOMEM;
    t->device = device;
    cudaError_t e = cudaSetDevice(device);
    if (e == cudaSuccess) {
        if (stream) {
            t->stream = static_cast<cudaStream_t>(stream);
        } else {
            e = cudaStreamCreateWithFlags(&t->stream, cudaStreamNonBlocking);
            t->own_stream = (e == cudaSuccess);
        }
    }
    if (e == cudaSuccess) e = cudaMalloc(&t->d_state, 2 * sizeof(int));
    if (e == cudaSuccess) e = cudaMemset(t->d_state, 0, 2 * sizeof(int));
    if (e == cudaSuccess) e = cudaMallocHost(&t->h_ctl, sizeof(DirCtl));
    if (e != cudaSuccess) {
        cudaFree(t->d_state);
        if (t->h_ctl) cudaFreeHost(t->h_ctl);
        if (t->own_stream && t->stream) cudaStreamDestroy(t->stream);
        delete t;
        return AFMM_ECUDA;
    }
    *out = t;
    return AFMM_OK;
}

extern "C" void afmm_tree_destroy(afmm_tree *t) {
    if (!t) return;
    cudaSetDevice(t->device);
    if (t->stream) cudaStreamSynchronize(t->stream);
    free_all(t);
    cudaFree(t->pv_prefix);
    cudaFree(t->pv_nchild);
    cudaFree(t->pv_base);
    cudaFree(t->d_state);
    if (t->h_ctl) cudaFreeHost(t->h_ctl);
    for (auto &g : t->tg_exec)
        if (g) cudaGraphExecDestroy(g);
    if (t->own_stream && t->stream) cudaStreamDestroy(t->stream);
    delete t;
}

extern "C" const char *afmm_tree_last_error(const afmm_tree *t) { return t ? t->err.c_str() : "null handle"; }

static afmm_status build_impl(afmm_tree *t, long long n, const float *x, const float *y, const float *z,
                              int S, int fixed_domain, const double *lo_in, int k_in, int mode,
                              Edits ed = Edits{nullptr, nullptr, nullptr, 0}) {
    nvtxRangePushA(mode == kModeFresh ? "afmm.tree_build" : mode == kModeEnforce ? "afmm.tree_enforce" : "afmm.tree_rebuild");
    struct Pop { ~Pop() { nvtxRangePop(); } } pop_;
    if (!t) return AFMM_EINVAL;
    if (t->poisoned) return AFMM_ESTATE;
    if (n < 1 || n >= (1LL << 31)) return tfail(t, AFMM_EINVAL, "tree_build: n=%lld out of range", n);
    if (S < 1) return tfail(t, AFMM_EINVAL, "tree_build: S=%d < 1", S);
    if (!x || !y || !z) return tfail(t, AFMM_EINVAL, "tree_build: null coordinate pointer");
    if (fixed_domain && (!lo_in || !std::isfinite(lo_in[0]) || !std::isfinite(lo_in[1]) ||
                         !std::isfinite(lo_in[2]) || k_in < -1000 || k_in > 1000))
        return tfail(t, AFMM_EINVAL, "tree_build: bad fixed domain");
    TCU(t, cudaSetDevice(t->device));
    // the previous build's domain and leaves (for the bucket sort of step 3)
    const bool had_prev = t->built && t->L > 0 && t->n == n;
    const double prev_lo[3] = {t->lo[0], t->lo[1], t->lo[2]};
    const int prev_k = t->k, prev_L = t->L;
    t->built = false;
    cudaStream_t st = t->stream;
    const int TH = 256;

    // 1. domain (reading R6): lo = min, side = smallest power of two > max extent
    if (fixed_domain) {
        for (int a = 0; a < 3; ++a) t->lo[a] = lo_in[a];
        t->k = k_in;
    } else {
        const int g = 296;
        float *part;
        if (afmm_status s = wsalloc(t, kPart, &part, (size_t)g * 6)) return s;
        minmax_kernel<<<g, TH, 0, st>>>(n, x, y, z, part);
        TCU(t, cudaGetLastError());
        std::vector<float> h(g * 6);
        TCU(t, cudaMemcpyAsync(h.data(), part, h.size() * sizeof(float), cudaMemcpyDeviceToHost, st));
        TCU(t, cudaStreamSynchronize(st));
        double ext = 0.0;
        for (int a = 0; a < 3; ++a) {
            float mn = h[a], mx = h[3 + a];
            for (int b = 1; b < g; ++b) {
                mn = std::min(mn, h[b * 6 + a]);
                mx = std::max(mx, h[b * 6 + 3 + a]);
            }
            t->lo[a] = (double)mn;
            ext = std::max(ext, (double)mx - (double)mn);
        }
        int e = 0;
        if (ext > 0.0) std::frexp(ext, &e);
        t->k = e;
    }
    const double scale = std::ldexp(1.0, kMaxLevel - t->k);

    // 2. keys; 3. stable radix sort by (key, index)
    unsigned long long *keys;
    int *idx;
    if (afmm_status s = wsalloc(t, kKeys, &keys, n)) return s;
    if (afmm_status s = wsalloc(t, kIdx, &idx, n)) return s;
    if (afmm_status s = wsalloc(t, kKeysSorted, &t->keys_sorted, n)) return s;
    if (afmm_status s = wsalloc(t, kPerm, &t->perm, n)) return s;
    auto full_sort = [&]() -> afmm_status {                   // first build / new domain / bucket overflow
        keys_kernel<<<grid_for(n, TH), TH, 0, st>>>(n, x, y, z, t->lo[0], t->lo[1], t->lo[2], scale, keys, idx);
        TCU(t, cudaGetLastError());
        size_t tb = 0;
        TCU(t, cub::DeviceRadixSort::SortPairs(nullptr, tb, keys, t->keys_sorted, idx, t->perm, (int)n, 0,
                                               3 * kMaxLevel, st));
        void *tbuf;
        if (afmm_status s = wsalloc(t, kSortTmp, reinterpret_cast<char **>(&tbuf), tb)) return s;
        TCU(t, cub::DeviceRadixSort::SortPairs(tbuf, tb, keys, t->keys_sorted, idx, t->perm, (int)n, 0,
                                               3 * kMaxLevel, st));
        return AFMM_OK;
    };
    const char *cub_env = getenv("AFMM_TREE_FULL_SORT");
    const bool buckets = had_prev && t->coop_ok && prev_k == t->k && prev_lo[0] == t->lo[0] &&
                         prev_lo[1] == t->lo[1] && prev_lo[2] == t->lo[2] && !(cub_env && cub_env[0] == '1');
    const char *lv_env = getenv("AFMM_TREE_LEVELS");                 // tests / A-B: force the level loop
    const char *dfs_env = getenv("AFMM_ULIST_DFS");                  // tests: force the DFS U-list fallback
    const char *gr_env = getenv("AFMM_TREE_GRAPH");                  // 0: no CUDA graph for the direct build
    const bool direct = (mode == kModeKeep || S <= kDirMaxS) && !(lv_env && lv_env[0] == '1');
    if (direct) {
        const char *small_env = getenv("AFMM_TREE_SMALL_CAPS");        // tests: start every capacity tiny
        const bool small = small_env && small_env[0] == '1';
        if (t->dir_leaf_cap == 0)                                    // first guess: ~ 4 n / S leaves
            t->dir_leaf_cap = small ? 1 : std::min<long long>(n, 1024 + 4 * n / std::max(1, S));
        if (t->dir_nnz_cap == 0) t->dir_nnz_cap = small ? 1 : 64 * t->dir_leaf_cap;
    }
    if (buckets && prev_L > t->dir_leaf_cap) t->dir_leaf_cap = prev_L;   // the bucket arrays hold the previous leaves
    // bucket sort by the previous leaves' cells (see bucket_sort_kernel): buffers sized by the leaf
    // capacity, the previous leaf count read on the device (so a captured graph stays valid)
    int *bovf = nullptr;
    unsigned long long *b_clo = nullptr, *b_chi = nullptr, *b_keys = nullptr;
    int *b_bucket = nullptr, *b_slot = nullptr, *b_count = nullptr, *b_off = nullptr, *b_idx = nullptr;
    int *b_big = nullptr, *b_mid = nullptr;
    char *b_sbuf = nullptr;
    size_t b_sb = 0;
    int kb_grid = 0;
    const long long bcap = std::max<long long>(t->dir_leaf_cap, 1), nbcap = 2 * bcap + 1;
    if (buckets) {
        if (afmm_status s = wsalloc(t, kCellLo, &b_clo, bcap)) return s;
        if (afmm_status s = wsalloc(t, kCellHi, &b_chi, bcap)) return s;
        if (afmm_status s = wsalloc(t, kBucket, &b_bucket, n)) return s;
        if (afmm_status s = wsalloc(t, kSlot, &b_slot, n)) return s;
        if (afmm_status s = wsalloc(t, kBCount, &b_count, (size_t)nbcap + 1)) return s;
        if (afmm_status s = wsalloc(t, kBOff, &b_off, (size_t)nbcap + 1)) return s;
        if (afmm_status s = wsalloc(t, kBKeys, &b_keys, n)) return s;
        if (afmm_status s = wsalloc(t, kBIdx, &b_idx, n)) return s;
        if (afmm_status s = wsalloc(t, kBOvf, &bovf, 1)) return s;
        if (afmm_status s = wsalloc(t, kBBig, &b_big, 1 + kBigList)) return s;
        if (afmm_status s = wsalloc(t, kBMid, &b_mid, (size_t)nbcap + 1)) return s;
        TCU(t, cudaFuncSetAttribute(bucket_big_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kBigSmem));
        TCU(t, cub::DeviceScan::ExclusiveSum(nullptr, b_sb, b_count, b_off, (int)(nbcap + 1), st));
        if (afmm_status s = wsalloc(t, kBScan, &b_sbuf, b_sb)) return s;
        int dev_sms = 0;
        TCU(t, cudaOccupancyMaxActiveBlocksPerMultiprocessor(&kb_grid, keys_bucket_kernel, kKeysThreads, 0));
        TCU(t, cudaDeviceGetAttribute(&dev_sms, cudaDevAttrMultiProcessorCount, t->device));
        kb_grid = (int)std::min<long long>((n + kKeysThreads - 1) / kKeysThreads, (long long)std::max(1, kb_grid) * dev_sms);
    }
    auto enq_buckets = [&]() -> afmm_status {
        TCU(t, cudaMemsetAsync(b_count, 0, ((size_t)nbcap + 1) * sizeof(int), st));
        TCU(t, cudaMemsetAsync(bovf, 0, sizeof(int), st));
        TCU(t, cudaMemsetAsync(b_big, 0, sizeof(int), st));
        TCU(t, cudaMemsetAsync(b_mid, 0, sizeof(int), st));
        cell_range_kernel<<<grid_for(bcap, TH), TH, 0, st>>>(t->d_state, t->ll, t->lp, b_clo, b_chi);
        keys_bucket_kernel<<<kb_grid, kKeysThreads, 0, st>>>(n, x, y, z, t->lo[0], t->lo[1], t->lo[2], scale, keys,
                                                             t->d_state, b_clo, b_chi, b_bucket, b_slot, b_count);
        size_t sb = b_sb;
        TCU(t, cub::DeviceScan::ExclusiveSum(b_sbuf, sb, b_count, b_off, (int)(nbcap + 1), st));
        bucket_scatter_kernel<<<grid_for(n, TH), TH, 0, st>>>(n, keys, b_bucket, b_slot, b_off, b_keys, b_idx);
        bucket_sort_kernel<<<(int)((nbcap + kBucketWarps - 1) / kBucketWarps), 32 * kBucketWarps, 0, st>>>(
            t->d_state, b_off, b_keys, b_idx, t->keys_sorted, t->perm, bovf, b_big, b_mid);
        bucket_mid_kernel<<<148 * 8, 32 * kBucketWarps, 0, st>>>(b_mid, b_off, b_keys, b_idx, t->keys_sorted, t->perm);
        bucket_big_kernel<<<kBigList / 2, kBigThreads, kBigSmem, st>>>(b_big, b_off, b_keys, b_idx, t->keys_sorted,
                                                                      t->perm);
        TCU(t, cudaGetLastError());
        return AFMM_OK;
    };
    if (!direct) {                                            // the level loop checks the bucket sort's flag itself
        if (buckets) {
            if (afmm_status s = enq_buckets()) return s;
        } else if (afmm_status s = full_sort()) {
            return s;
        }
    }

    // 4. level-synchronous split into one node array (level-major)
    size_t cap = t->node_cap;                 // grow-only across builds
    Nodes nd{};
    int node_set = kNodeA;
    auto alloc_nodes = [&](size_t c, Nodes &o, int set) -> afmm_status {
        if (afmm_status s = wsalloc(t, set + 0, &o.b, c)) return s;
        if (afmm_status s = wsalloc(t, set + 1, &o.e, c)) return s;
        if (afmm_status s = wsalloc(t, set + 2, &o.first_child, c)) return s;
        if (afmm_status s = wsalloc(t, set + 3, &o.nchild, c)) return s;
        if (afmm_status s = wsalloc(t, set + 4, &o.level, c)) return s;
        if (afmm_status s = wsalloc(t, set + 5, &o.prefix, c)) return s;
        return AFMM_OK;
    };
    if (afmm_status s = alloc_nodes(cap, nd, node_set)) return s;
    if (!t->coop_ok) {
        root_kernel<<<1, 1, 0, st>>>(nd, (int)n);
        TCU(t, cudaGetLastError());
    }
    PrevTree pv{t->pv_prefix, t->pv_nchild, t->pv_base, mode != kModeFresh ? t->pv_levels : 0};
    std::vector<long long> lvl_base;
    long long base = 0, m = 1;     // current level occupies [base, base+m)
    int level = 0;
    int *cb = nullptr, *nc = nullptr, *off = nullptr;
    bool done_levels = false;
    // 4d. direct construction from the sorted keys (fresh / Enforce_S with S <= kDirMaxS; KEEP; edits on either):
    //     leaves, nodes and U-lists by flat kernels that read their sizes on the device,
    //     into grow-only capacities checked on the device; ONE host readback at the end
    //     (sizes + overflow flags; an overflow grows the capacities and reruns, a warp
    //     U-list overflow continues on the host-driven path below).  With the bucket
    //     sort (a rebuild in the previous build's domain: every C5 step) the whole
    //     sequence -- sort, leaves, nodes, U-lists, previous-tree copy, readback -- is
    //     captured once into a CUDA graph and replayed (re-captured when the inputs,
    //     S, the mode or any buffer change): one launch instead of ~25 per build.
    int *flag = nullptr, *leaf_at = nullptr, *node_leaf = nullptr, *leaf_node = nullptr;
    int L = 0;
    bool use_buckets = buckets, need_sort = !buckets;
    for (int attempt = 0; direct && attempt < 8 && !done_levels; ++attempt) {
        unsigned char *lvl, *llo;
        unsigned long long *fk;
        int *chunk_cnt, *chunk_base, *level_cnt, *rank, *rows;
        long long *counts;
        NodeRec *rec;
        DirCtl *dctl;
        const long long nchunk = (n + kDirLeafBlock - 1) / kDirLeafBlock;
        const char *small_env = getenv("AFMM_TREE_SMALL_CAPS");
        if (!(small_env && small_env[0] == '1') && (long long)cap < 2 * n + 64) {
            cap = (size_t)(2 * n + 64);
            if (afmm_status s = alloc_nodes(cap, nd, node_set)) return s;
        }
        const int lcap = (int)t->dir_leaf_cap;
        if (afmm_status s = wsalloc(t, kFlag, &flag, n + 1)) return s;
        if (afmm_status s = wsalloc(t, kLeafAt, &leaf_at, n + 1)) return s;
        if (afmm_status s = wsalloc(t, kDirLvl, &lvl, n)) return s;
        if (afmm_status s = wsalloc(t, kLs, &t->ls, n)) return s;
        if (afmm_status s = wsalloc(t, kLc, &t->lc, n)) return s;
        if (afmm_status s = wsalloc(t, kLl, &t->ll, n)) return s;
        if (afmm_status s = wsalloc(t, kLp, &t->lp, n)) return s;
        if (afmm_status s = wsalloc(t, kDirFk, &fk, n)) return s;
        if (afmm_status s = wsalloc(t, kDirLlo, &llo, n)) return s;
        if (afmm_status s = wsalloc(t, kDirChunkCnt, &chunk_cnt, (size_t)nchunk * kDirLevels)) return s;
        if (afmm_status s = wsalloc(t, kDirChunkBase, &chunk_base, (size_t)nchunk * kDirLevels)) return s;
        if (afmm_status s = wsalloc(t, kDirLevelCnt, &level_cnt, kDirLevels)) return s;
        if (afmm_status s = wsalloc(t, kDirCtl, reinterpret_cast<char **>(&dctl), sizeof(DirCtl))) return s;
        if (afmm_status s = wsalloc(t, kNodeLeaf, &node_leaf, cap)) return s;
        if (afmm_status s = wsalloc(t, kLeafNode, &leaf_node, n)) return s;
        if (afmm_status s = wsalloc(t, kDirRank, &rank, (size_t)kDirLevels * ((size_t)lcap + 1))) return s;
        if (afmm_status s = wsalloc(t, kAnc, &rec, cap)) return s;
        if (afmm_status s = wsalloc(t, kCounts, &counts, (size_t)lcap + 1)) return s;
        if (afmm_status s = wsalloc(t, kUoff, &t->u_off, (size_t)lcap + 1)) return s;
        if (afmm_status s = wsalloc(t, kURows, &rows, (size_t)lcap * kURow)) return s;
        if (afmm_status s = wsalloc(t, kUidx, &t->u_idx, (size_t)t->dir_nnz_cap)) return s;
        size_t sb2 = 0, sb3 = 0;
        char *sbuf2, *sbuf3;
        TCU(t, cub::DeviceScan::ExclusiveSum(nullptr, sb2, flag, leaf_at, (int)(n + 1), st));
        if (afmm_status s = wsalloc(t, kScan2, &sbuf2, sb2)) return s;
        TCU(t, cub::DeviceScan::ExclusiveSum(nullptr, sb3, counts, t->u_off, lcap + 1, st));
        if (afmm_status s = wsalloc(t, kScan3, &sbuf3, sb3)) return s;
        if (cap > t->pv_cap) {                        // the previous tree's copy grows, keeping its contents (a rerun
            unsigned long long *np = nullptr;         // of this build reads them); this build overwrites it on success
            int *nc2 = nullptr;
            TCU(t, cudaMalloc(&np, cap * sizeof(unsigned long long)));
            TCU(t, cudaMalloc(&nc2, cap * sizeof(int)));
            if (t->pv_prefix && t->n_nodes > 0) {
                TCU(t, cudaMemcpyAsync(np, t->pv_prefix, (size_t)t->n_nodes * sizeof(unsigned long long),
                                       cudaMemcpyDeviceToDevice, st));
                TCU(t, cudaMemcpyAsync(nc2, t->pv_nchild, (size_t)t->n_nodes * sizeof(int), cudaMemcpyDeviceToDevice, st));
                TCU(t, cudaStreamSynchronize(st));
            }
            cudaFree(t->pv_prefix);
            cudaFree(t->pv_nchild);
            t->pv_prefix = np;
            t->pv_nchild = nc2;
            t->pv_cap = cap;
            pv.prefix = np;
            pv.nchild = nc2;
            ++t->ws_gen;
        }
        if (!t->pv_base) {
            TCU(t, cudaMalloc(&t->pv_base, (kMaxLevel + 2) * sizeof(long long)));
            ++t->ws_gen;
        }
        // KEEP after the bucket sort: a body's bucket names the previous leaf it stayed in, whose
        // level (t->ll, still the previous build's on a first attempt only) is its leaf level
        const bool hints = mode == kModeKeep && use_buckets && attempt == 0;
        auto enq_direct = [&]() -> afmm_status {
            TCU(t, cudaMemsetAsync(dctl, 0, sizeof(DirCtl), st));
            if (use_buckets) TCU(t, cudaMemcpyAsync(&dctl->sort_overflow, bovf, sizeof(int), cudaMemcpyDeviceToDevice, st));
            leaf_level_kernel<<<(int)((n + kDirTile - 1) / kDirTile), kDirThreads, 0, st>>>(
                n, t->keys_sorted, S, mode, pv, t->d_state + 1, ed, hints ? b_bucket : nullptr, t->perm, t->ll,
                lvl, flag);
            TCU(t, cudaGetLastError());
            size_t sb = sb2;
            TCU(t, cub::DeviceScan::ExclusiveSum(sbuf2, sb, flag, leaf_at, (int)(n + 1), st));
            leaf_info_kernel<<<grid_for(n, TH), TH, 0, st>>>(n, t->keys_sorted, lvl, flag, leaf_at, t->ls, t->ll,
                                                             t->lp, fk, llo);
            node_count_kernel<<<(int)nchunk, kDirLeafBlock, 0, st>>>(n, leaf_at, t->ls, t->ll, llo, t->lc, chunk_cnt);
            node_scan_kernel<<<1, 32 * kDirLevels, 0, st>>>(n, leaf_at, chunk_cnt, chunk_base, level_cnt, dctl);
            node_rank_kernel<<<(lcap + kDirLeafBlock - 1) / kDirLeafBlock, kDirLeafBlock, 0, st>>>(
                dctl, chunk_base, level_cnt, t->ls, t->lc, t->ll, llo, fk, rank, nd, node_leaf, leaf_node,
                (long long)cap, lcap);
            node_links_kernel<<<grid_for(std::min<long long>(lcap, 148LL * 64 * 4), TH), TH, 0, st>>>(
                n, dctl, t->ls, t->ll, llo, rank, nd, (long long)cap, lcap);
            anchors_kernel<<<grid_for((long long)cap, TH), TH, 0, st>>>((int)cap, nd, node_leaf, rec, dctl);
            const int ublocks = (int)std::min<long long>((lcap + kUWarps - 1) / kUWarps, 148LL * 16);
            ulist_warp_kernel<<<ublocks, 32 * kUWarps, 0, st>>>(lcap, nd, node_leaf, leaf_node, rec, rows, counts,
                                                                 nullptr, dctl, lcap);
            sb = sb3;
            TCU(t, cub::DeviceScan::ExclusiveSum(sbuf3, sb, counts, t->u_off, lcap + 1, st));
            ulist_copy_kernel<<<(int)(((long long)lcap * 32 + 255) / 256), 256, 0, st>>>(lcap, rows, t->u_off,
                                                                                        t->u_idx, dctl,
                                                                                        t->dir_nnz_cap);
            dir_finish_kernel<<<(int)std::min<long long>(grid_for((long long)cap, TH), 148LL * 8), TH, 0, st>>>(
                dctl, nd, t->u_off, t->pv_prefix, t->pv_nchild, t->pv_base, t->d_state);
            TCU(t, cudaGetLastError());
            TCU(t, cudaMemcpyAsync(t->h_ctl, dctl, sizeof(DirCtl), cudaMemcpyDeviceToHost, st));
            return AFMM_OK;
        };
        // not with edits: FineGrainedOptimize's trial rebuilds are one-offs (a capture each would cost more)
        const bool graph = use_buckets && ed.n == 0 && !(gr_env && gr_env[0] == '0') && !t->graph_broken;
        if (graph) {
            const GraphKey key{x, y, z, n, S, mode, t->ws_gen, cap, (long long)lcap, t->dir_nnz_cap,
                               {t->lo[0], t->lo[1], t->lo[2]}, t->k};
            int slot = -1;
            for (int g = 0; g < afmm_tree::kSlots; ++g)
                if (t->tg_exec[g] && t->tg_key[g] == key) slot = g;
            bool seen = false;                        // a key used once (a Search step's S) is not worth a capture
            for (int g = 0; g < afmm_tree::kSlots; ++g) seen |= t->tg_seen[g] == key;
            if (slot < 0 && !seen) t->tg_seen[t->tg_seen_next++ % afmm_tree::kSlots] = key;
            if (slot < 0 && seen) {                   // capture into the least recently used slot
                slot = 0;
                for (int g = 1; g < afmm_tree::kSlots; ++g)
                    if (t->tg_used[g] < t->tg_used[slot]) slot = g;
                if (t->tg_exec[slot]) cudaGraphExecDestroy(t->tg_exec[slot]);
                t->tg_exec[slot] = nullptr;
                cudaGraph_t gph = nullptr;
                cudaError_t e = cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal);
                afmm_status s1 = AFMM_OK, s2 = AFMM_OK;
                if (e == cudaSuccess) {
                    s1 = enq_buckets();
                    s2 = s1 ? s1 : enq_direct();
                    e = cudaStreamEndCapture(st, &gph);
                }
                if (s1 || s2) return s1 ? s1 : s2;
                if (e == cudaSuccess) e = cudaGraphInstantiate(&t->tg_exec[slot], gph, 0);
                if (gph) cudaGraphDestroy(gph);
                if (e != cudaSuccess) {               // no graph here: launch directly from now on
                    cudaGetLastError();
                    t->tg_exec[slot] = nullptr;
                    t->graph_broken = true;
                } else {
                    t->tg_key[slot] = key;
                }
            }
            if (slot >= 0 && t->tg_exec[slot]) {
                t->tg_used[slot] = ++t->tg_clock;
                TCU(t, cudaGraphLaunch(t->tg_exec[slot], st));
                ++t->graph_launches;
            } else {
                if (afmm_status s = enq_buckets()) return s;
                if (afmm_status s = enq_direct()) return s;
            }
        } else {
            if (use_buckets) {
                if (afmm_status s = enq_buckets()) return s;
            } else if (need_sort) {
                if (afmm_status s = full_sort()) return s;
                need_sort = false;
            }
            if (afmm_status s = enq_direct()) return s;
        }
        TCU(t, cudaStreamSynchronize(st));
        const DirCtl hc = *t->h_ctl;
        if (hc.sort_overflow) {                       // a bucket exceeded kBucketCap: sort in full, redo
            use_buckets = false;
            need_sort = true;
            ++t->sort_fallbacks;
            if (getenv("AFMM_TREE_DEBUG")) fprintf(stderr, "afmm tree: bucket sort overflow %lld\n", t->sort_fallbacks);
            continue;
        }
        if (hc.cap_overflow) {                        // grow the node / leaf capacities, redo (the sort stands)
            if (hc.nn > (long long)cap) {
                cap = (size_t)(hc.nn + hc.nn / 4);
                if (afmm_status s = alloc_nodes(cap, nd, node_set)) return s;
            }
            if (hc.L > t->dir_leaf_cap) t->dir_leaf_cap = std::min<long long>(n, hc.L + hc.L / 4);
            use_buckets = false;
            continue;
        }
        L = hc.L;
        t->max_level = hc.levels - 1;
        if (hc.ulist_overflow || (dfs_env && dfs_env[0] == '1')) {
            // the host-driven path below recounts the U-lists per thread (nodes and
            // leaves are complete; the previous-tree copy is made there)
            lvl_base.assign(hc.base, hc.base + hc.levels);
            base = hc.nn;
            done_levels = true;
            break;
        }
        if (hc.nnz_overflow) {                        // grow the U-list entry capacity, redo (the sort stands)
            t->dir_nnz_cap = hc.nnz + hc.nnz / 4 + 64;
            use_buckets = false;
            continue;
        }
        // complete: sizes for the host, done
        t->nnz = hc.nnz;
        t->n_nodes = hc.nn;
        t->node_cap = cap;
        t->pv_levels = hc.levels;
        t->L = L;
        t->n = n;
        t->built = true;
        return AFMM_OK;
    }
    const bool direct_done = done_levels;
    if (direct && !done_levels) return tfail(t, AFMM_ECUDA, "tree_build: direct construction kept overflowing");
    // 4a. all levels in one cooperative launch (grid barriers between phases); the
    //     node arrays start at >= 2n + 64 nodes and are doubled on overflow
    if (!done_levels && t->coop_ok) {
        if (cap < (size_t)(2 * n + 64)) {
            cap = (size_t)(2 * n + 64);
            if (afmm_status s = alloc_nodes(cap, nd, node_set)) return s;
        }
        LevelCtl *ctl;
        unsigned long long *tstat;
        if (afmm_status s = wsalloc(t, kCb, &cb, (size_t)(n + 1) * 9)) return s;
        if (afmm_status s = wsalloc(t, kNc, &nc, (size_t)n + 1)) return s;
        if (afmm_status s = wsalloc(t, kOff, &off, (size_t)n + 1)) return s;
        if (afmm_status s = wsalloc(t, kLvlCtl, reinterpret_cast<char **>(&ctl), sizeof(LevelCtl))) return s;
        int per_sm = 0, dev_sms = 0;
        TCU(t, cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, levels_kernel, kLvlThreads, 0));
        TCU(t, cudaDeviceGetAttribute(&dev_sms, cudaDevAttrMultiProcessorCount, t->device));
        const int blocks = std::max(1, std::min(per_sm, 1) * dev_sms);     // one per SM: cheaper grid barriers
        if (afmm_status s = wsalloc(t, kTsum, &tstat, (size_t)blocks)) return s;
        for (int attempt = 0; attempt < 8 && !done_levels; ++attempt) {
            root_kernel<<<1, 1, 0, st>>>(nd, (int)n);
            TCU(t, cudaGetLastError());
            TCU(t, cudaMemsetAsync(ctl, 0, sizeof(LevelCtl), st));
            if (bovf)                         // read back with the levels' LevelCtl: no extra sync
                TCU(t, cudaMemcpyAsync(&ctl->sort_overflow, bovf, sizeof(int), cudaMemcpyDeviceToDevice, st));
            long long capll = (long long)cap;
            unsigned epoch = ++t->lvl_epoch & 0x3fffffu;                 // status words of this launch
            if (epoch <= 1) {                  // first launch (fresh buffer) or the 22-bit tag wrapped: clear
                TCU(t, cudaMemsetAsync(tstat, 0, (size_t)blocks * sizeof(unsigned long long), st));
                if (epoch == 0) epoch = ++t->lvl_epoch & 0x3fffffu;
            }
            void *args[] = {&nd, &t->keys_sorted, &S, &mode, &pv, &ed, &cb, &nc, &off, &tstat, &epoch, &ctl, &capll};
            const cudaError_t e = cudaLaunchCooperativeKernel((const void *)levels_kernel, blocks, kLvlThreads, args,
                                                              0, st);
            if (e != cudaSuccess) {                   // no cooperative launch here: the per-level host loop
                cudaGetLastError();
                t->coop_ok = false;
                if (bovf) {                           // the bucket sort's overflow is not checked there
                    bovf = nullptr;
                    if (afmm_status s = full_sort()) return s;
                }
                break;
            }
            LevelCtl hc;
            TCU(t, cudaMemcpyAsync(&hc, ctl, sizeof(LevelCtl), cudaMemcpyDeviceToHost, st));
            TCU(t, cudaStreamSynchronize(st));
            if (hc.sort_overflow) {                   // a bucket exceeded kBucketCap: sort in full, redo the levels
                bovf = nullptr;
                ++t->sort_fallbacks;
                if (getenv("AFMM_TREE_DEBUG")) fprintf(stderr, "afmm tree: bucket sort overflow %lld\n", t->sort_fallbacks);
                if (afmm_status s = full_sort()) return s;
                continue;
            }
            if (hc.overflow) {                        // grow and rebuild the levels
                cap *= 2;
                node_set = node_set == kNodeA ? kNodeB : kNodeA;
                if (afmm_status s = alloc_nodes(cap, nd, node_set)) return s;
                continue;
            }
            lvl_base.assign(hc.base, hc.base + hc.levels);
            base = hc.base[hc.levels];
            t->max_level = hc.levels - 1;
            done_levels = true;
        }
        if (!done_levels && t->coop_ok) return tfail(t, AFMM_ENOMEM, "tree_build: node arrays kept overflowing");
        if (!done_levels) {
            root_kernel<<<1, 1, 0, st>>>(nd, (int)n);
            TCU(t, cudaGetLastError());
        }
    }
    if (!done_levels) {
    // 4b. per-level host loop (no cooperative launch)
    size_t lvl_cap = 0;
    void *scan_tmp = nullptr;
    size_t scan_tmp_bytes = 0;
    while (m > 0) {
        if ((size_t)m + 1 > lvl_cap) {
            lvl_cap = std::max<size_t>((size_t)m + 1, 2 * lvl_cap);
            if (afmm_status s = wsalloc(t, kCb, &cb, lvl_cap * 9)) return s;
            if (afmm_status s = wsalloc(t, kNc, &nc, lvl_cap)) return s;
            if (afmm_status s = wsalloc(t, kOff, &off, lvl_cap)) return s;
            size_t need = 0;
            TCU(t, cub::DeviceScan::ExclusiveSum(nullptr, need, nc, off, (int)lvl_cap, st));
            if (need > scan_tmp_bytes) {
                if (afmm_status s = wsalloc(t, kScanTmp, reinterpret_cast<char **>(&scan_tmp), need)) return s;
                scan_tmp_bytes = need;
            }
        }
        split_count_kernel<<<grid_for(8 * m, TH), TH, 0, st>>>((int)m, (int)base, nd, t->keys_sorted, S, mode, pv,
                                                                ed, cb, nc);
        TCU(t, cudaGetLastError());
        TCU(t, cudaMemsetAsync(nc + m, 0, sizeof(int), st));
        size_t sb = scan_tmp_bytes;
        TCU(t, cub::DeviceScan::ExclusiveSum(scan_tmp, sb, nc, off, (int)(m + 1), st));
        int total = 0;
        TCU(t, cudaMemcpyAsync(&total, off + m, sizeof(int), cudaMemcpyDeviceToHost, st));
        TCU(t, cudaStreamSynchronize(st));
        const long long next_base = base + m;
        if ((size_t)(next_base + total) > cap) {
            size_t ncap = std::max<size_t>(2 * cap, (size_t)(next_base + total));
            Nodes n2{};
            node_set = node_set == kNodeA ? kNodeB : kNodeA;
            if (afmm_status s = alloc_nodes(ncap, n2, node_set)) return s;
            TCU(t, cudaMemcpyAsync(n2.b, nd.b, next_base * sizeof(int), cudaMemcpyDeviceToDevice, st));
            TCU(t, cudaMemcpyAsync(n2.e, nd.e, next_base * sizeof(int), cudaMemcpyDeviceToDevice, st));
            TCU(t, cudaMemcpyAsync(n2.first_child, nd.first_child, next_base * sizeof(int), cudaMemcpyDeviceToDevice, st));
            TCU(t, cudaMemcpyAsync(n2.nchild, nd.nchild, next_base * sizeof(int), cudaMemcpyDeviceToDevice, st));
            TCU(t, cudaMemcpyAsync(n2.level, nd.level, next_base * sizeof(int), cudaMemcpyDeviceToDevice, st));
            TCU(t, cudaMemcpyAsync(n2.prefix, nd.prefix, next_base * sizeof(unsigned long long), cudaMemcpyDeviceToDevice, st));
            nd = n2;
            cap = ncap;
        }
        split_write_kernel<<<grid_for(m, TH), TH, 0, st>>>((int)m, (int)base, (int)next_base, nd, cb, nc, off);
        TCU(t, cudaGetLastError());
        t->max_level = level;
        lvl_base.push_back(base);
        base = next_base;
        m = total;
        ++level;
    }
    }
    const long long nn = base;     // total nodes
    t->n_nodes = nn;
    t->node_cap = cap;
    lvl_base.push_back(nn);
    // keep this tree's nodes as the "previous tree" of the next Enforce_S
    if ((size_t)nn > t->pv_cap) {
        cudaFree(t->pv_prefix);
        cudaFree(t->pv_nchild);
        t->pv_prefix = nullptr;
        t->pv_nchild = nullptr;
        t->pv_cap = 0;
        ++t->ws_gen;                               // a captured direct build referenced the old arrays
        TCU(t, cudaMalloc(&t->pv_prefix, (size_t)nn * sizeof(unsigned long long)));
        TCU(t, cudaMalloc(&t->pv_nchild, (size_t)nn * sizeof(int)));
        t->pv_cap = (size_t)nn;
    }
    if (!t->pv_base) {
        TCU(t, cudaMalloc(&t->pv_base, (kMaxLevel + 2) * sizeof(long long)));
        ++t->ws_gen;
    }
    TCU(t, cudaMemcpyAsync(t->pv_prefix, nd.prefix, nn * sizeof(unsigned long long), cudaMemcpyDeviceToDevice, st));
    TCU(t, cudaMemcpyAsync(t->pv_nchild, nd.nchild, nn * sizeof(int), cudaMemcpyDeviceToDevice, st));
    TCU(t, cudaMemcpyAsync(t->pv_base, lvl_base.data(), lvl_base.size() * sizeof(long long),
                           cudaMemcpyHostToDevice, st));
    t->pv_levels = (int)lvl_base.size() - 1;

    // 5. leaves in Morton order: flag first bodies, scan (the direct path has them)
    if (!direct_done) {
    if (afmm_status s = wsalloc(t, kFlag, &flag, n + 1)) return s;
    if (afmm_status s = wsalloc(t, kLeafAt, &leaf_at, n + 1)) return s;
    if (afmm_status s = wsalloc(t, kNodeLeaf, &node_leaf, nn)) return s;
    TCU(t, cudaMemsetAsync(flag, 0, (n + 1) * sizeof(int), st));
    leaf_flag_kernel<<<grid_for(nn, TH), TH, 0, st>>>((int)nn, nd, flag);
    TCU(t, cudaGetLastError());
    {
        size_t sb = 0;
        TCU(t, cub::DeviceScan::ExclusiveSum(nullptr, sb, flag, leaf_at, (int)(n + 1), st));
        char *sbuf;
        if (afmm_status s = wsalloc(t, kScan2, &sbuf, sb)) return s;
        TCU(t, cub::DeviceScan::ExclusiveSum(sbuf, sb, flag, leaf_at, (int)(n + 1), st));
    }
    TCU(t, cudaMemcpyAsync(&L, leaf_at + n, sizeof(int), cudaMemcpyDeviceToHost, st));
    TCU(t, cudaStreamSynchronize(st));
    if (afmm_status s = wsalloc(t, kLs, &t->ls, L)) return s;
    if (afmm_status s = wsalloc(t, kLc, &t->lc, L)) return s;
    if (afmm_status s = wsalloc(t, kLl, &t->ll, L)) return s;
    if (afmm_status s = wsalloc(t, kLp, &t->lp, L)) return s;
    leaf_write_kernel<<<grid_for(nn, TH), TH, 0, st>>>((int)nn, nd, leaf_at, node_leaf, t->ls, t->lc, t->ll, t->lp);
    TCU(t, cudaGetLastError());
    if (afmm_status s = wsalloc(t, kLeafNode, &leaf_node, L)) return s;
    leaf_node_kernel<<<grid_for(nn, TH), TH, 0, st>>>((int)nn, node_leaf, leaf_node);
    TCU(t, cudaGetLastError());
    }
    t->L = L;

    // 6. U-lists: warp-cooperative descent into fixed-capacity rows, scan, compact
    //    (rows longer than kURow or frontiers wider than kUFront: per-thread DFS count + fill)
    long long *counts;
    int *rows, *ovf;
    if (afmm_status s = wsalloc(t, kCounts, &counts, (size_t)L + 1)) return s;
    if (afmm_status s = wsalloc(t, kUoff, &t->u_off, (size_t)L + 1)) return s;
    if (afmm_status s = wsalloc(t, kURows, &rows, (size_t)L * kURow)) return s;
    if (afmm_status s = wsalloc(t, kUOvf, &ovf, 1)) return s;
    TCU(t, cudaMemsetAsync(counts + L, 0, sizeof(long long), st));
    TCU(t, cudaMemsetAsync(ovf, 0, sizeof(int), st));
    {
        const int blocks = (int)std::min<long long>((L + kUWarps - 1) / kUWarps, 148LL * 16);
        NodeRec *rec;
        if (afmm_status s = wsalloc(t, kAnc, &rec, (size_t)nn)) return s;
        anchors_kernel<<<grid_for(nn, TH), TH, 0, st>>>((int)nn, nd, node_leaf, rec);
        ulist_warp_kernel<<<blocks, 32 * kUWarps, 0, st>>>(L, nd, node_leaf, leaf_node, rec, rows, counts, ovf);
        TCU(t, cudaGetLastError());
    }
    // row offsets by a scan of the counts, read back together with the overflow flag
    // (one synchronise); on overflow the per-thread DFS recounts and the scan reruns
    auto scan_counts = [&]() -> afmm_status {
        size_t sb = 0;
        TCU(t, cub::DeviceScan::ExclusiveSum(nullptr, sb, counts, t->u_off, L + 1, st));
        char *sbuf;
        if (afmm_status s = wsalloc(t, kScan3, &sbuf, sb)) return s;
        TCU(t, cub::DeviceScan::ExclusiveSum(sbuf, sb, counts, t->u_off, L + 1, st));
        TCU(t, cudaMemcpyAsync(&t->nnz, t->u_off + L, sizeof(long long), cudaMemcpyDeviceToHost, st));
        return AFMM_OK;
    };
    int hovf = 0;
    if (afmm_status s = scan_counts()) return s;
    TCU(t, cudaMemcpyAsync(&hovf, ovf, sizeof(int), cudaMemcpyDeviceToHost, st));
    TCU(t, cudaStreamSynchronize(st));
    const char *dfs = getenv("AFMM_ULIST_DFS");                   // tests: force the fallback path
    if (dfs && dfs[0] == '1') hovf = 1;
    if (hovf) {
        ulist_kernel<<<grid_for(L, 128), 128, 0, st>>>(L, nd, node_leaf, leaf_node, nullptr, nullptr, counts);
        TCU(t, cudaGetLastError());
        TCU(t, cudaMemsetAsync(counts + L, 0, sizeof(long long), st));
        if (afmm_status s = scan_counts()) return s;
        TCU(t, cudaStreamSynchronize(st));
    }
    if (afmm_status s = wsalloc(t, kUidx, &t->u_idx, (size_t)t->nnz)) return s;
    if (hovf)
        ulist_kernel<<<grid_for(L, 128), 128, 0, st>>>(L, nd, node_leaf, leaf_node, t->u_off, t->u_idx, nullptr);
    else
        ulist_copy_kernel<<<(int)(((long long)L * 32 + 255) / 256), 256, 0, st>>>(L, rows, t->u_off, t->u_idx);
    TCU(t, cudaGetLastError());
    {                                             // the next build's device-side view of this one
        const int hs[2] = {L, t->pv_levels};
        TCU(t, cudaMemcpyAsync(t->d_state, hs, sizeof(hs), cudaMemcpyHostToDevice, st));
    }
    TCU(t, cudaStreamSynchronize(st));
    t->n = n;
    t->built = true;
    return AFMM_OK;
}

extern "C" afmm_status afmm_tree_build(afmm_tree *t, long long n, const float *x, const float *y,
                                       const float *z, int S, int fixed_domain, const double *lo_in,
                                       int k_in) {
    return build_impl(t, n, x, y, z, S, fixed_domain, lo_in, k_in, kModeFresh);
}

// Enforce_S (PAPER L20 SVI.A): the tree the last build becomes after its bodies
// moved -- same domain; a node splits iff it holds > S bodies, or exactly S and
// it was a parent in the previous tree (see split_count_kernel).
extern "C" afmm_status afmm_tree_enforce(afmm_tree *t, long long n, const float *x, const float *y,
                                         const float *z, int S) {
    if (!t) return AFMM_EINVAL;
    if (t->poisoned) return AFMM_ESTATE;
    if (!t->built || t->pv_levels < 1) return tfail(t, AFMM_ESTATE, "tree_enforce: no previous tree");
    if (n != t->n) return tfail(t, AFMM_EINVAL, "tree_enforce: n=%lld differs from the previous tree (%lld)", n, t->n);
    const double lo[3] = {t->lo[0], t->lo[1], t->lo[2]};
    return build_impl(t, n, x, y, z, S, 1, lo, t->k, kModeEnforce);
}

// Rebuild with per-node edits (Collapse / PushDown, L18 SIV.B-C) on top of the
// KEEP (structure of the last build) or ENFORCE rule -- FineGrainedOptimize's
// primitive (L20 SVI.B).
extern "C" afmm_status afmm_tree_rebuild(afmm_tree *t, long long n, const float *x, const float *y,
                                         const float *z, int S, int mode, int n_edits, const int *edit_level,
                                         const unsigned long long *edit_prefix, const int *edit_action) {
    if (!t) return AFMM_EINVAL;
    if (t->poisoned) return AFMM_ESTATE;
    if (!t->built || t->pv_levels < 1) return tfail(t, AFMM_ESTATE, "tree_rebuild: no previous tree");
    if (n != t->n) return tfail(t, AFMM_EINVAL, "tree_rebuild: n=%lld differs from the previous tree", n);
    if (mode != AFMM_TREE_KEEP && mode != AFMM_TREE_ENFORCE) return tfail(t, AFMM_EINVAL, "tree_rebuild: bad mode");
    if (n_edits < 0 || (n_edits > 0 && (!edit_level || !edit_prefix || !edit_action)))
        return tfail(t, AFMM_EINVAL, "tree_rebuild: bad edit list");
    std::vector<std::pair<std::pair<int, unsigned long long>, int>> e(n_edits);
    for (int i = 0; i < n_edits; ++i) {
        if (edit_level[i] < 0 || edit_level[i] > kMaxLevel || (edit_action[i] != 1 && edit_action[i] != 2))
            return tfail(t, AFMM_EINVAL, "tree_rebuild: edit %d invalid", i);
        e[i] = {{edit_level[i], edit_prefix[i]}, edit_action[i]};
    }
    std::sort(e.begin(), e.end());
    for (int i = 1; i < n_edits; ++i)
        if (e[i].first == e[i - 1].first && e[i].second != e[i - 1].second)
            return tfail(t, AFMM_EINVAL, "tree_rebuild: conflicting edits for one node");
    std::vector<long long> base(kMaxLevel + 2, 0);
    std::vector<unsigned long long> pre(std::max(n_edits, 1));
    std::vector<int> act(std::max(n_edits, 1));
    for (int i = 0; i < n_edits; ++i) {
        pre[i] = e[i].first.second;
        act[i] = e[i].second;
        base[e[i].first.first + 1]++;
    }
    for (int l = 0; l <= kMaxLevel; ++l) base[l + 1] += base[l];
    TCU(t, cudaSetDevice(t->device));
    unsigned long long *dp;
    int *da;
    long long *db;
    if (afmm_status s = wsalloc(t, kEditPrefix, &dp, pre.size())) return s;
    if (afmm_status s = wsalloc(t, kEditAction, &da, act.size())) return s;
    if (afmm_status s = wsalloc(t, kEditBase, &db, base.size())) return s;
    TCU(t, cudaMemcpyAsync(dp, pre.data(), pre.size() * sizeof(unsigned long long), cudaMemcpyHostToDevice, t->stream));
    TCU(t, cudaMemcpyAsync(da, act.data(), act.size() * sizeof(int), cudaMemcpyHostToDevice, t->stream));
    TCU(t, cudaMemcpyAsync(db, base.data(), base.size() * sizeof(long long), cudaMemcpyHostToDevice, t->stream));
    const double lo[3] = {t->lo[0], t->lo[1], t->lo[2]};
    return build_impl(t, n, x, y, z, S, 1, lo, t->k, mode == AFMM_TREE_KEEP ? kModeKeep : kModeEnforce,
                      Edits{dp, da, db, n_edits});
}

// All nodes of the last build (host outputs, nullable): level, prefix, child count.
extern "C" afmm_status afmm_tree_nodes(afmm_tree *t, int *level, unsigned long long *prefix, int *nchild) {
    if (!t) return AFMM_EINVAL;
    if (!t->built) return AFMM_ESTATE;
    TCU(t, cudaSetDevice(t->device));
    const long long nn = t->n_nodes;
    std::vector<long long> base(t->pv_levels + 1);
    TCU(t, cudaMemcpyAsync(base.data(), t->pv_base, base.size() * sizeof(long long), cudaMemcpyDeviceToHost, t->stream));
    if (prefix) TCU(t, cudaMemcpyAsync(prefix, t->pv_prefix, nn * sizeof(unsigned long long), cudaMemcpyDeviceToHost, t->stream));
    if (nchild) TCU(t, cudaMemcpyAsync(nchild, t->pv_nchild, nn * sizeof(int), cudaMemcpyDeviceToHost, t->stream));
    TCU(t, cudaStreamSynchronize(t->stream));
    if (level)
        for (int l = 0; l < t->pv_levels; ++l)
            for (long long i = base[l]; i < base[l + 1]; ++i) level[i] = l;
    return AFMM_OK;
}

extern "C" afmm_status afmm_tree_counters(const afmm_tree *t, long long *graph_launches, long long *sort_fallbacks) {
    if (!t) return AFMM_EINVAL;
    if (graph_launches) *graph_launches = t->graph_launches;
    if (sort_fallbacks) *sort_fallbacks = t->sort_fallbacks;
    return AFMM_OK;
}

extern "C" afmm_status afmm_tree_info(const afmm_tree *t, int *n_leaves, long long *nnz, double *lo,
                                      int *k, int *max_level, long long *n_nodes) {
    if (!t) return AFMM_EINVAL;
    if (!t->built) return AFMM_ESTATE;
    if (n_leaves) *n_leaves = t->L;
    if (nnz) *nnz = t->nnz;
    if (lo)
        for (int a = 0; a < 3; ++a) lo[a] = t->lo[a];
    if (k) *k = t->k;
    if (max_level) *max_level = t->max_level;
    if (n_nodes) *n_nodes = t->n_nodes;
    return AFMM_OK;
}

extern "C" afmm_status afmm_tree_copy_out(const afmm_tree *tc, int *perm, int *leaf_start, int *leaf_count,
                                          int *leaf_level, unsigned long long *leaf_prefix,
                                          long long *u_off, int *u_idx) {
    afmm_tree *t = const_cast<afmm_tree *>(tc);
    if (!t) return AFMM_EINVAL;
    if (!t->built) return AFMM_ESTATE;
    TCU(t, cudaSetDevice(t->device));
    cudaStream_t st = t->stream;
    if (perm) TCU(t, cudaMemcpyAsync(perm, t->perm, t->n * sizeof(int), cudaMemcpyDeviceToHost, st));
    if (leaf_start) TCU(t, cudaMemcpyAsync(leaf_start, t->ls, t->L * sizeof(int), cudaMemcpyDeviceToHost, st));
    if (leaf_count) TCU(t, cudaMemcpyAsync(leaf_count, t->lc, t->L * sizeof(int), cudaMemcpyDeviceToHost, st));
    if (leaf_level) TCU(t, cudaMemcpyAsync(leaf_level, t->ll, t->L * sizeof(int), cudaMemcpyDeviceToHost, st));
    if (leaf_prefix)
        TCU(t, cudaMemcpyAsync(leaf_prefix, t->lp, t->L * sizeof(unsigned long long), cudaMemcpyDeviceToHost, st));
    if (u_off) TCU(t, cudaMemcpyAsync(u_off, t->u_off, (t->L + 1) * sizeof(long long), cudaMemcpyDeviceToHost, st));
    if (u_idx && t->nnz > 0)
        TCU(t, cudaMemcpyAsync(u_idx, t->u_idx, t->nnz * sizeof(int), cudaMemcpyDeviceToHost, st));
    TCU(t, cudaStreamSynchronize(st));
    return AFMM_OK;
}

extern "C" afmm_status afmm_tree_farfield_counts(afmm_tree *t, long long *counts) {
    if (!t || !counts) return AFMM_EINVAL;
    if (!t->built) return AFMM_ESTATE;
    TCU(t, cudaSetDevice(t->device));
    unsigned long long *d = nullptr;
    if (afmm_status s = wsalloc(t, kFarfield, &d, 2)) return s;
    TCU(t, cudaMemsetAsync(d, 0, 2 * sizeof(unsigned long long), t->stream));
    PrevTree pv{t->pv_prefix, t->pv_nchild, t->pv_base, t->pv_levels};
    vlist_count_kernel<<<grid_for(t->n_nodes, 256), 256, 0, t->stream>>>(t->n_nodes, pv, d);
    TCU(t, cudaGetLastError());
    p2p_count_kernel<<<grid_for(t->L, 256), 256, 0, t->stream>>>(t->L, t->lc, t->u_off, t->u_idx, d + 1);
    TCU(t, cudaGetLastError());
    unsigned long long h[2];
    TCU(t, cudaMemcpyAsync(h, d, sizeof(h), cudaMemcpyDeviceToHost, t->stream));
    TCU(t, cudaStreamSynchronize(t->stream));
    counts[0] = t->L;
    counts[1] = t->n_nodes - 1;
    counts[2] = (long long)h[0];
    counts[3] = t->n_nodes - 1;
    counts[4] = t->L;
    counts[5] = (long long)h[1];
    return AFMM_OK;
}

extern "C" afmm_status afmm_tree_device_arrays(const afmm_tree *t, const int **perm, const int **leaf_start,
                                               const int **leaf_count, const long long **u_off,
                                               const int **u_idx) {
    if (!t) return AFMM_EINVAL;
    if (!t->built) return AFMM_ESTATE;
    if (perm) *perm = t->perm;
    if (leaf_start) *leaf_start = t->ls;
    if (leaf_count) *leaf_count = t->lc;
    if (u_off) *u_off = t->u_off;
    if (u_idx) *u_idx = t->u_idx;
    return AFMM_OK;
}

extern "C" afmm_status afmm_tree_gather(afmm_tree *t, const float *in, float *out) {
    if (!t || !in || !out) return AFMM_EINVAL;
    if (!t->built) return AFMM_ESTATE;
    TCU(t, cudaSetDevice(t->device));
    gather_kernel<<<grid_for(t->n, 256), 256, 0, t->stream>>>(t->n, t->perm, in, out);
    TCU(t, cudaGetLastError());
    return AFMM_OK;
}

extern "C" afmm_status afmm_tree_gather_rows(afmm_tree *t, int rows, const float *in, float *out) {
    if (!t || !in || !out || rows < 1) return AFMM_EINVAL;
    if (!t->built) return AFMM_ESTATE;
    TCU(t, cudaSetDevice(t->device));
    gather_rows_kernel<<<grid_for(t->n, 256), 256, 0, t->stream>>>(t->n, rows, t->perm, in, out);
    TCU(t, cudaGetLastError());
    return AFMM_OK;
}

extern "C" afmm_status afmm_tree_scatter(afmm_tree *t, const float *in, float *out) {
    if (!t || !in || !out) return AFMM_EINVAL;
    if (!t->built) return AFMM_ESTATE;
    TCU(t, cudaSetDevice(t->device));
    scatter_kernel<<<grid_for(t->n, 256), 256, 0, t->stream>>>(t->n, t->perm, in, out);
    TCU(t, cudaGetLastError());
    return AFMM_OK;
}
