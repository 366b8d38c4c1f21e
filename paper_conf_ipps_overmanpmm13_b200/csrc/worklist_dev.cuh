// worklist_dev.cuh -- device-side tree ingest (afmm_p2p_set_tree_device), included by afmm_p2p.cu.
//
// Same contract and same results as the host path (validation, Interactions(t),
// the literal / coefficient partition, the per-leaf segment lists and the
// cost-model target slices of worklist.inc, largest-cost-first order), computed
// by kernels on arrays that already live on the GPU (e.g. afmm_tree outputs),
// so a time step never round-trips the tree through host memory.
#pragma once
#include <cub/cub.cuh>

namespace afmm {
namespace dev {

enum : int {
    kErrStart = 1, kErrCount = 2, kErrCover = 4, kErrOff = 8, kErrIdx = 16, kErrOrder = 32
};

__device__ __forceinline__ int bucket_of_d(int nt) {
    int b = 0, cap = 8;
    while (nt > cap && b < 7) {
        cap <<= 1;
        ++b;
    }
    return b;
}

// validation + Interactions(t) = n_t * sum_{s in U(t)} n_s, and for the work list
// each leaf's segment count (runs of consecutive source leaves, the leaf itself
// apart) and source total: one warp per leaf, a lane per U-list entry
__device__ __forceinline__ unsigned lanes_below(int lane) { return (1u << lane) - 1u; }
__global__ void validate_interactions_kernel(int L, long long n, int max_leaf, const int *__restrict__ ls,
                                             const int *__restrict__ lc, const long long *__restrict__ uo,
                                             const int *__restrict__ ui, long long *__restrict__ I,
                                             int *__restrict__ nseg_all, long long *__restrict__ nsrc_all,
                                             int *__restrict__ err) {
    const long long gw = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    if (gw >= L) return;                                     // whole warps
    const int t = (int)gw;
    int e = 0;
    const int c = lc[t];
    if (lane == 0) {
        if (c < 1 || c > max_leaf) e |= kErrCount;
        if (t == 0 && ls[0] != 0) e |= kErrStart;
        if (t + 1 < L && ls[t + 1] != ls[t] + c) e |= kErrStart;
        if (t + 1 == L && (long long)ls[t] + c != n) e |= kErrCover;
        if (t == 0 && uo[0] != 0) e |= kErrOff;
    }
    const long long b = uo[t], en = uo[t + 1], nnz = uo[L];
    long long src = 0;
    int runs = 0;
    bool self = false;
    if (en < b || b < 0 || en > nnz) {               // (reads stay inside u_idx[0, u_off[L]))
        e |= kErrOff;
    } else {
        for (long long u0 = b; u0 < en; u0 += 32) {
            const long long u = u0 + lane;
            const bool in = u < en;
            const int s = in ? ui[u] : -1;
            const bool ok = in && s >= 0 && s < L;
            if (in && !ok) e |= kErrIdx;
            const int prev = in && u > b ? ui[u - 1] : -1;
            if (ok && s <= prev) e |= kErrOrder;
            if (ok) src += lc[s];
            self |= ok && s == t;
            // the previous entry other than the leaf itself; a run continues iff s follows it
            // (leaves are contiguous once validated: ls[p + 1] == ls[p] + lc[p])
            int p = prev;
            if (p == t) p = in && u - 1 > b ? ui[u - 2] : -1;
            runs += ok && s != t && !(p >= 0 && s == p + 1);
        }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        e |= __shfl_xor_sync(0xffffffffu, e, o);
        src += __shfl_xor_sync(0xffffffffu, src, o);
        runs += __shfl_xor_sync(0xffffffffu, runs, o);
    }
    self = __any_sync(0xffffffffu, self);
    if (lane == 0) {
        I[t] = (long long)c * src;
        nseg_all[t] = runs + (self ? 1 : 0);
        nsrc_all[t] = src;
        if (e) atomicOr(err, e);
    }
}

// Literal greedy cut (PAPER L16 SIII.C) from the inclusive prefix sums P[t] =
// sum_{u <= t} I(u): cut r+1 = 1 + first t >= cut_r whose running count
// P[t] - P[cut_r - 1] satisfies count * G >= total.  Single thread, G <= 64 binary searches.
// (+ the body range of every slice, bsplit[g] = first body of leaf split[g], n past the end)
__global__ void literal_cut_kernel(int L, int G, const long long *__restrict__ P, long long *__restrict__ split,
                                   long long n, const int *__restrict__ ls, long long *__restrict__ bsplit) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    const long long total = P[L - 1];
    long long start = 0;
    split[0] = 0;
    int g = 0;
    for (; g < G - 1 && start < L; ++g) {
        const long long base = start > 0 ? P[start - 1] : 0;
        long long lo = start, hi = L;                 // first t with (P[t] - base) * G >= total
        while (lo < hi) {
            const long long mid = lo + ((hi - lo) >> 1);
            if ((__int128)(P[mid] - base) * G >= (__int128)total) hi = mid;
            else lo = mid + 1;
        }
        if (lo >= L) break;
        start = lo + 1;
        split[g + 1] = start;
    }
    for (int r = g + 1; r <= G; ++r) split[r] = L;
    for (int r = 0; r <= G; ++r) bsplit[r] = split[r] >= L ? n : ls[split[r]];
}

// The same rule on weights w(t) = I(t) * coef[bucket(n_t)] (prefix sums in fp64).
__global__ void weights_kernel(int L, const int *__restrict__ lc, const long long *__restrict__ I,
                               const double *__restrict__ coef, double *__restrict__ w) {
    const int t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t < L) w[t] = (double)I[t] * coef[bucket_of_d(lc[t])];
}
__global__ void weighted_cut_kernel(int L, int G, const double *__restrict__ P, long long *__restrict__ split) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    const double total = P[L - 1];
    long long start = 0;
    split[0] = 0;
    int g = 0;
    for (; g < G - 1 && start < L; ++g) {
        const double base = start > 0 ? P[start - 1] : 0.0;
        long long lo = start, hi = L;
        while (lo < hi) {
            const long long mid = lo + ((hi - lo) >> 1);
            if ((P[mid] - base) * G >= total) hi = mid;
            else lo = mid + 1;
        }
        if (lo >= L) break;
        start = lo + 1;
        split[g + 1] = start;
    }
    for (int r = g + 1; r <= G; ++r) split[r] = L;
}


// pass 1 over this rank's leaves [lo, lo+m) = [split[r], split[r+1]): segment and
// slice counts (zero from m to L, so scans over L+1 entries end at the totals),
// nsrc, the leaf's slice plan (the DP runs once per leaf) under the task cap of
// the total P[L-1], bucket statistics and the largest task cost (int64 atomics,
// summed per warp first: order-independent).  Nothing when validation failed.
__global__ void count_kernel(int L, int r, const long long *__restrict__ split, const long long *__restrict__ P,
                             int sw, long long warps, const int *__restrict__ err, const int *__restrict__ lc,
                             const int *__restrict__ nseg_all, const long long *__restrict__ nsrc_all,
                             const long long *__restrict__ I, unsigned long long *__restrict__ nst,
                             long long *__restrict__ nsrc, unsigned long long *__restrict__ stats,
                             unsigned short *__restrict__ plan, int4 *__restrict__ plan_hdr) {
    if (*err) return;
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    const int lo = (int)split[r], m = (int)(split[r + 1] - split[r]);
    const long long cap = task_cap(P[L - 1] / sw, warps);
    if (i >= m && i <= L) nst[i] = 0;
    const bool live = i < m;
    unsigned long long inter = 0, cm = 0;
    int bk = -1;
    if (live) {
        const int t = lo + i;
        const long long src = nsrc_all[t];
        nsrc[i] = src;
        int n_full = 0, full_m = 0, max_m = 0;
        const int k = plan_slices(lc[t], src, cap, &n_full, &full_m, plan + (size_t)i * kMaxDpSlices, &max_m);
        plan_hdr[i] = make_int4(n_full, full_m, k, 0);
        // segment and task counts packed (tasks << 32 | segments): one scan gives both offsets
        nst[i] = (unsigned long long)(n_full + k) << 32 | (unsigned)nseg_all[t];
        inter = (unsigned long long)I[t];
        bk = bucket_of_d(lc[t]);
        cm = (unsigned long long)slice_iters(src, max_m);    // the largest slice has the largest cost
    }
    const int lane = threadIdx.x & 31;
    unsigned long long tot = inter;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        tot += __shfl_xor_sync(0xffffffffu, tot, o);
        const unsigned long long c2 = __shfl_xor_sync(0xffffffffu, cm, o);
        cm = c2 > cm ? c2 : cm;
    }
    if (lane == 0 && tot) atomicAdd(&stats[0], tot);
    if (lane == 0 && cm) atomicMax(&stats[9], cm);
    for (unsigned todo = __ballot_sync(0xffffffffu, bk >= 0); todo;) {   // per bucket present in the warp
        const int lb = __shfl_sync(0xffffffffu, bk, __ffs(todo) - 1);
        unsigned long long v = bk == lb ? inter : 0ull;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        if (lane == 0 && v) atomicAdd(&stats[1 + lb], v);
        todo &= ~__ballot_sync(0xffffffffu, bk == lb);
    }
}

// pass 2, one warp per leaf: segments (self first, then the runs of consecutive
// source leaves) and the leaf's tasks with their LPT cost keys
__global__ void write_kernel(int r, const long long *__restrict__ split, const int *__restrict__ gate,
                             const int *__restrict__ ls, const int *__restrict__ lc,
                             const long long *__restrict__ uo, const int *__restrict__ ui,
                             const unsigned long long *__restrict__ off2,
                             const long long *__restrict__ nsrc, Seg *__restrict__ segs, Task *__restrict__ tasks,
                             unsigned long long *__restrict__ keys, int *__restrict__ vals,
                             const unsigned short *__restrict__ plan, const int4 *__restrict__ plan_hdr,
                             const unsigned long long *__restrict__ cmax_ptr) {
    const long long gw = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
    const int lane = threadIdx.x & 31;
    const int lo = (int)split[r], m = (int)(split[r + 1] - split[r]);
    if (gw >= m || *gate == 0) return;                        // whole warps; gate: valid and fits
    const int i = (int)gw, t = lo + i;
    const int ts = ls[t], tn = lc[t];
    const int seg_begin = (int)(unsigned)off2[i], task_begin = (int)(off2[i] >> 32);
    const long long b = uo[t], en = uo[t + 1];
    bool self = false;
    for (long long u = b + lane; u < en; u += 32) self |= ui[u] == t;
    self = __any_sync(0xffffffffu, self);
    if (self && lane == 0) segs[seg_begin] = Seg{ts, tn};
    const int w0 = seg_begin + (self ? 1 : 0);
    int run = -1, run_gs = 0, prev_s = -1;                    // the open run (index, first body) and last source
    for (long long u0 = b; u0 < en; u0 += 32) {
        const long long u = u0 + lane;
        const int s = u < en ? ui[u] : t;
        const bool ns = s != t;
        const unsigned mask = __ballot_sync(0xffffffffu, ns);
        if (!mask) continue;
        const unsigned below = mask & lanes_below(lane);
        const int pl = below ? 31 - __clz(below) : 0;
        int p = __shfl_sync(0xffffffffu, s, pl);
        if (!below) p = prev_s;
        const bool nr = ns && !(p >= 0 && s == p + 1);
        const unsigned nrm = __ballot_sync(0xffffffffu, nr);
        const int my_run = run + __popc(nrm & (lanes_below(lane) | (1u << lane)));
        const int g_own = ns ? ls[s] : 0, end = ns ? g_own + lc[s] : 0;
        const unsigned upto = nrm & (lanes_below(lane) | (1u << lane));
        const int rl = upto ? 31 - __clz(upto) : 0;
        int gs = __shfl_sync(0xffffffffu, g_own, rl);
        if (!upto) gs = run_gs;
        const unsigned above = mask & ~(lanes_below(lane) | (1u << lane));
        const int nl = above ? __ffs(above) - 1 : -1;
        const bool last_of_run = ns && (nl < 0 || ((nrm >> nl) & 1u));
        if (last_of_run) segs[w0 + my_run] = Seg{gs, end - gs};   // (a run crossing chunks is rewritten longer)
        const int top = 31 - __clz(mask);
        prev_s = __shfl_sync(0xffffffffu, s, top);
        run = __shfl_sync(0xffffffffu, my_run, top);
        run_gs = __shfl_sync(0xffffffffu, gs, top);
    }
    const int seg_count = (self ? 1 : 0) + run + 1;
    const long long src = nsrc[i];
    const unsigned short *sz = plan + (size_t)i * kMaxDpSlices;           // count_kernel's plan
    const int4 hd = plan_hdr[i];
    const int n_full = hd.x, full_m = hd.y, total = hd.x + hd.z;
    const unsigned long long cmax = *cmax_ptr;
    int carry = 0;
    for (int j0 = 0; j0 < total; j0 += 32) {
        const int j = j0 + lane;
        const int cnt = j < total ? plan_size(j, n_full, full_m, sz) : 0;
        int inc = cnt;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int v = __shfl_up_sync(0xffffffffu, inc, o);
            if (lane >= o) inc += v;
        }
        if (j < total) {
            const int q = task_begin + j;
            tasks[q] = Task{ts + carry + inc - cnt, cnt, ts, self ? tn : 0, seg_begin, seg_count, (int)src, 0};
            keys[q] = cmax - (unsigned long long)slice_iters(src, cnt);   // ascending = largest cost first
            vals[q] = q;
        }
        carry += __shfl_sync(0xffffffffu, inc, 31);
    }
}

// Stable LSD radix sort of the tasks by key (cmax - cost, so ascending = largest
// cost first), 8-bit digits, as many passes as cmax has bytes -- ONE cooperative
// launch (round 1: CUB's radix sort + a gather kernel).  nt and cmax are read on
// the device.  The first Geff = ceil(nt / kSortTile) blocks own contiguous tiles.
// Per pass every tile publishes its digit counts in status words tagged with the
// launch epoch and the pass (nothing is reset between passes or launches); every
// tile then reads ALL tiles' words -- the earlier ones give its exclusive start in
// each digit, the sum the digit totals -- with batched independent loads (no
// look-back chain), and scatters its keys in order (warp match_any ranks +
// per-warp digit counts).  One grid barrier per pass; the last pass writes the Task
// records themselves.
struct SortCtl {
    unsigned bar_count, bar_gen;
};
constexpr int kSortThreads = 512, kSortWarps = kSortThreads / 32, kRadix = 256, kMaxSortPasses = 8,
              kSortTile = 1024;
__device__ __forceinline__ void sort_grid_barrier(SortCtl *c) {
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
__device__ __forceinline__ unsigned long long ld_relaxed_u64(const unsigned long long *p) {
    unsigned long long v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__global__ void __launch_bounds__(kSortThreads) task_sort_kernel(
    const int *__restrict__ nt_ptr, const unsigned long long *__restrict__ cmax_ptr, unsigned long long *k0, int *v0,
    unsigned long long *k1, int *v1, const Task *__restrict__ tasks_u, Task *__restrict__ out,
    unsigned long long *__restrict__ status, unsigned epoch, SortCtl *ctl) {
    __shared__ unsigned wh[kSortWarps][kRadix];
    __shared__ unsigned cnt[kRadix], run[kRadix], part[2][2][kRadix], wsum[kSortWarps];
    const int nt = *nt_ptr;
    if (nt <= 0) return;                                       // (every block: no barrier is reached)
    const unsigned long long cmax = *cmax_ptr;
    const int P = (64 - __clzll(cmax | 1ull) + 7) / 8;
    const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
    const int b = (int)blockIdx.x;
    const int Geff = min((int)gridDim.x, (nt + kSortTile - 1) / kSortTile);
    const int tile = (nt + Geff - 1) / Geff;
    const int t0 = b < Geff ? min(nt, b * tile) : nt, t1 = b < Geff ? min(nt, t0 + tile) : nt;
    for (int p = 0; p < P; ++p) {
        const unsigned long long *sk = (p & 1) ? k1 : k0;
        const int *sv = (p & 1) ? v1 : v0;
        unsigned long long *dk = (p & 1) ? k0 : k1;
        int *dv = (p & 1) ? v0 : v1;
        const bool last = p == P - 1;
        const int sh = 8 * p;
        const unsigned tag = ((epoch << 3) | (unsigned)p) & 0x3fffffffu;
        if (b < Geff) {
            if (tid < kRadix) cnt[tid] = 0;
            __syncthreads();
            for (int i = t0 + tid; i < t1; i += kSortThreads) atomicAdd(&cnt[(sk[i] >> sh) & 255u], 1u);
            __syncthreads();
            if (tid < kRadix)
                atomicExch(status + (size_t)b * kRadix + tid, ((unsigned long long)tag << 32) | cnt[tid]);
            // all tiles' counts of digit d (two threads per digit, each half of the tiles, 8 loads in flight)
            const int d = tid & (kRadix - 1), half = tid >> 8;
            const int g0 = half ? Geff / 2 : 0, g1 = half ? Geff : Geff / 2;
            unsigned ex = 0, tot = 0;
            for (int g = g0; g < g1; g += 8) {
                unsigned long long v[8];
#pragma unroll
                for (int k = 0; k < 8; ++k)
                    v[k] = g + k < g1 ? ld_relaxed_u64(status + (size_t)(g + k) * kRadix + d) : 0ull;
#pragma unroll
                for (int k = 0; k < 8; ++k) {
                    if (g + k >= g1) break;
                    while ((unsigned)(v[k] >> 32) != tag) {
                        __nanosleep(20);
                        v[k] = ld_relaxed_u64(status + (size_t)(g + k) * kRadix + d);
                    }
                    tot += (unsigned)v[k];
                    if (g + k < b) ex += (unsigned)v[k];
                }
            }
            part[0][half][d] = ex;
            part[1][half][d] = tot;
            __syncthreads();
            // the digits' global starts: exclusive scan of the totals over digits
            const unsigned my_tot = tid < kRadix ? part[1][0][tid] + part[1][1][tid] : 0u;
            unsigned inc = my_tot;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const unsigned u = __shfl_up_sync(0xffffffffu, inc, o);
                if (lane >= o) inc += u;
            }
            if (lane == 31 && w < kRadix / 32) wsum[w] = inc;
            __syncthreads();
            if (tid < kRadix) {
                unsigned pre = 0;
                for (int k = 0; k < w; ++k) pre += wsum[k];
                run[tid] = pre + inc - my_tot + part[0][0][tid] + part[0][1][tid];
            }
            __syncthreads();
            // stable scatter of the tile, kSortThreads keys at a time
            for (int c0 = t0; c0 < t1; c0 += kSortThreads) {
                const int i = c0 + tid;
                const bool valid = i < t1;
                const unsigned long long key = valid ? sk[i] : 0ull;
                const int val = valid ? sv[i] : 0;
                const int dg = valid ? (int)((key >> sh) & 255u) : kRadix + lane;
                const unsigned peers = __match_any_sync(0xffffffffu, dg);
                const int rank = __popc(peers & ((1u << lane) - 1u));
                for (int e = tid; e < kSortWarps * kRadix; e += kSortThreads) (&wh[0][0])[e] = 0u;
                __syncthreads();
                if (valid && rank == 0) wh[w][dg] = (unsigned)__popc(peers);
                __syncthreads();
                if (tid < kRadix) {
                    unsigned r = run[tid];
#pragma unroll
                    for (int k = 0; k < kSortWarps; ++k) {
                        const unsigned c = wh[k][tid];
                        wh[k][tid] = r;
                        r += c;
                    }
                    run[tid] = r;
                }
                __syncthreads();
                if (valid) {
                    const unsigned pos = wh[w][dg] + (unsigned)rank;
                    if (last) {
                        out[pos] = tasks_u[val];
                    } else {
                        dk[pos] = key;
                        dv[pos] = val;
                    }
                }
                __syncthreads();
            }
        }
        if (!last) sort_grid_barrier(ctl);
    }
}

__global__ void gather_tasks_kernel(int nt, const int *__restrict__ order, const Task *__restrict__ in,
                                    Task *__restrict__ out) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < nt) out[i] = in[order[i]];
}

}  // namespace dev
}  // namespace afmm
