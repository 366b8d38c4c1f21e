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

// validation (one thread per leaf) + Interactions(t) = n_t * sum_{s in U(t)} n_s
__global__ void validate_interactions_kernel(int L, long long n, int max_leaf, const int *__restrict__ ls,
                                             const int *__restrict__ lc, const long long *__restrict__ uo,
                                             const int *__restrict__ ui, long long *__restrict__ I,
                                             int *__restrict__ err) {
    const int t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= L) return;
    int e = 0;
    const int c = lc[t];
    if (c < 1 || c > max_leaf) e |= kErrCount;
    if (t == 0 && ls[0] != 0) e |= kErrStart;
    if (t + 1 < L && ls[t + 1] != ls[t] + c) e |= kErrStart;
    if (t + 1 == L && (long long)ls[t] + c != n) e |= kErrCover;
    if (t == 0 && uo[0] != 0) e |= kErrOff;
    const long long b = uo[t], en = uo[t + 1], nnz = uo[L];
    long long src = 0;
    if (en < b || b < 0 || en > nnz) {               // (reads stay inside u_idx[0, u_off[L]))
        e |= kErrOff;
    } else {
        int prev = -1;
        for (long long u = b; u < en; ++u) {
            const int s = ui[u];
            if (s < 0 || s >= L) {
                e |= kErrIdx;
                break;
            }
            if (s <= prev) e |= kErrOrder;
            prev = s;
            src += lc[s];
        }
    }
    I[t] = (long long)c * src;
    if (e) atomicOr(err, e);
}

// Literal greedy cut (PAPER L16 SIII.C) from the inclusive prefix sums P[t] =
// sum_{u <= t} I(u): cut r+1 = 1 + first t >= cut_r whose running count
// P[t] - P[cut_r - 1] satisfies count * G >= total.  Single thread, G <= 64 binary searches.
__global__ void literal_cut_kernel(int L, int G, const long long *__restrict__ P, long long *__restrict__ split) {
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


// pass 1 over this rank's leaves [lo, lo+m): segment and slice counts, nsrc,
// bucket statistics (int64 atomics: order-independent)
__global__ void count_kernel(int m, int lo, const int *__restrict__ ls, const int *__restrict__ lc,
                             const long long *__restrict__ uo, const int *__restrict__ ui,
                             const long long *__restrict__ I, int *__restrict__ nseg, int *__restrict__ ntask,
                             long long *__restrict__ nsrc, unsigned long long *__restrict__ stats,
                             long long cap, unsigned short *__restrict__ plan, int4 *__restrict__ plan_hdr) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= m) return;
    const int t = lo + i;
    int segs = 0;
    bool self = false;
    long long src = 0;
    int prev_end = -1;                               // body end of the current run
    for (long long u = uo[t]; u < uo[t + 1]; ++u) {
        const int s = ui[u];
        src += lc[s];
        if (s == t) {
            self = true;
            continue;
        }
        if (segs == 0 || ls[s] != prev_end) ++segs;  // merges runs of consecutive leaves
        prev_end = ls[s] + lc[s];
    }
    nseg[i] = segs + (self ? 1 : 0);
    nsrc[i] = src;
    // the leaf's slice plan, kept for write_kernel (the DP runs once per leaf)
    int n_full = 0, full_m = 0;
    const int k = plan_slices(lc[t], src, cap, &n_full, &full_m, plan + (size_t)i * kMaxDpSlices);
    plan_hdr[i] = make_int4(n_full, full_m, k, 0);
    ntask[i] = n_full + k;
    atomicAdd(&stats[0], (unsigned long long)I[t]);
    atomicAdd(&stats[1 + bucket_of_d(lc[t])], (unsigned long long)I[t]);
    // the largest task cost (stats[9]): the sort keys need only its bits
    unsigned long long cmax = 0;
    for (int j = 0; j < n_full + k; ++j) {
        const unsigned long long c = (unsigned long long)slice_iters(src, plan_size(j, n_full, full_m,
                                                                                  plan + (size_t)i * kMaxDpSlices));
        cmax = c > cmax ? c : cmax;
    }
    atomicMax(&stats[9], cmax);
}

// pass 2: write segments (self first) and tasks with their LPT cost keys
__global__ void write_kernel(int m, int lo, const int *__restrict__ ls, const int *__restrict__ lc,
                             const long long *__restrict__ uo, const int *__restrict__ ui,
                             const int *__restrict__ seg_off, const int *__restrict__ task_off,
                             const int *__restrict__ ntask, const long long *__restrict__ nsrc,
                             Seg *__restrict__ segs, Task *__restrict__ tasks,
                             unsigned long long *__restrict__ keys, int *__restrict__ vals,
                             const unsigned short *__restrict__ plan, const int4 *__restrict__ plan_hdr,
                             unsigned long long cmax) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= m) return;
    const int t = lo + i;
    const int ts = ls[t], tn = lc[t];
    int w = seg_off[i];
    const int seg_begin = w;
    bool self = false;
    for (long long u = uo[t]; u < uo[t + 1]; ++u)
        if (ui[u] == t) self = true;
    if (self) segs[w++] = Seg{ts, tn};
    const int first_other = w;
    for (long long u = uo[t]; u < uo[t + 1]; ++u) {
        const int s = ui[u];
        if (s == t) continue;
        if (w > first_other && segs[w - 1].gstart + segs[w - 1].len == ls[s]) segs[w - 1].len += lc[s];
        else segs[w++] = Seg{ls[s], lc[s]};
    }
    const long long src = nsrc[i];
    const unsigned short *sz = plan + (size_t)i * kMaxDpSlices;           // count_kernel's plan
    const int4 hd = plan_hdr[i];
    const int n_full = hd.x, full_m = hd.y, k_dp = hd.z;
    for (int j = 0, a = 0; j < n_full + k_dp; a += plan_size(j, n_full, full_m, sz), ++j) {
        const int q = task_off[i] + j;
        const int cnt = plan_size(j, n_full, full_m, sz);
        tasks[q] = Task{ts + a, cnt, ts, self ? tn : 0, seg_begin, w - seg_begin, (int)src, 0};
        const unsigned long long cost = (unsigned long long)slice_iters(src, cnt);
        keys[q] = cmax - cost;                        // ascending = largest cost first; < 2^bits(cmax)
        vals[q] = q;
    }
}

__global__ void gather_tasks_kernel(int nt, const int *__restrict__ order, const Task *__restrict__ in,
                                    Task *__restrict__ out) {
    const int i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < nt) out[i] = in[order[i]];
}

}  // namespace dev
}  // namespace afmm
