// afmm_p2p.cu -- host side of the C ABI (include/afmm_p2p.h) and launches.
//
// Rows of SURVEY.md S8(a) implemented here: a1 body ingest (pack kernel),
// a2 tree ingest (validation, Interactions(t), segment merge, chunking, LPT
// order), a3 partition (literal greedy rule of PAPER L16 SIII.C + the
// incremental rebalance of L18 SIV.D), a5/a6 launch of the P2P kernel, a8
// cudaEvent timing (PAPER L20 SVII.A).  Rows a4/a7 (replication, gather) are
// collectives issued by the caller on the buffers this library exposes.
#include <algorithm>
#include <atomic>
#include <climits>
#include <cmath>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <numeric>
#include <string>
#include <vector>

#include <cuda.h>               // driver types for cuStreamWaitValue32 (resolved at run time)
#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>   // NVTX ranges (header-only; no-ops unless a profiler is attached)

#include "../../include/afmm_p2p.h"
#include "nccl_api.h"
#include "p2p_kernel.cuh"

using afmm::Seg;
using afmm::Task;

// NVTX range for the duration of a scope ("afmm.<entry point>"): nsys / ncu
// timelines show the library's host-side phases (SURVEY S5 tracing).
struct NvtxScope {
    explicit NvtxScope(const char *name) { nvtxRangePushA(name); }
    ~NvtxScope() { nvtxRangePop(); }
};

// Kernels of this library launched so far (afmm_launch_count): every <<<>>> site
// below counts itself; CUB's scans / sorts inside the device ingest are not ours
// and are not counted.  A pipelined eval whose input chain replays from a CUDA
// graph counts the graph's K pack kernels.
static std::atomic<long long> g_launches{0};
#define COUNT_LAUNCH(k) g_launches.fetch_add((k), std::memory_order_relaxed)

struct afmm_p2p {
    afmm_p2p_config cfg{};
    cudaStream_t stream = nullptr;
    bool own_stream = false;
    bool poisoned = false;
    std::string err;
    int num_sms = 148;
    int blocks_per_sm = 1;
    bool co_resident_pack = true;    // a pack_chunk_kernel block fits beside a streamed P2P CTA

    // bodies
    long long n = 0;
    float4 *d_bodies = nullptr;
    long long bodies_cap = 0;
    float *d_soa = nullptr;          // staging for host ingest (4n floats)
    long long soa_cap = 0;
    float *d_out = nullptr;          // eval_host outputs (4n floats)
    long long out_cap = 0;

    // tree (host copies)
    bool have_tree = false;
    int L = 0;
    std::vector<int> leaf_start, leaf_count;
    std::vector<long long> u_off;
    std::vector<int> u_idx;
    std::vector<long long> I;
    long long I_total = 0;

    // partition
    bool user_partition = false;
    bool have_coef = false;                 // per-bucket cost coefficients for set_tree's cut
    double coef[8] = {1, 1, 1, 1, 1, 1, 1, 1};
    std::vector<long long> leaf_split, body_split;

    // this rank's work list
    std::vector<Task> h_tasks;
    std::vector<Seg> h_segs;
    Task *d_tasks = nullptr;
    Seg *d_segs = nullptr;
    size_t tasks_cap = 0, segs_cap = 0;
    int *d_queue = nullptr;
    int n_tasks = 0;                        // tasks of the current work list (host or device built)
    bool tree_on_device = false;            // set_tree_device: no host mirror of the tree
    // device-ingest workspace (grow-only)
    std::vector<void *> dws_ptr;
    std::vector<size_t> dws_cap;
    long long rank_interactions = 0;
    long long bucket_inter[8] = {0};

    cudaEvent_t ev0 = nullptr, ev1 = nullptr;   // aliases of the newest ring entry
    static constexpr int kRing = 64;             // kernel-time history (afmm_p2p_kernel_times)
    cudaEvent_t ring0[kRing] = {}, ring1[kRing] = {};
    long long n_evals = 0;
    bool evaluated = false;
    bool last_zero_copy = false;                     // last eval_host_pipelined ran zero-copy
    bool last_streamed = false;                      // ... and overlapped its input chain with the kernel
    bool last_input_graph = false;                   // ... and replayed its input chain from a graph
    afmm_p2p_stats last{};

    // pipelined host evaluation (afmm_p2p_eval_host_pipelined): the rank's tasks
    // regrouped into P Morton-contiguous pieces, LPT order kept inside each
    bool pipe_valid = false;
    unsigned sort_epoch = 0;         // task_sort_kernel launches (tags its status words)
    bool sort_ready = false;         // its status words and barrier were cleared
    int pipe_P = 0;
    std::vector<int> pipe_off;                       // P + 1 offsets into d_ptasks
    std::vector<long long> pipe_need, pipe_lo, pipe_hi;   // bodies needed (prefix), output range per piece
    int pipe_K = 0;                                   // input chunks (streamed H2D)
    int last_tail_ctas = 0;                           // chunked eval: CTAs of the tail grid on the comm SMs
    afmm::Task *d_ptasks = nullptr;
    size_t ptasks_cap = 0;
    int *d_pqueue = nullptr;                         // kMaxPieces counters
    cudaStream_t s_in = nullptr, s_out = nullptr;
    void *wait_value32 = nullptr;                    // cuStreamWaitValue32 (driver entry point)
    void *write_value32 = nullptr;                   // cuStreamWriteValue32 (driver entry point)
    cudaEvent_t ev_start = nullptr, ev_in[64] = {}, ev_k[64] = {}, ev_done = nullptr, ev_in_done = nullptr;
    // zero-copy input chain (K pack launches + K stream writes) captured once as a
    // CUDA graph and replayed with one launch; re-captured when its key changes
    int *h_err = nullptr;                            // pinned: the input-wait timeout flag after an eval
    long long *h_rb = nullptr;                       // pinned: set_tree_device's one readback (RbSlot)
    size_t h_rb_len = 0;
    cudaGraphExec_t in_graph = nullptr;
    bool in_graph_off = false;                       // capture unsupported: direct launches
    const float *ig_src[4] = {nullptr, nullptr, nullptr, nullptr};
    long long ig_n = 0;
    int ig_K = 0;
    unsigned ig_m0 = 0;
    const void *ig_bodies = nullptr;

    // peer output windows (fused gather, afmm_p2p_set_peer_windows)
    int n_peers = 0;
    float *peers[afmm::kMaxWin - 1][4] = {};

    // library communicator (afmm_p2p_config.nccl_id) and the chunked replication
    ncclComm_t comm = nullptr;
    cudaStream_t s_comm = nullptr;                   // NCCL work + chunk publication
    cudaEvent_t ev_c0 = nullptr, ev_c1 = nullptr, ev_c2 = nullptr, ev_c3 = nullptr;
    bool bodies_pending = false;                     // set_bodies since the last eval: replicate in the next
    const float *def_soa[4] = {nullptr, nullptr, nullptr, nullptr};   // set_bodies_deferred: the root's SoA,
    bool deferred = false;                           // packed chunk by chunk inside the next chunked eval
    bool last_chunked = false;
    // device words: [0] chunk mask (epoch << 16 | mask), [1] wait-timeout flag, then
    // tspan[2] (u64, %globaltimer), kernel_ms[2] (double: own span, max over ranks)
    unsigned char *d_words = nullptr;
    double *h_kms = nullptr;                         // pinned: kernel_ms max over ranks
    int *h_cerr = nullptr;                           // pinned: the chunked eval's wait-timeout flag
    unsigned epoch = 0;                              // chunked evals so far (16 bits in the flag word)
    bool chunk_valid = false;                        // the plan below matches the work list
    int chunk_K = 0;
    std::vector<long long> chunk_bounds;             // K + 1 body offsets
    std::vector<int> chunk_order;                    // delivery order (permutation of 0..K-1)
    afmm::Task *d_ctasks = nullptr;                  // the work list in delivery order, need masks in piece
    size_t ctasks_cap = 0;
};

namespace {

afmm_status fail(afmm_p2p *h, afmm_status st, const char *fmt, ...) {
    if (h) {
        char buf[512];
        va_list ap;
        va_start(ap, fmt);
        vsnprintf(buf, sizeof(buf), fmt, ap);
        va_end(ap);
        h->err = buf;
        if (st == AFMM_ECUDA || st == AFMM_ENOMEM || st == AFMM_ENCCL) h->poisoned = true;   // (header: poisoned)
    }
    return st;
}

#define CUDA_TRY(h, call)                                                                    \
    do {                                                                                     \
        cudaError_t e_ = (call);                                                             \
        if (e_ != cudaSuccess)                                                               \
            return fail((h), e_ == cudaErrorMemoryAllocation ? AFMM_ENOMEM : AFMM_ECUDA,      \
                        "%s failed: %s (%s:%d)", #call, cudaGetErrorString(e_), __FILE__,    \
                        __LINE__);                                                           \
    } while (0)

#define CHECK_HANDLE(h)                                                                      \
    do {                                                                                     \
        if (!(h)) return AFMM_EINVAL;                                                        \
        if ((h)->poisoned) return AFMM_ESTATE;                                               \
    } while (0)

int bucket_of(int nt) {
    int b = 0;
    int cap = 8;
    while (nt > cap && b < 7) {
        cap <<= 1;
        ++b;
    }
    return b;
}

template <typename T>
afmm_status ensure_device(afmm_p2p *h, T **ptr, size_t &cap, size_t count) {
    if (count <= cap && *ptr) return AFMM_OK;
    if (*ptr) cudaFree(*ptr);
    *ptr = nullptr;
    cap = 0;
    // grow-only with 50% headroom: a time-stepping caller re-ingests slowly
    // growing trees every step, and cudaMalloc/cudaFree are device-wide syncs
    size_t c = std::max<size_t>(count, 1);
    c += c / 2;
    CUDA_TRY(h, cudaMalloc(reinterpret_cast<void **>(ptr), c * sizeof(T)));
    cap = c;
    return AFMM_OK;
}

int slice_world(const afmm_p2p *h) { return h->cfg.slice_world > 0 ? h->cfg.slice_world : h->cfg.world; }

// Bound on one in-kernel wait for an input chunk (P2PParams.wait_ns):
// AFMM_WAIT_MS (default 2000 ms) -- generous, it only matters when a producer died.
unsigned long long wait_ns(const afmm_p2p *) {
    static const unsigned long long ns = [] {
        const char *e = getenv("AFMM_WAIT_MS");
        const double ms = e ? atof(e) : 2000.0;
        return (unsigned long long)((ms > 0 ? ms : 2000.0) * 1e6);
    }();
    return ns;
}

// Can one pack_chunk_kernel block (the streamed input chain) run on an SM that
// holds a streamed P2P CTA?  From the built kernels' attributes: registers
// (allocated per warp in units of 256), threads, shared memory (+ the per-block
// reservation) and the block slots of one SM.  AFMM_PACK_CORESIDENT=0 forces "no"
// (tests of the fallback).
cudaError_t co_residency(int device, bool *ok) {
    cudaFuncAttributes fp{}, fk{};
    cudaError_t e = cudaFuncGetAttributes(&fp, afmm::p2p_stream_kernel_t<afmm::Gravity>);
    if (e == cudaSuccess) e = cudaFuncGetAttributes(&fk, afmm::pack_chunk_kernel);
    int regs = 0, smem = 0, thr = 0, rsv = 0, blk = 0;
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&regs, cudaDevAttrMaxRegistersPerMultiprocessor, device);
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&smem, cudaDevAttrMaxSharedMemoryPerMultiprocessor, device);
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&thr, cudaDevAttrMaxThreadsPerMultiProcessor, device);
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&rsv, cudaDevAttrReservedSharedMemoryPerBlock, device);
    if (e == cudaSuccess) e = cudaDeviceGetAttribute(&blk, cudaDevAttrMaxBlocksPerMultiprocessor, device);
    if (e != cudaSuccess) return e;
    const int kPackThreads = 128;
    auto warp_regs = [](int r) { return ((r + 7) / 8) * 8 * 32; };
    const long long rp = (long long)warp_regs(fp.numRegs) * afmm::kWarps, rk = (long long)warp_regs(fk.numRegs) * (kPackThreads / 32);
    const long long sp = (long long)fp.sharedSizeBytes + afmm::kDynSmem + rsv, sk = (long long)fk.sharedSizeBytes + rsv;
    const char *env = getenv("AFMM_PACK_CORESIDENT");
    *ok = rp + rk <= regs && sp + sk <= smem && afmm::kThreads + kPackThreads <= thr && blk >= 2 &&
          !(env && env[0] == '0');
    return cudaSuccess;
}

afmm_status set_device(afmm_p2p *h) {
    CUDA_TRY(h, cudaSetDevice(h->cfg.device));
    return AFMM_OK;
}

}  // namespace

// ------------------------------------------------------------------ host-only

extern "C" afmm_status afmm_interactions(int n_leaves, const int *leaf_count,
                                         const long long *u_off, const int *u_idx,
                                         long long *I) {
    if (n_leaves < 0 || (n_leaves > 0 && (!leaf_count || !u_off || !u_idx || !I)))
        return AFMM_EINVAL;
    for (int t = 0; t < n_leaves; ++t) {
        long long src = 0;
        for (long long u = u_off[t]; u < u_off[t + 1]; ++u) {
            const int s = u_idx[u];
            if (s < 0 || s >= n_leaves) return AFMM_EINVAL;
            src += leaf_count[s];
        }
        I[t] = (long long)leaf_count[t] * src;
    }
    return AFMM_OK;
}

extern "C" afmm_status afmm_partition_literal(int n_leaves, const long long *I, int G,
                                              long long *leaf_split) {
    if (n_leaves < 0 || G < 1 || !leaf_split || (n_leaves > 0 && !I)) return AFMM_EINVAL;
    __int128 total = 0;
    for (int t = 0; t < n_leaves; ++t) {
        if (I[t] < 0) return AFMM_EINVAL;
        total += I[t];
    }
    // walk leaves; once the running count c satisfies c*G >= total the next
    // leaf opens the next GPU (PAPER L16 SIII.C); the last GPU takes the rest
    int g = 0;
    __int128 c = 0;
    leaf_split[0] = 0;
    for (int t = 0; t < n_leaves; ++t) {
        c += I[t];
        if (g < G - 1 && c * G >= total) {
            leaf_split[++g] = t + 1;
            c = 0;
        }
    }
    for (int r = g + 1; r <= G; ++r) leaf_split[r] = n_leaves;
    return AFMM_OK;
}

extern "C" afmm_status afmm_partition_weighted(int n_leaves, const double *w, int G,
                                               long long *leaf_split) {
    if (n_leaves < 0 || G < 1 || !leaf_split || (n_leaves > 0 && !w)) return AFMM_EINVAL;
    long double total = 0;
    for (int t = 0; t < n_leaves; ++t) {
        if (!(w[t] >= 0.0) || !std::isfinite(w[t])) return AFMM_EINVAL;
        total += w[t];
    }
    int g = 0;
    long double c = 0;
    leaf_split[0] = 0;
    for (int t = 0; t < n_leaves; ++t) {
        c += w[t];
        if (g < G - 1 && c * G >= total) {
            leaf_split[++g] = t + 1;
            c = 0;
        }
    }
    for (int r = g + 1; r <= G; ++r) leaf_split[r] = n_leaves;
    return AFMM_OK;
}

// ------------------------------------------------------------------ handle

extern "C" afmm_status afmm_p2p_config_init(afmm_p2p_config *cfg) {
    if (!cfg) return AFMM_EINVAL;
    cfg->device = 0;
    cfg->rank = 0;
    cfg->world = 1;
    cfg->G = 1.0f;
    cfg->eps2 = 0.0f;
    cfg->max_leaf = AFMM_MAX_LEAF;
    cfg->stream = nullptr;
    cfg->law = AFMM_LAW_GRAVITY;
    cfg->mu = 1.0f;
    cfg->slice_world = 0;
    cfg->nccl_id = nullptr;
    cfg->comm_sms = 0;
    return AFMM_OK;
}

extern "C" afmm_status afmm_p2p_nccl_id(void *out128) {
    if (!out128) return AFMM_EINVAL;
    const afmm::NcclApi &nc = afmm::nccl_api();
    if (!nc.ok) return AFMM_ENOTSUP;
    ncclUniqueId id;
    static_assert(sizeof(id) == 128, "ncclUniqueId is 128 bytes");
    if (nc.GetUniqueId(&id) != ncclSuccess) return AFMM_ENCCL;
    std::memcpy(out128, &id, sizeof(id));
    return AFMM_OK;
}

namespace {
int comm_sms(const afmm_p2p *h) { return h->cfg.comm_sms > 0 ? h->cfg.comm_sms : 8; }

#define NCCL_TRY(h, call)                                                                    \
    do {                                                                                     \
        ncclResult_t r_ = (call);                                                            \
        if (r_ != ncclSuccess)                                                               \
            return fail((h), AFMM_ENCCL, "%s failed: %s (%s:%d)", #call,                     \
                        afmm::nccl_api().GetErrorString(r_), __FILE__, __LINE__);            \
    } while (0)

// The library communicator (afmm_p2p_config.nccl_id): world ranks, at most
// comm_sms CTAs per NCCL kernel (ncclConfig_t.maxCTAs, NCCL >= 2.28; earlier
// versions: ncclCommInitRank and NCCL's own channel count), its own stream.
afmm_status init_comm(afmm_p2p *h) {
    const afmm::NcclApi &nc = afmm::nccl_api();
    if (!nc.ok) return fail(h, AFMM_ENOTSUP, "create: nccl_id given but libnccl.so.2 could not be loaded");
    ncclUniqueId id;
    std::memcpy(&id, h->cfg.nccl_id, sizeof(id));
    if (nc.CommInitRankConfig && nc.version >= 22800) {
        ncclConfig_t c = NCCL_CONFIG_INITIALIZER;
        c.blocking = 1;
        c.minCTAs = 1;
        c.maxCTAs = comm_sms(h);
        NCCL_TRY(h, nc.CommInitRankConfig(&h->comm, h->cfg.world, id, h->cfg.rank, &c));
    } else {
        NCCL_TRY(h, nc.CommInitRank(&h->comm, h->cfg.world, id, h->cfg.rank));
    }
    CUDA_TRY(h, cudaStreamCreateWithFlags(&h->s_comm, cudaStreamNonBlocking));
    for (cudaEvent_t *e : {&h->ev_c0, &h->ev_c1, &h->ev_c2, &h->ev_c3})
        CUDA_TRY(h, cudaEventCreateWithFlags(e, cudaEventDisableTiming));
    CUDA_TRY(h, cudaMallocHost(&h->h_kms, sizeof(double)));
    return AFMM_OK;
}
}  // namespace

extern "C" const char *afmm_version(void) { return "afmm_p2p 0.1 sm_100a"; }

extern "C" afmm_status afmm_p2p_create(const afmm_p2p_config *cfg, afmm_p2p **out) {
    if (!out) return AFMM_EINVAL;
    *out = nullptr;
    if (!cfg) return AFMM_EINVAL;
    if (cfg->max_leaf > AFMM_MAX_LEAF) return AFMM_ENOTSUP;
    if (cfg->max_leaf < 1 || cfg->world < 1 || cfg->rank < 0 || cfg->rank >= cfg->world ||
        !std::isfinite(cfg->G) || !std::isfinite(cfg->eps2) || !(cfg->eps2 >= 0.0f) ||
        cfg->device < 0 || (cfg->law != AFMM_LAW_GRAVITY && cfg->law != AFMM_LAW_STOKESLET) ||
        !std::isfinite(cfg->mu) || !(cfg->mu > 0.0f) || cfg->slice_world < 0 || cfg->comm_sms < 0 ||
        cfg->comm_sms > 64)
        return AFMM_EINVAL;
    afmm_p2p *h = new (std::nothrow) afmm_p2p();
    if (!h) return AFMM_ENOMEM;
    h->cfg = *cfg;
    afmm_status st = set_device(h);
    if (st == AFMM_OK) {
        cudaError_t e = cudaSuccess;
        if (cfg->stream) {
            h->stream = static_cast<cudaStream_t>(cfg->stream);
        } else {
            e = cudaStreamCreateWithFlags(&h->stream, cudaStreamNonBlocking);
            h->own_stream = (e == cudaSuccess);
        }
        for (int i = 0; i < afmm_p2p::kRing && e == cudaSuccess; ++i) {
            e = cudaEventCreate(&h->ring0[i]);
            if (e == cudaSuccess) e = cudaEventCreate(&h->ring1[i]);
        }
        if (e == cudaSuccess) e = cudaMalloc(&h->d_queue, sizeof(int));
        if (e == cudaSuccess) e = cudaDeviceGetAttribute(&h->num_sms, cudaDevAttrMultiProcessorCount, cfg->device);
        if (e == cudaSuccess)
            e = cudaFuncSetAttribute(afmm::p2p_kernel_t<afmm::Gravity>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                     afmm::kDynSmem);
        if (e == cudaSuccess)
            e = cudaFuncSetAttribute(afmm::p2p_stream_kernel_t<afmm::Gravity>,
                                     cudaFuncAttributeMaxDynamicSharedMemorySize, afmm::kDynSmem);
        if (e == cudaSuccess)
            e = cudaFuncSetAttribute(afmm::p2p_kernel_t<afmm::Stokeslet>,
                                     cudaFuncAttributeMaxDynamicSharedMemorySize, afmm::kDynSmem);
        if (e == cudaSuccess)
            e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&h->blocks_per_sm, afmm::p2p_kernel_t<afmm::Gravity>,
                                                              afmm::kThreads, afmm::kDynSmem);
        if (e == cudaSuccess) e = co_residency(cfg->device, &h->co_resident_pack);
        if (e == cudaSuccess) e = cudaMalloc(&h->d_words, 64);
        if (e == cudaSuccess) e = cudaMemset(h->d_words, 0, 64);
        if (e == cudaSuccess) e = cudaMallocHost(&h->h_cerr, sizeof(int));
        if (e != cudaSuccess) st = fail(h, AFMM_ECUDA, "create: %s", cudaGetErrorString(e));
        if (h->blocks_per_sm < 1) h->blocks_per_sm = 1;
        if (h->h_cerr) *h->h_cerr = 0;
        if (st == AFMM_OK && cfg->nccl_id && cfg->law != AFMM_LAW_GRAVITY)
            st = fail(h, AFMM_ENOTSUP, "create: the library communicator replicates gravity bodies only");
        if (st == AFMM_OK && cfg->nccl_id) st = init_comm(h);
        h->cfg.nccl_id = nullptr;                   // the caller's buffer is not kept
    }
    if (st != AFMM_OK) {
        afmm_p2p_destroy(h);
        return st;
    }
    *out = h;
    return AFMM_OK;
}

extern "C" void afmm_p2p_destroy(afmm_p2p *h) {
    if (!h) return;
    cudaSetDevice(h->cfg.device);
    // a poisoned handle's communicator is aborted first (ncclCommAbort on fatal errors), so
    // outstanding NCCL work waiting on a failed peer does not block the stream synchronises below
    if (h->comm && h->poisoned && afmm::nccl_api().CommAbort) {
        afmm::nccl_api().CommAbort(h->comm);
        h->comm = nullptr;
    }
    if (h->stream) cudaStreamSynchronize(h->stream);
    cudaFree(h->d_bodies);
    cudaFree(h->d_soa);
    cudaFree(h->d_out);
    cudaFree(h->d_tasks);
    cudaFree(h->d_segs);
    for (void *q : h->dws_ptr) cudaFree(q);
    cudaFree(h->d_queue);
    cudaFree(h->d_ptasks);
    cudaFree(h->d_pqueue);
    if (h->s_comm) cudaStreamSynchronize(h->s_comm);
    if (h->comm) afmm::nccl_api().CommDestroy(h->comm);
    if (h->s_comm) cudaStreamDestroy(h->s_comm);
    for (cudaEvent_t e : {h->ev_c0, h->ev_c1, h->ev_c2, h->ev_c3})
        if (e) cudaEventDestroy(e);
    cudaFree(h->d_words);
    cudaFree(h->d_ctasks);
    if (h->h_kms) cudaFreeHost(h->h_kms);
    if (h->h_cerr) cudaFreeHost(h->h_cerr);
    if (h->s_in) cudaStreamSynchronize(h->s_in), cudaStreamDestroy(h->s_in);
    if (h->in_graph) cudaGraphExecDestroy(h->in_graph);
    if (h->h_err) cudaFreeHost(h->h_err);
    if (h->h_rb) cudaFreeHost(h->h_rb);
    if (h->s_out) cudaStreamSynchronize(h->s_out), cudaStreamDestroy(h->s_out);

    for (int i = 0; i < 64; ++i) {
        if (h->ev_in[i]) cudaEventDestroy(h->ev_in[i]);
        if (h->ev_k[i]) cudaEventDestroy(h->ev_k[i]);
    }
    if (h->ev_start) cudaEventDestroy(h->ev_start);
    if (h->ev_done) cudaEventDestroy(h->ev_done);
    if (h->ev_in_done) cudaEventDestroy(h->ev_in_done);
    for (int i = 0; i < afmm_p2p::kRing; ++i) {
        if (h->ring0[i]) cudaEventDestroy(h->ring0[i]);
        if (h->ring1[i]) cudaEventDestroy(h->ring1[i]);
    }
    if (h->own_stream && h->stream) cudaStreamDestroy(h->stream);
    delete h;
}

extern "C" const char *afmm_p2p_last_error(const afmm_p2p *h) {
    if (!h) return "null handle";
    return h->err.c_str();
}

extern "C" void *afmm_p2p_stream(const afmm_p2p *h) { return h ? (void *)h->stream : nullptr; }

// ------------------------------------------------------------------ bodies

static int words_of(const afmm_p2p *h) { return h->cfg.law == AFMM_LAW_STOKESLET ? 2 : 1; }

static afmm_status alloc_bodies(afmm_p2p *h, long long n) {
    // float4 per body: 1 (gravity) or 2 (Stokeslet), plus one trailer float4 holding the
    // equal-mass flag (travels with the packed array when it is broadcast)
    const long long words = n * words_of(h) + 1;
    if (words > h->bodies_cap) {
        cudaFree(h->d_bodies);
        h->d_bodies = nullptr;
        h->bodies_cap = 0;
        CUDA_TRY(h, cudaMalloc(&h->d_bodies, (size_t)words * sizeof(float4)));
        h->bodies_cap = words;
    }
    if (h->n != n) h->have_tree = false;   // a tree for another n is stale
    h->n = n;
    h->evaluated = false;
    return AFMM_OK;
}

// the equal-mass flag: first int of the trailer float4 after the packed bodies
static int *mass_flag(afmm_p2p *h) { return reinterpret_cast<int *>(h->d_bodies + h->n * words_of(h)); }

static afmm_status pack(afmm_p2p *h, const float *x, const float *y, const float *z,
                        const float *m) {
    const int threads = 256;
    long long blocks = std::min<long long>((h->n + threads - 1) / threads, (long long)h->num_sms * 16);
    int *flag = mass_flag(h);
    CUDA_TRY(h, cudaMemsetAsync(flag, 0, sizeof(int), h->stream));
    afmm::pack_bodies_kernel<<<(int)blocks, threads, 0, h->stream>>>(h->n, x, y, z, m, h->d_bodies, flag);
    COUNT_LAUNCH(1);
    CUDA_TRY(h, cudaGetLastError());
    return AFMM_OK;
}

// set_bodies_deferred (library communicator, root): the trailer -- "some mass differs
// from m_0" and m_0 -- from the caller's SoA before any chunk is broadcast, then each
// chunk packed right before its broadcast (pack_range_kernel), so the root's pack
// overlaps the replication instead of preceding it.
__global__ void mass_trailer_kernel(long long n, const float *__restrict__ m, int *__restrict__ trailer) {
    const float m0 = m[0];
    if (blockIdx.x == 0 && threadIdx.x == 0) trailer[1] = __float_as_int(m0);
    bool diff = false;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        diff |= m[i] != m0;
    if (__any_sync(0xffffffffu, diff) && (threadIdx.x & 31) == 0) atomicOr(trailer, -1);
}
__global__ void pack_range_kernel(long long n, const float *__restrict__ x, const float *__restrict__ y,
                                  const float *__restrict__ z, const float *__restrict__ m, float4 *__restrict__ out) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
        out[i] = make_float4(x[i], y[i], z[i], m[i]);
}
// a deferred pack that something other than the chunked eval needs now: pack in full
static afmm_status flush_deferred(afmm_p2p *h) {
    if (!h->deferred) return AFMM_OK;
    h->deferred = false;
    return pack(h, h->def_soa[0], h->def_soa[1], h->def_soa[2], h->def_soa[3]);
}

extern "C" afmm_status afmm_p2p_set_bodies_deferred(afmm_p2p *h, long long n, const float *x, const float *y,
                                                    const float *z, const float *m) {
    NvtxScope nvtx_("afmm.set_bodies_deferred");
    CHECK_HANDLE(h);
    if (h->cfg.law != AFMM_LAW_GRAVITY) return fail(h, AFMM_EINVAL, "set_bodies_deferred: handle law is not gravity");
    if (n < 1 || n >= (1LL << 31)) return fail(h, AFMM_EINVAL, "set_bodies_deferred: n=%lld out of [1, 2^31)", n);
    if (!x || !y || !z || !m) return fail(h, AFMM_EINVAL, "set_bodies_deferred: null pointer");
    afmm_status st = set_device(h);
    if (st) return st;
    if ((st = alloc_bodies(h, n))) return st;
    if (!h->comm || h->cfg.rank != 0) {                     // nothing to overlap: pack now
        h->deferred = false;
        h->bodies_pending = h->comm != nullptr;
        return pack(h, x, y, z, m);
    }
    h->def_soa[0] = x;
    h->def_soa[1] = y;
    h->def_soa[2] = z;
    h->def_soa[3] = m;
    h->deferred = true;
    h->bodies_pending = true;
    return AFMM_OK;
}

extern "C" afmm_status afmm_p2p_set_bodies(afmm_p2p *h, long long n, const float *x,
                                           const float *y, const float *z, const float *m) {
    NvtxScope nvtx_("afmm.set_bodies");
    CHECK_HANDLE(h);
    if (h->cfg.law != AFMM_LAW_GRAVITY) return fail(h, AFMM_EINVAL, "set_bodies: handle law is not gravity");
    if (n < 1 || n >= (1LL << 31)) return fail(h, AFMM_EINVAL, "set_bodies: n=%lld out of [1, 2^31)", n);
    const int nn = (x != nullptr) + (y != nullptr) + (z != nullptr) + (m != nullptr);
    if (nn != 0 && nn != 4) return fail(h, AFMM_EINVAL, "set_bodies: pass all four pointers or none");
    afmm_status st = set_device(h);
    if (st) return st;
    if ((st = alloc_bodies(h, n))) return st;
    h->bodies_pending = h->comm != nullptr;          // the next eval replicates them (library communicator)
    h->deferred = false;
    if (nn == 4) return pack(h, x, y, z, m);
    // allocate only: the equal-mass flag reads "unequal" until a full-buffer
    // broadcast (afmm_p2p_bodies_buffer, trailer included) brings the root's
    CUDA_TRY(h, cudaMemsetAsync(mass_flag(h), 0xff, sizeof(int), h->stream));   // -1: "unequal"
    return AFMM_OK;
}

extern "C" afmm_status afmm_p2p_set_bodies_host(afmm_p2p *h, long long n, const float *x,
                                                const float *y, const float *z, const float *m) {
    NvtxScope nvtx_("afmm.set_bodies_host");
    CHECK_HANDLE(h);
    if (h->cfg.law != AFMM_LAW_GRAVITY) return fail(h, AFMM_EINVAL, "set_bodies_host: handle law is not gravity");
    if (n < 1 || n >= (1LL << 31)) return fail(h, AFMM_EINVAL, "set_bodies_host: n=%lld out of [1, 2^31)", n);
    if (!x || !y || !z || !m) return fail(h, AFMM_EINVAL, "set_bodies_host: null pointer");
    afmm_status st = set_device(h);
    if (st) return st;
    if ((st = alloc_bodies(h, n))) return st;
    h->bodies_pending = h->comm != nullptr;
    h->deferred = false;
    if (4 * n > h->soa_cap) {
        cudaFree(h->d_soa);
        h->d_soa = nullptr;
        h->soa_cap = 0;
        CUDA_TRY(h, cudaMalloc(&h->d_soa, (size_t)(4 * n) * sizeof(float)));
        h->soa_cap = 4 * n;
    }
    const size_t b = (size_t)n * sizeof(float);
    CUDA_TRY(h, cudaMemcpyAsync(h->d_soa + 0 * n, x, b, cudaMemcpyHostToDevice, h->stream));
    CUDA_TRY(h, cudaMemcpyAsync(h->d_soa + 1 * n, y, b, cudaMemcpyHostToDevice, h->stream));
    CUDA_TRY(h, cudaMemcpyAsync(h->d_soa + 2 * n, z, b, cudaMemcpyHostToDevice, h->stream));
    CUDA_TRY(h, cudaMemcpyAsync(h->d_soa + 3 * n, m, b, cudaMemcpyHostToDevice, h->stream));
    if ((st = pack(h, h->d_soa, h->d_soa + n, h->d_soa + 2 * n, h->d_soa + 3 * n))) return st;
    CUDA_TRY(h, cudaStreamSynchronize(h->stream));
    return AFMM_OK;
}

extern "C" afmm_status afmm_p2p_set_bodies_stokeslet(afmm_p2p *h, long long n, const float *x, const float *y,
                                                     const float *z, const float *fx, const float *fy,
                                                     const float *fz) {
    CHECK_HANDLE(h);
    if (h->cfg.law != AFMM_LAW_STOKESLET)
        return fail(h, AFMM_EINVAL, "set_bodies_stokeslet: handle law is not the Stokeslet");
    if (n < 1 || n >= (1LL << 31)) return fail(h, AFMM_EINVAL, "set_bodies_stokeslet: n=%lld out of [1, 2^31)", n);
    const int nn = !!x + !!y + !!z + !!fx + !!fy + !!fz;
    if (nn != 0 && nn != 6) return fail(h, AFMM_EINVAL, "set_bodies_stokeslet: pass all six pointers or none");
    afmm_status st = set_device(h);
    if (st) return st;
    if ((st = alloc_bodies(h, n))) return st;
    if (nn == 0) return AFMM_OK;
    const int threads = 256;
    long long blocks = std::min<long long>((n + threads - 1) / threads, (long long)h->num_sms * 16);
    afmm::pack_stokeslet_kernel<<<(int)blocks, threads, 0, h->stream>>>(n, x, y, z, fx, fy, fz, h->d_bodies);
    COUNT_LAUNCH(1);
    CUDA_TRY(h, cudaGetLastError());
    return AFMM_OK;
}

extern "C" afmm_status afmm_p2p_bodies_buffer(afmm_p2p *h, void **dev_ptr, long long *bytes) {
    CHECK_HANDLE(h);
    if (afmm_status st0 = flush_deferred(h)) return st0;
    if (!h->d_bodies || h->n < 1) return fail(h, AFMM_ESTATE, "bodies_buffer: no bodies set");
    if (dev_ptr) *dev_ptr = h->d_bodies;
    if (bytes) *bytes = (h->n * words_of(h) + 1) * (long long)sizeof(float4);   // + the flag trailer
    return AFMM_OK;
}

// ------------------------------------------------------------------ tree / work list

static void compute_body_split(afmm_p2p *h) {
    const int W = h->cfg.world;
    h->body_split.assign(W + 1, 0);
    for (int r = 0; r <= W; ++r) {
        const long long ls = h->leaf_split[r];
        h->body_split[r] = (ls >= h->L) ? h->n : h->leaf_start[ls];
    }
}

#include "worklist.inc"
#include "worklist_dev.cuh"

// The host work-list builder (worklist.inc): validation, Interactions(t), the
// partition and this rank's tasks computed on the CPU.  The reference the device
// ingest is tested against (AFMM_HOST_INGEST=1 selects it for afmm_p2p_set_tree).
static afmm_status set_tree_host_builder(afmm_p2p *h, int n_leaves, const int *leaf_start, const int *leaf_count,
                                         const long long *u_off, const int *u_idx) {
    // leaves must tile [0, n) exactly, 1 <= count <= max_leaf
    long long expect = 0;
    for (int t = 0; t < n_leaves; ++t) {
        if (leaf_start[t] != expect)
            return fail(h, AFMM_EINVAL, "set_tree: leaf %d starts at %d, expected %lld", t, leaf_start[t], expect);
        if (leaf_count[t] < 1 || leaf_count[t] > h->cfg.max_leaf)
            return fail(h, AFMM_EINVAL, "set_tree: leaf %d count %d outside [1, max_leaf=%d]", t,
                        leaf_count[t], h->cfg.max_leaf);
        expect += leaf_count[t];
    }
    if (expect != h->n) return fail(h, AFMM_EINVAL, "set_tree: leaves cover %lld bodies, n=%lld", expect, h->n);
    if (u_off[0] != 0) return fail(h, AFMM_EINVAL, "set_tree: u_off[0]=%lld != 0", u_off[0]);
    for (int t = 0; t < n_leaves; ++t)
        if (u_off[t + 1] < u_off[t]) return fail(h, AFMM_EINVAL, "set_tree: u_off not monotone at %d", t);
    const long long nnz = u_off[n_leaves];
    if (nnz > 0 && !u_idx) return fail(h, AFMM_EINVAL, "set_tree: u_idx is null");
    for (int t = 0; t < n_leaves; ++t) {
        for (long long u = u_off[t]; u < u_off[t + 1]; ++u) {
            if (u_idx[u] < 0 || u_idx[u] >= n_leaves)
                return fail(h, AFMM_EINVAL, "set_tree: u_idx[%lld]=%d outside [0,%d)", u, u_idx[u], n_leaves);
            if (u > u_off[t] && u_idx[u] <= u_idx[u - 1])
                return fail(h, AFMM_EINVAL, "set_tree: row %d of u_idx not strictly ascending", t);
        }
    }
    afmm_status st = set_device(h);
    if (st) return st;
    h->L = n_leaves;
    h->leaf_start.assign(leaf_start, leaf_start + n_leaves);
    h->leaf_count.assign(leaf_count, leaf_count + n_leaves);
    h->u_off.assign(u_off, u_off + n_leaves + 1);
    h->u_idx.assign(u_idx, u_idx + nnz);
    h->I.assign(n_leaves, 0);
    afmm_interactions(n_leaves, leaf_count, u_off, u_idx, h->I.data());
    h->I_total = 0;
    for (long long v : h->I) h->I_total += v;
    const int W = h->cfg.world;
    if (!h->user_partition || (long long)h->leaf_split.size() != W + 1 || h->leaf_split[W] != n_leaves) {
        h->user_partition = false;
        h->leaf_split.assign(W + 1, 0);
        if (h->have_coef && W > 1) {        // incremental adjustment carried across trees (L18 SIV.D)
            std::vector<double> w(n_leaves);
            for (int t = 0; t < n_leaves; ++t) w[t] = (double)h->I[t] * h->coef[bucket_of(leaf_count[t])];
            afmm_partition_weighted(n_leaves, w.data(), W, h->leaf_split.data());
        } else {
            afmm_partition_literal(n_leaves, h->I.data(), W, h->leaf_split.data());
        }
    }
    compute_body_split(h);
    h->have_tree = true;
    return build_worklist(h);
}


// grow-only device workspace for set_tree_device
template <typename T>
static afmm_status dws(afmm_p2p *h, int slot, T **p, size_t count) {
    const size_t bytes = std::max<size_t>(count, 1) * sizeof(T);
    if ((size_t)slot >= h->dws_ptr.size()) {
        h->dws_ptr.resize(slot + 1, nullptr);
        h->dws_cap.resize(slot + 1, 0);
    }
    if (h->dws_cap[slot] < bytes) {
        cudaFree(h->dws_ptr[slot]);
        h->dws_ptr[slot] = nullptr;
        h->dws_cap[slot] = 0;
        const size_t want = bytes + bytes / 2;
        CUDA_TRY(h, cudaMalloc(&h->dws_ptr[slot], want));
        h->dws_cap[slot] = want;
    }
    *p = static_cast<T *>(h->dws_ptr[slot]);
    return AFMM_OK;
}
static size_t slot_capacity(const afmm_p2p *h, int slot) {
    return (size_t)slot < h->dws_cap.size() ? h->dws_cap[slot] : 0;
}

__global__ void body_split_kernel(int G, int L, long long n, const long long *__restrict__ split,
                                  const int *__restrict__ ls, long long *__restrict__ bsplit) {
    const int r = blockIdx.x * blockDim.x + threadIdx.x;
    if (r <= G) bsplit[r] = split[r] >= L ? n : ls[split[r]];
}

enum DwsSlot { sI, sP, sW, sPW, sSplit, sNseg, sNsrc, sSegOff, sStats, sKeys, sVals, sKeys2,
               sVals2, sTasksU, sCoef, sTmp, sBsplit, sPlan, sPlanHdr, sNnz,
               sOwnLS, sOwnLC, sOwnUO, sOwnUI,               // the handle's own copy of the tree (re-ingest)
               sSortStat, sSortCtl, sNsegAll, sNsrcAll, sRb, sNtEff };              // task_sort_kernel's digit totals, status words, barrier

// Device ingest (validation, Interactions(t), partition, this rank's work list)
// of the tree arrays ls/lc/uo/ui in device memory.  keep: afterwards also copy
// them into the handle's own buffers (sOwn*), from which set_partition /
// rebalance re-ingest the same tree (the caller's arrays may be gone by then).
//
// Everything is enqueued back to back and the host synchronises ONCE, at the end
// (round 1: nine host round trips).  The kernels read what the host used to read
// back -- this rank's leaf range (split), the task cap (from the total P[L-1]),
// the list sizes -- on the device; a failed validation gates every later kernel
// (no read through an invalid index), and the work list is written into the
// current capacities: when it does not fit (first ingest, a grown tree), the
// host grows them after the sync and enqueues the list writing again.
enum RbSlot { rbErr, rbOverflow, rbNsegs, rbNt, rbItot, rbNnz, rbStats, rbSplit = rbStats + 10 };
enum : long long { kOvSegs = 1, kOvTasks = 2, kOvOwnUI = 4 };
namespace dev_ingest {
__global__ void collect_kernel(int L, int W, int r, const long long *__restrict__ split,
                               const long long *__restrict__ bsplit, const long long *__restrict__ P,
                               const long long *__restrict__ uo, const unsigned long long *__restrict__ off2,
                               const unsigned long long *__restrict__ stats,
                               const int *__restrict__ err, long long segs_cap, long long tasks_cap,
                               long long *__restrict__ rb, int *__restrict__ nt_eff) {
    if (threadIdx.x != 0 || blockIdx.x != 0) return;
    const int e = *err;
    const long long m = split[r + 1] - split[r];
    const long long nsegs = e ? 0 : (long long)(unsigned)off2[m], nt = e ? 0 : (long long)(off2[m] >> 32);
    const long long ov = (nsegs > segs_cap ? kOvSegs : 0) | (nt > tasks_cap ? kOvTasks : 0);
    rb[rbErr] = e;
    rb[rbOverflow] = ov;
    rb[rbNsegs] = nsegs;
    rb[rbNt] = nt;
    rb[rbItot] = P[L - 1];
    rb[rbNnz] = uo[L];
    for (int k = 0; k < 10; ++k) rb[rbStats + k] = (long long)stats[k];
    for (int k = 0; k <= W; ++k) {
        rb[rbSplit + k] = split[k];
        rb[rbSplit + W + 1 + k] = bsplit[k];
    }
    *nt_eff = (e || ov) ? 0 : (int)nt;                      // gates write_kernel and the sort
}
// the tree into the handle's own buffers: leaf arrays, and the U-list indices (capacity
// cap; nnz = uo[L] on the device)
__global__ void copy_ui_kernel(int L, const long long *__restrict__ uo, const int *__restrict__ src,
                               int *__restrict__ dst, long long cap, const int *__restrict__ err,
                               long long *__restrict__ rb, const int *__restrict__ ls, const int *__restrict__ lc,
                               int *__restrict__ ols, int *__restrict__ olc, long long *__restrict__ ouo) {
    const long long g0 = blockIdx.x * (long long)blockDim.x + threadIdx.x, gs = (long long)gridDim.x * blockDim.x;
    for (long long i = g0; i <= L; i += gs) {               // the leaf arrays too (one kernel, not three copies)
        if (i < L) {
            ols[i] = ls[i];
            olc[i] = lc[i];
        }
        ouo[i] = uo[i];
    }
    if (*err) return;
    const long long nnz = uo[L];
    if (nnz > cap) {
        if (blockIdx.x == 0 && threadIdx.x == 0) atomicOr((unsigned long long *)&rb[rbOverflow], (unsigned long long)kOvOwnUI);
        return;
    }
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < nnz; i += (long long)gridDim.x * blockDim.x)
        dst[i] = src[i];
}
}  // namespace dev_ingest

static afmm_status ingest(afmm_p2p *h, int n_leaves, const int *leaf_start, const int *leaf_count,
                          const long long *u_off, const int *u_idx, bool keep) {
    using namespace afmm;
    afmm_status st;
    cudaStream_t s = h->stream;
    const int L = n_leaves, W = h->cfg.world, r = h->cfg.rank, TH = 256;
    auto grid = [&](long long m) { return (int)std::max<long long>(1, (m + TH - 1) / TH); };
    long long *I, *P, *split, *nsrc, *bsplit, *nsrc_all, *rb;
    unsigned short *plan;
    int4 *plan_hdr;
    int *err, *nseg_all, *nt_eff;
    unsigned long long *nst, *off2;
    unsigned long long *stats;
    const size_t rb_len = (size_t)rbSplit + 2 * (W + 1);
    if ((st = dws(h, sI, &I, L)) || (st = dws(h, sP, &P, L)) || (st = dws(h, sSplit, &split, W + 1)) ||
        (st = dws(h, sBsplit, &bsplit, W + 1)) ||
        (st = dws(h, sNsegAll, &nseg_all, L)) || (st = dws(h, sNsrcAll, &nsrc_all, L)) ||
        (st = dws(h, sNseg, &nst, (size_t)L + 1)) || (st = dws(h, sNsrc, &nsrc, (size_t)L + 1)) ||
        (st = dws(h, sSegOff, &off2, (size_t)L + 1)) || (st = dws(h, sStats, &stats, 11)) ||
        (st = dws(h, sPlan, &plan, (size_t)(L + 1) * afmm::kMaxDpSlices)) ||
        (st = dws(h, sPlanHdr, &plan_hdr, (size_t)L + 1)) || (st = dws(h, sRb, &rb, rb_len)) ||
        (st = dws(h, sNtEff, &nt_eff, 1)))
        return st;
    if (h->h_rb_len < rb_len) {                     // pinned: the one readback is an async copy
        if (h->h_rb) cudaFreeHost(h->h_rb);
        h->h_rb = nullptr;
        h->h_rb_len = 0;
        CUDA_TRY(h, cudaMallocHost(&h->h_rb, rb_len * sizeof(long long)));
        h->h_rb_len = rb_len;
    }
    // 1. validation + Interactions(t) + per-leaf segment counts and source totals
    err = reinterpret_cast<int *>(stats + 10);     // the error flags share the stats' reset
    CUDA_TRY(h, cudaMemsetAsync(stats, 0, 11 * sizeof(unsigned long long), s));
    dev::validate_interactions_kernel<<<grid(32LL * L), TH, 0, s>>>(L, h->n, h->cfg.max_leaf, leaf_start,
                                                                   leaf_count, u_off, u_idx, I, nseg_all, nsrc_all,
                                                                   err);
    COUNT_LAUNCH(1);
    CUDA_TRY(h, cudaGetLastError());
    bool clear_user = false;                        // applied once the tree is known valid
    // 2. partition (literal rule, or the per-bucket coefficients of the last step)
    {
        size_t tb = 0;
        CUDA_TRY(h, cub::DeviceScan::InclusiveSum(nullptr, tb, I, P, L, s));
        char *tmp;
        if ((st = dws(h, sTmp, &tmp, tb))) return st;
        CUDA_TRY(h, cub::DeviceScan::InclusiveSum(tmp, tb, I, P, L, s));
    }
    bool literal = false;
    if (h->user_partition && (long long)h->leaf_split.size() == W + 1 && h->leaf_split[W] == L) {
        CUDA_TRY(h, cudaMemcpyAsync(split, h->leaf_split.data(), (W + 1) * sizeof(long long),
                                    cudaMemcpyHostToDevice, s));
    } else if (h->have_coef && W > 1) {
        double *w, *pw, *coef;
        if ((st = dws(h, sW, &w, L)) || (st = dws(h, sPW, &pw, L)) || (st = dws(h, sCoef, &coef, 8))) return st;
        CUDA_TRY(h, cudaMemcpyAsync(coef, h->coef, 8 * sizeof(double), cudaMemcpyHostToDevice, s));
        dev::weights_kernel<<<grid(L), TH, 0, s>>>(L, leaf_count, I, coef, w);
        COUNT_LAUNCH(1);
        size_t tb = 0;
        CUDA_TRY(h, cub::DeviceScan::InclusiveSum(nullptr, tb, w, pw, L, s));
        char *tmp;
        if ((st = dws(h, sTmp, &tmp, tb))) return st;
        CUDA_TRY(h, cub::DeviceScan::InclusiveSum(tmp, tb, w, pw, L, s));
        dev::weighted_cut_kernel<<<1, 1, 0, s>>>(L, W, pw, split);
        COUNT_LAUNCH(1);
        clear_user = true;
    } else {
        literal = true;
        dev::literal_cut_kernel<<<1, 1, 0, s>>>(L, W, P, split, h->n, leaf_start, bsplit);   // + the body split
        COUNT_LAUNCH(1);
        clear_user = true;
    }
    CUDA_TRY(h, cudaGetLastError());
    if (!literal) {
        body_split_kernel<<<(W + 1 + 63) / 64, 64, 0, s>>>(W, L, h->n, split, leaf_start, bsplit);
        COUNT_LAUNCH(1);
    }
    // 3. this rank's segment / slice counts (leaves split[r] .. split[r+1], read on the device)
    dev::count_kernel<<<grid((long long)L + 1), TH, 0, s>>>(L, r, split, P, slice_world(h),
                                                           (long long)h->num_sms * h->blocks_per_sm * afmm::kWarps,
                                                           err, leaf_count, nseg_all, nsrc_all, I, nst, nsrc,
                                                           stats, plan, plan_hdr);
    COUNT_LAUNCH(1);
    CUDA_TRY(h, cudaGetLastError());
    {
        size_t tb = 0;
        CUDA_TRY(h, cub::DeviceScan::ExclusiveSum(nullptr, tb, nst, off2, L + 1, s));
        char *tmp;
        if ((st = dws(h, sTmp, &tmp, tb))) return st;
        CUDA_TRY(h, cub::DeviceScan::ExclusiveSum(tmp, tb, nst, off2, L + 1, s));   // segment | task offsets
    }
    // 4. the lists, into the current capacities (a first guess from L when there are none)
    if ((st = ensure_device(h, &h->d_segs, h->segs_cap, std::max<size_t>(h->segs_cap, (size_t)12 * L))) ||
        (st = ensure_device(h, &h->d_tasks, h->tasks_cap, std::max<size_t>(h->tasks_cap, (size_t)4 * L))))
        return st;
    auto write_lists = [&]() -> afmm_status {
        const size_t tcap = h->tasks_cap;
        Task *tasks_u;
        unsigned long long *keys, *keys2;
        int *vals, *vals2;
        afmm_status s2;
        if ((s2 = dws(h, sTasksU, &tasks_u, tcap)) || (s2 = dws(h, sKeys, &keys, tcap)) ||
            (s2 = dws(h, sVals, &vals, tcap)) || (s2 = dws(h, sKeys2, &keys2, tcap)) ||
            (s2 = dws(h, sVals2, &vals2, tcap)))
            return s2;
        dev_ingest::collect_kernel<<<1, 1, 0, s>>>(L, W, r, split, bsplit, P, u_off, off2, stats, err,
                                                   (long long)h->segs_cap, (long long)tcap, rb, nt_eff);
        COUNT_LAUNCH(1);
        dev::write_kernel<<<grid(32LL * L), TH, 0, s>>>(r, split, nt_eff, leaf_start, leaf_count, u_off, u_idx,
                                                       off2, nsrc, h->d_segs, tasks_u, keys, vals, plan,
                                                       plan_hdr, stats + 9);
        COUNT_LAUNCH(1);
        CUDA_TRY(h, cudaGetLastError());
        // keys = cmax - cost < 2^bits(cmax): stable sort, ascending (task_sort_kernel)
        const int G = std::max(1, h->num_sms);
        unsigned long long *sstat;
        dev::SortCtl *sctl;
        if ((s2 = dws(h, sSortStat, &sstat, (size_t)G * dev::kRadix)) || (s2 = dws(h, sSortCtl, &sctl, 1))) return s2;
        unsigned epoch = ++h->sort_epoch & 0x7ffffffu;
        if (!h->sort_ready || epoch == 0) {      // fresh status words (the tags must not match stale ones)
            CUDA_TRY(h, cudaMemsetAsync(sstat, 0, (size_t)G * dev::kRadix * sizeof(unsigned long long), s));
            CUDA_TRY(h, cudaMemsetAsync(sctl, 0, sizeof(dev::SortCtl), s));
            h->sort_ready = true;
            if (epoch == 0) epoch = ++h->sort_epoch & 0x7ffffffu;
        }
        const int *ntp = nt_eff;
        const unsigned long long *cmax_ptr = stats + 9;
        Task *out = h->d_tasks;
        void *args[] = {&ntp, &cmax_ptr, &keys, &vals, &keys2, &vals2, &tasks_u, &out, &sstat, &epoch, &sctl};
        CUDA_TRY(h, cudaLaunchCooperativeKernel((const void *)dev::task_sort_kernel, G, dev::kSortThreads, args, 0, s));
        COUNT_LAUNCH(1);
        return AFMM_OK;
    };
    if ((st = write_lists())) return st;
    // 5. the handle's own copy of the tree (set_partition / rebalance re-ingest it)
    int *oui = nullptr, *ols = nullptr, *olc = nullptr;
    long long *ouo = nullptr;
    auto copy_ui = [&](size_t cap) -> afmm_status {
        if (afmm_status s2 = dws(h, sOwnUI, &oui, cap)) return s2;
        dev_ingest::copy_ui_kernel<<<h->num_sms * 4, TH, 0, s>>>(L, u_off, u_idx, oui, (long long)cap, err, rb,
                                                                 leaf_start, leaf_count, ols, olc, ouo);
        COUNT_LAUNCH(1);
        CUDA_TRY(h, cudaGetLastError());
        return AFMM_OK;
    };
    if (keep) {
        if ((st = dws(h, sOwnLS, &ols, L)) || (st = dws(h, sOwnLC, &olc, L)) || (st = dws(h, sOwnUO, &ouo, L + 1)))
            return st;
        const size_t have = slot_capacity(h, sOwnUI) / sizeof(int);
        if ((st = copy_ui(std::max<size_t>(have, (size_t)32 * L)))) return st;
    }
    // 6. the one readback
    long long *hb = h->h_rb;
    CUDA_TRY(h, cudaMemcpyAsync(hb, rb, rb_len * sizeof(long long), cudaMemcpyDeviceToHost, s));
    CUDA_TRY(h, cudaStreamSynchronize(s));
    if (hb[rbErr])
        return fail(h, AFMM_EINVAL, "set_tree: invalid tree (flags 0x%x: 1 start, 2 count, 4 cover, "
                                    "8 u_off, 16 u_idx range, 32 row order)", (int)hb[rbErr]);
    if (hb[rbOverflow] & (kOvSegs | kOvTasks)) {   // the lists did not fit: grow, write them again
        if ((st = ensure_device(h, &h->d_segs, h->segs_cap, (size_t)hb[rbNsegs])) ||
            (st = ensure_device(h, &h->d_tasks, h->tasks_cap, (size_t)hb[rbNt])))
            return st;
        const long long own_ov = hb[rbOverflow] & kOvOwnUI;
        if ((st = write_lists())) return st;
        if (keep && own_ov && (st = copy_ui((size_t)hb[rbNnz]))) return st;
        CUDA_TRY(h, cudaMemcpyAsync(hb, rb, rb_len * sizeof(long long), cudaMemcpyDeviceToHost, s));
        CUDA_TRY(h, cudaStreamSynchronize(s));
        if (hb[rbOverflow] & (kOvSegs | kOvTasks))
            return fail(h, AFMM_ECUDA, "set_tree: work list still overflowing after growth");
    } else if (keep && (hb[rbOverflow] & kOvOwnUI)) {
        if ((st = copy_ui((size_t)hb[rbNnz]))) return st;  // (ordered before any later use)
    }
    if (clear_user) h->user_partition = false;
    h->leaf_split.assign(hb + rbSplit, hb + rbSplit + W + 1);
    h->body_split.assign(hb + rbSplit + W + 1, hb + rbSplit + 2 * (W + 1));
    h->I_total = hb[rbItot];
    h->n_tasks = (int)hb[rbNt];
    h->pipe_valid = false;
    h->chunk_valid = false;
    h->L = L;
    h->rank_interactions = hb[rbStats + 0];
    for (int b = 0; b < 8; ++b) h->bucket_inter[b] = hb[rbStats + 1 + b];
    h->tree_on_device = true;
    h->have_tree = true;
    h->h_tasks.clear();
    h->h_segs.clear();
    h->leaf_start.clear();
    h->leaf_count.clear();
    h->u_off.clear();
    h->u_idx.clear();
    h->I.clear();
    h->evaluated = false;
    return AFMM_OK;
}

// re-ingest the current tree from the handle's own copy (after a partition change)
static afmm_status reingest(afmm_p2p *h) {
    int *ols, *olc, *oui;
    long long *ouo;
    afmm_status st;
    const int L = h->L;
    if ((st = dws(h, sOwnLS, &ols, L)) || (st = dws(h, sOwnLC, &olc, L)) || (st = dws(h, sOwnUO, &ouo, L + 1)) ||
        (st = dws(h, sOwnUI, &oui, 1)))
        return st;
    return ingest(h, L, ols, olc, ouo, oui, false);
}

extern "C" afmm_status afmm_p2p_set_tree_device(afmm_p2p *h, int n_leaves, const int *leaf_start,
                                                const int *leaf_count, const long long *u_off,
                                                const int *u_idx) {
    NvtxScope nvtx_("afmm.set_tree_device");
    CHECK_HANDLE(h);
    if (h->n < 1 || !h->d_bodies) return fail(h, AFMM_ESTATE, "set_tree_device: call set_bodies first");
    if (n_leaves < 1 || !leaf_start || !leaf_count || !u_off || !u_idx)
        return fail(h, AFMM_EINVAL, "set_tree_device: n_leaves=%d / null pointer", n_leaves);
    afmm_status st = set_device(h);
    if (st) return st;
    return ingest(h, n_leaves, leaf_start, leaf_count, u_off, u_idx, true);
}

// Host tree ingest: the arrays are copied into the handle's own device buffers
// and ingested there by the kernels of afmm_p2p_set_tree_device (validation,
// Interactions(t), partition and work list on the GPU; a few scalars come back).
// AFMM_HOST_INGEST=1: the host builder instead (reference for the tests).
extern "C" afmm_status afmm_p2p_set_tree(afmm_p2p *h, int n_leaves, const int *leaf_start,
                                         const int *leaf_count, const long long *u_off,
                                         const int *u_idx) {
    NvtxScope nvtx_("afmm.set_tree");
    CHECK_HANDLE(h);
    if (h->n < 1 || !h->d_bodies) return fail(h, AFMM_ESTATE, "set_tree: call set_bodies first");
    if (n_leaves < 1 || !leaf_start || !leaf_count || !u_off)
        return fail(h, AFMM_EINVAL, "set_tree: n_leaves=%d / null pointer", n_leaves);
    const long long nnz = u_off[n_leaves];
    if (nnz < 0 || (nnz > 0 && !u_idx)) return fail(h, AFMM_EINVAL, "set_tree: u_off[n_leaves]=%lld / u_idx null", nnz);
    afmm_status st = set_device(h);
    if (st) return st;
    const char *hb = getenv("AFMM_HOST_INGEST");
    if (hb && hb[0] == '1') return set_tree_host_builder(h, n_leaves, leaf_start, leaf_count, u_off, u_idx);
    const int L = n_leaves;
    int *ols, *olc, *oui;
    long long *ouo;
    if ((st = dws(h, sOwnLS, &ols, L)) || (st = dws(h, sOwnLC, &olc, L)) || (st = dws(h, sOwnUO, &ouo, L + 1)) ||
        (st = dws(h, sOwnUI, &oui, (size_t)std::max<long long>(nnz, 1))))
        return st;
    CUDA_TRY(h, cudaMemcpyAsync(ols, leaf_start, L * sizeof(int), cudaMemcpyHostToDevice, h->stream));
    CUDA_TRY(h, cudaMemcpyAsync(olc, leaf_count, L * sizeof(int), cudaMemcpyHostToDevice, h->stream));
    CUDA_TRY(h, cudaMemcpyAsync(ouo, u_off, (L + 1) * sizeof(long long), cudaMemcpyHostToDevice, h->stream));
    if (nnz > 0) CUDA_TRY(h, cudaMemcpyAsync(oui, u_idx, nnz * sizeof(int), cudaMemcpyHostToDevice, h->stream));
    return ingest(h, L, ols, olc, ouo, oui, false);
}

extern "C" afmm_status afmm_p2p_set_partition(afmm_p2p *h, const long long *leaf_split) {
    CHECK_HANDLE(h);
    const int W = h->cfg.world;
    if (h->tree_on_device) {                           // re-ingest the handle's copy of the tree
        if (!leaf_split) {
            h->user_partition = false;
        } else {
            if (leaf_split[0] != 0) return fail(h, AFMM_EINVAL, "set_partition: leaf_split[0] != 0");
            for (int r = 0; r < W; ++r)
                if (leaf_split[r + 1] < leaf_split[r]) return fail(h, AFMM_EINVAL, "set_partition: not monotone");
            if (h->have_tree && leaf_split[W] != h->L)
                return fail(h, AFMM_EINVAL, "set_partition: leaf_split[world]=%lld != n_leaves=%d", leaf_split[W], h->L);
            h->leaf_split.assign(leaf_split, leaf_split + W + 1);
            h->user_partition = true;
        }
        if (!h->have_tree) return AFMM_OK;
        afmm_status st = set_device(h);
        if (st) return st;
        return reingest(h);
    }
    if (!leaf_split) {
        h->user_partition = false;
        if (!h->have_tree) return AFMM_OK;
        afmm_partition_literal(h->L, h->I.data(), W, h->leaf_split.data());
    } else {
        if (leaf_split[0] != 0) return fail(h, AFMM_EINVAL, "set_partition: leaf_split[0] != 0");
        for (int r = 0; r < W; ++r)
            if (leaf_split[r + 1] < leaf_split[r]) return fail(h, AFMM_EINVAL, "set_partition: not monotone");
        if (h->have_tree && leaf_split[W] != h->L)
            return fail(h, AFMM_EINVAL, "set_partition: leaf_split[world]=%lld != n_leaves=%d", leaf_split[W], h->L);
        h->leaf_split.assign(leaf_split, leaf_split + W + 1);
        h->user_partition = true;
        if (!h->have_tree) return AFMM_OK;
    }
    afmm_status st = set_device(h);
    if (st) return st;
    compute_body_split(h);
    return build_worklist(h);
}

extern "C" afmm_status afmm_p2p_set_cost_coef(afmm_p2p *h, const double *coef) {
    CHECK_HANDLE(h);
    if (!coef) {
        h->have_coef = false;
        return AFMM_OK;
    }
    for (int b = 0; b < 8; ++b)
        if (!(coef[b] > 0.0) || !std::isfinite(coef[b])) return fail(h, AFMM_EINVAL, "set_cost_coef: coef[%d] invalid", b);
    std::copy(coef, coef + 8, h->coef);
    h->have_coef = true;
    return AFMM_OK;
}

extern "C" afmm_status afmm_p2p_get_partition(const afmm_p2p *h, long long *leaf_split,
                                              long long *body_split) {
    if (!h) return AFMM_EINVAL;
    if (!h->have_tree) return AFMM_ESTATE;
    const int W = h->cfg.world;
    if (leaf_split) std::copy(h->leaf_split.begin(), h->leaf_split.end(), leaf_split);
    if (body_split) std::copy(h->body_split.begin(), h->body_split.end(), body_split);
    (void)W;
    return AFMM_OK;
}

// Solve the small SPD system M c = b (Gaussian elimination with partial pivoting).
static bool solve_small(std::vector<double> M, std::vector<double> b, int k, std::vector<double> &x) {
    for (int col = 0; col < k; ++col) {
        int piv = col;
        for (int r = col + 1; r < k; ++r)
            if (std::fabs(M[r * k + col]) > std::fabs(M[piv * k + col])) piv = r;
        if (std::fabs(M[piv * k + col]) < 1e-300) return false;
        if (piv != col) {
            for (int cc = 0; cc < k; ++cc) std::swap(M[col * k + cc], M[piv * k + cc]);
            std::swap(b[col], b[piv]);
        }
        for (int r = col + 1; r < k; ++r) {
            const double f = M[r * k + col] / M[col * k + col];
            for (int cc = col; cc < k; ++cc) M[r * k + cc] -= f * M[col * k + cc];
            b[r] -= f * b[col];
        }
    }
    x.assign(k, 0.0);
    for (int r = k - 1; r >= 0; --r) {
        double s = b[r];
        for (int cc = r + 1; cc < k; ++cc) s -= M[r * k + cc] * x[cc];
        x[r] = s / M[r * k + r];
    }
    return true;
}

// Per-bucket GPU cost coefficients (ms per interaction) from per-rank kernel
// times: the paper's observational coefficient "dividing the maximum kernel
// time by the total number of P2P operations" (L18 SIV.D) refined per
// target-leaf-size bucket by ridge-regularised least squares over ranks:
//   min sum_r (sum_b B_rb c_b - T_r)^2 + lam sum_b (Bsum_b/G)^2 (c_b - k0)^2,
// k0 = sum T / sum I; coefficients kept >= 0.05 k0.
extern "C" afmm_status afmm_cost_fit(int G, const double *bucket_inter, const double *rank_ms, double *coef) {
    if (G < 1 || !bucket_inter || !rank_ms || !coef) return AFMM_EINVAL;
    double Isum = 0, Tsum = 0;
    for (int r = 0; r < G; ++r) {
        if (!(rank_ms[r] >= 0.0) || !std::isfinite(rank_ms[r])) return AFMM_EINVAL;
        Tsum += rank_ms[r];
        for (int b = 0; b < 8; ++b) {
            if (!(bucket_inter[r * 8 + b] >= 0.0)) return AFMM_EINVAL;
            Isum += bucket_inter[r * 8 + b];
        }
    }
    if (Isum <= 0 || Tsum <= 0) {
        for (int b = 0; b < 8; ++b) coef[b] = 1.0;
        return AFMM_OK;
    }
    const double k0 = Tsum / Isum;
    std::vector<double> M(64, 0.0), rhs(8, 0.0), Bs(8, 0.0);
    for (int r = 0; r < G; ++r)
        for (int b = 0; b < 8; ++b) Bs[b] += bucket_inter[r * 8 + b];
    const double lam = 0.1;
    for (int r = 0; r < G; ++r)
        for (int a = 0; a < 8; ++a) {
            for (int b = 0; b < 8; ++b) M[a * 8 + b] += bucket_inter[r * 8 + a] * bucket_inter[r * 8 + b];
            rhs[a] += bucket_inter[r * 8 + a] * rank_ms[r];
        }
    for (int b = 0; b < 8; ++b) {
        const double wgt = lam * (Bs[b] / G) * (Bs[b] / G) + 1e-30;
        M[b * 8 + b] += wgt;
        rhs[b] += wgt * k0;
    }
    std::vector<double> c;
    if (!solve_small(M, rhs, 8, c)) c.assign(8, k0);
    for (int b = 0; b < 8; ++b) coef[b] = (c[b] > 0.05 * k0) ? c[b] : 0.05 * k0;
    return AFMM_OK;
}

extern "C" afmm_status afmm_partition_rebalance(int n_leaves, const int *leaf_count, const long long *I,
                                                int G, const long long *cur_split, const double *rank_ms,
                                                double threshold, long long *new_split, int *changed) {
    if (changed) *changed = 0;
    if (n_leaves < 1 || G < 1 || !leaf_count || !I || !cur_split || !rank_ms || !new_split)
        return AFMM_EINVAL;
    if (cur_split[0] != 0 || cur_split[G] != n_leaves) return AFMM_EINVAL;
    for (int r = 0; r < G; ++r)
        if (cur_split[r + 1] < cur_split[r] || !(rank_ms[r] >= 0.0) || !std::isfinite(rank_ms[r]))
            return AFMM_EINVAL;
    std::copy(cur_split, cur_split + G + 1, new_split);
    if (G == 1) return AFMM_OK;
    // per-rank bucket interaction counts for the current cut
    std::vector<double> B((size_t)G * 8, 0.0);
    double Tsum = 0;
    for (int r = 0; r < G; ++r) {
        for (long long t = cur_split[r]; t < cur_split[r + 1]; ++t)
            B[r * 8 + bucket_of(leaf_count[t])] += (double)I[t];
        Tsum += rank_ms[r];
    }
    if (Tsum <= 0) return AFMM_OK;
    double coef[8];
    afmm_status fst = afmm_cost_fit(G, B.data(), rank_ms, coef);
    if (fst) return fst;
    std::vector<double> w(n_leaves);
    for (int t = 0; t < n_leaves; ++t) w[t] = (double)I[t] * coef[bucket_of(leaf_count[t])];
    std::vector<long long> split(G + 1);
    afmm_partition_weighted(n_leaves, w.data(), G, split.data());
    // adopt only if the predicted imbalance beats the measured one by > threshold
    // (hysteresis in the spirit of the paper's 5% observation rule, L22 SVII.B)
    double tmax = 0, pmax = 0, psum = 0;
    for (int r = 0; r < G; ++r) tmax = std::max(tmax, rank_ms[r]);
    for (int r = 0; r < G; ++r) {
        double pr = 0;
        for (long long t = split[r]; t < split[r + 1]; ++t) pr += w[t];
        pmax = std::max(pmax, pr);
        psum += pr;
    }
    const double cur_imb = tmax / (Tsum / G);
    const double new_imb = psum > 0 ? pmax / (psum / G) : 1.0;
    if (cur_imb - new_imb > threshold && !std::equal(split.begin(), split.end(), cur_split)) {
        std::copy(split.begin(), split.end(), new_split);
        if (changed) *changed = 1;
    }
    return AFMM_OK;
}

extern "C" afmm_status afmm_p2p_rebalance(afmm_p2p *h, const double *rank_ms, double threshold,
                                          int *changed) {
    NvtxScope nvtx_("afmm.rebalance");
    CHECK_HANDLE(h);
    if (changed) *changed = 0;
    if (!h->have_tree) return fail(h, AFMM_ESTATE, "rebalance: no tree");
    if (!rank_ms) return fail(h, AFMM_EINVAL, "rebalance: rank_ms is null");
    const int W = h->cfg.world;
    std::vector<long long> split(W + 1);
    int ch = 0;
    afmm_status st;
    if (h->tree_on_device) {
        // the work list was built on the GPU: leaf sizes and Interactions(t) of the
        // current tree come back from the handle's buffers, the new cut re-ingests it
        if ((st = set_device(h))) return st;
        std::vector<int> lc(h->L);
        std::vector<long long> I(h->L);
        int *olc;
        long long *dI;
        if ((st = dws(h, sOwnLC, &olc, h->L)) || (st = dws(h, sI, &dI, h->L))) return st;
        CUDA_TRY(h, cudaMemcpyAsync(lc.data(), olc, h->L * sizeof(int), cudaMemcpyDeviceToHost, h->stream));
        CUDA_TRY(h, cudaMemcpyAsync(I.data(), dI, h->L * sizeof(long long), cudaMemcpyDeviceToHost, h->stream));
        CUDA_TRY(h, cudaStreamSynchronize(h->stream));
        st = afmm_partition_rebalance(h->L, lc.data(), I.data(), W, h->leaf_split.data(), rank_ms, threshold,
                                      split.data(), &ch);
        if (st) return fail(h, st, "rebalance: invalid rank_ms or partition");
        if (ch) {
            h->leaf_split = split;
            h->user_partition = true;
            if ((st = reingest(h))) return st;
            if (changed) *changed = 1;
        }
        return AFMM_OK;
    }
    st = afmm_partition_rebalance(h->L, h->leaf_count.data(), h->I.data(), W,
                                  h->leaf_split.data(), rank_ms, threshold, split.data(), &ch);
    if (st) return fail(h, st, "rebalance: invalid rank_ms or partition");
    if (ch) {
        h->leaf_split = split;
        h->user_partition = true;
        compute_body_split(h);
        if ((st = set_device(h))) return st;
        if ((st = build_worklist(h))) return st;
        if (changed) *changed = 1;
    }
    return AFMM_OK;
}

// ------------------------------------------------------------------ eval

// window 0 = the caller's outputs; windows 1.. = the registered peer windows (fused gather, row a7)
static void set_windows(afmm_p2p *h, afmm::P2PParams &p, float *ax, float *ay, float *az, float *phi) {
    p.out[0][0] = ax;
    p.out[0][1] = ay;
    p.out[0][2] = az;
    p.out[0][3] = phi;
    p.n_win = 1 + h->n_peers;
    for (int w = 1; w < afmm::kMaxWin; ++w)
        for (int a = 0; a < 4; ++a) p.out[w][a] = w <= h->n_peers ? h->peers[w - 1][a] : nullptr;
}

// the handle's device words (d_words, 64 bytes)
static unsigned *w_ready(afmm_p2p *h) { return reinterpret_cast<unsigned *>(h->d_words); }
static int *w_err(afmm_p2p *h) { return reinterpret_cast<int *>(h->d_words + 4); }
static unsigned long long *w_tspan(afmm_p2p *h) { return reinterpret_cast<unsigned long long *>(h->d_words + 16); }
static double *w_kms(afmm_p2p *h) { return reinterpret_cast<double *>(h->d_words + 32); }

// tspan = {max, 0}: the kernel's CTAs atomicMin their start, warps atomicMax their end
static afmm_status reset_tspan(afmm_p2p *h) {
    CUDA_TRY(h, cudaMemsetAsync(w_tspan(h), 0xff, sizeof(unsigned long long), h->stream));
    CUDA_TRY(h, cudaMemsetAsync(w_tspan(h) + 1, 0, sizeof(unsigned long long), h->stream));
    return AFMM_OK;
}

static afmm_status launch_chunked(afmm_p2p *h, float *ax, float *ay, float *az, float *phi, bool deliver);
static afmm_status comm_finish(afmm_p2p *h);

static afmm_status launch_eval(afmm_p2p *h, float *ax, float *ay, float *az, float *phi) {
    afmm::P2PParams p;
    p.bodies = h->d_bodies;
    p.tasks = h->d_tasks;
    p.segs = h->d_segs;
    p.n_tasks = h->n_tasks;
    p.queue = h->d_queue;
    set_windows(h, p, ax, ay, az, phi);
    p.eps2 = h->cfg.eps2;
    p.G = h->cfg.law == AFMM_LAW_STOKESLET ? 1.0 / (8.0 * 3.14159265358979323846 * (double)h->cfg.mu)
                                           : (double)h->cfg.G;
    p.done = nullptr;
    p.in_ready = nullptr;
    p.in_err = nullptr;
    p.wait_ns = 0;
    p.in_epoch = 0;
    p.m0 = 0.f;
    p.m0_ptr = nullptr;
    p.tspan = h->comm ? w_tspan(h) : nullptr;
    if (h->comm) {
        afmm_status st = reset_tspan(h);
        if (st) return st;
    }
#ifndef AFMM_EQMASS
#define AFMM_EQMASS 1
#endif
    p.mass_unequal = (AFMM_EQMASS && h->cfg.law == AFMM_LAW_GRAVITY) ? mass_flag(h) : nullptr;
    p.mass_bits = nullptr;
    p.out_coalesce = 0;
    h->last_zero_copy = false;
    h->last_input_graph = false;
    h->last_streamed = false;
    h->last_chunked = false;
    CUDA_TRY(h, cudaMemsetAsync(h->d_queue, 0, sizeof(int), h->stream));
    const int ri = (int)(h->n_evals % afmm_p2p::kRing);
    h->ev0 = h->ring0[ri];
    h->ev1 = h->ring1[ri];
    CUDA_TRY(h, cudaEventRecord(h->ev0, h->stream));
    int nlaunch = 0;
    if (p.n_tasks > 0) {
        const int grid = std::max(1, std::min((p.n_tasks + afmm::kWarps - 1) / afmm::kWarps,
                                              h->num_sms * h->blocks_per_sm));
        p.static_rounds = afmm::static_rounds(p.n_tasks, grid * afmm::kWarps);
        if (h->cfg.law == AFMM_LAW_STOKESLET)
            afmm::p2p_kernel_t<afmm::Stokeslet><<<grid, afmm::kThreads, afmm::kDynSmem, h->stream>>>(p);
        else
            afmm::p2p_kernel_t<afmm::Gravity><<<grid, afmm::kThreads, afmm::kDynSmem, h->stream>>>(p);
        COUNT_LAUNCH(1);
        CUDA_TRY(h, cudaGetLastError());
        nlaunch = 1;
    }
    CUDA_TRY(h, cudaEventRecord(h->ev1, h->stream));
    h->n_evals++;
    h->evaluated = true;
    h->last.n_launches = nlaunch;
    return AFMM_OK;
}

static afmm_status fill_stats(afmm_p2p *h, afmm_p2p_stats *s) {
    CUDA_TRY(h, cudaStreamSynchronize(h->stream));
    float ms = 0.f;
    CUDA_TRY(h, cudaEventElapsedTime(&ms, h->ev0, h->ev1));
    afmm_p2p_stats o{};
    o.kernel_ms = ms;
    o.interactions_total = h->I_total;
    o.interactions_rank = h->rank_interactions;
    o.leaf_lo = h->leaf_split[h->cfg.rank];
    o.leaf_hi = h->leaf_split[h->cfg.rank + 1];
    o.body_lo = h->body_split[h->cfg.rank];
    o.body_hi = h->body_split[h->cfg.rank + 1];
    o.n_work_items = h->n_tasks;
    o.n_launches = h->last.n_launches;
    o.zero_copy = h->last_zero_copy ? 1 : 0;
    o.input_graph = h->last_input_graph ? 1 : 0;
    o.streamed_inputs = h->last_streamed ? 1 : 0;
    o.chunked_bodies = h->last_chunked ? 1 : 0;
    o.kernel_ms_max = h->comm ? *(volatile double *)h->h_kms : (double)ms;
    for (int b = 0; b < 8; ++b) o.bucket_interactions[b] = h->bucket_inter[b];
    h->last = o;
    if (s) *s = o;
    if (h->last_chunked && *(volatile int *)h->h_cerr)
        return fail(h, AFMM_ECUDA, "eval: body chunks never arrived (kernel wait timed out, AFMM_WAIT_MS)");
    return AFMM_OK;
}

// One evaluation on device outputs: the chunked replication when the library
// communicator has bodies to broadcast, else the plain launch; then (library
// communicator) the GPU time all-reduce that also completes the fused gather.
static afmm_status launch_any(afmm_p2p *h, float *ax, float *ay, float *az, float *phi) {
    afmm_status st;
    if (h->comm && h->bodies_pending) {
        if ((st = launch_chunked(h, ax, ay, az, phi, true))) return st;
        h->bodies_pending = false;
    } else if ((st = launch_eval(h, ax, ay, az, phi))) {
        return st;
    }
    return h->comm ? comm_finish(h) : AFMM_OK;
}

extern "C" afmm_status afmm_p2p_interactions(const afmm_p2p *h, long long *total, long long *rank) {
    if (!h) return AFMM_EINVAL;
    if (!h->have_tree) return AFMM_ESTATE;
    if (total) *total = h->I_total;
    if (rank) *rank = h->rank_interactions;
    return AFMM_OK;
}

extern "C" afmm_status afmm_p2p_eval(afmm_p2p *h, float *ax, float *ay, float *az, float *phi,
                                     afmm_p2p_stats *stats) {
    NvtxScope nvtx_("afmm.eval");
    CHECK_HANDLE(h);
    if (!h->d_bodies || !h->have_tree) return fail(h, AFMM_ESTATE, "eval: set_bodies and set_tree first");
    if (!ax || !ay || !az || !phi) return fail(h, AFMM_EINVAL, "eval: null output pointer");
    afmm_status st = set_device(h);
    if (st) return st;
    if ((st = launch_any(h, ax, ay, az, phi))) return st;
    if (stats) return fill_stats(h, stats);
    return AFMM_OK;
}

extern "C" afmm_status afmm_p2p_eval_host(afmm_p2p *h, float *ax, float *ay, float *az, float *phi,
                                          afmm_p2p_stats *stats) {
    NvtxScope nvtx_("afmm.eval_host");
    CHECK_HANDLE(h);
    if (!h->d_bodies || !h->have_tree) return fail(h, AFMM_ESTATE, "eval_host: set_bodies and set_tree first");
    if (!ax || !ay || !az || !phi) return fail(h, AFMM_EINVAL, "eval_host: null output pointer");
    afmm_status st = set_device(h);
    if (st) return st;
    const long long n = h->n;
    if (4 * n > h->out_cap) {
        cudaFree(h->d_out);
        h->d_out = nullptr;
        h->out_cap = 0;
        CUDA_TRY(h, cudaMalloc(&h->d_out, (size_t)(4 * n) * sizeof(float)));
        h->out_cap = 4 * n;
    }
    float *d[4] = {h->d_out, h->d_out + n, h->d_out + 2 * n, h->d_out + 3 * n};
    if ((st = launch_any(h, d[0], d[1], d[2], d[3]))) return st;
    const long long lo = h->body_split[h->cfg.rank], hi = h->body_split[h->cfg.rank + 1];
    float *hp[4] = {ax, ay, az, phi};
    if (hi > lo)
        for (int a = 0; a < 4; ++a)
            CUDA_TRY(h, cudaMemcpyAsync(hp[a] + lo, d[a] + lo, (size_t)(hi - lo) * sizeof(float),
                                        cudaMemcpyDeviceToHost, h->stream));
    return fill_stats(h, stats);
}

// ------------------------------------------------------------------ pipelined host evaluation

// A host pointer the device can dereference (page-locked, mapped: pinned memory
// under unified addressing); *dptr = its device address.  Pageable memory -> false.
static bool host_mapped(const void *p, void **dptr) {
    cudaPointerAttributes at{};
    if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
        cudaGetLastError();
        return false;
    }
    if (at.type != cudaMemoryTypeHost || !at.devicePointer) return false;
    *dptr = at.devicePointer;
    return true;
}

// cuStreamWaitValue32 / cuStreamWriteValue32 through the runtime's driver entry points
static afmm_status resolve_stream_ops(afmm_p2p *h) {
    if (h->wait_value32 && h->write_value32) return AFMM_OK;
    cudaDriverEntryPointQueryResult q;
    CUDA_TRY(h, cudaGetDriverEntryPoint("cuStreamWaitValue32", &h->wait_value32, cudaEnableDefault, &q));
    if (q != cudaDriverEntryPointSuccess || !h->wait_value32)
        return fail(h, AFMM_ENOTSUP, "cuStreamWaitValue32 unavailable");
    CUDA_TRY(h, cudaGetDriverEntryPoint("cuStreamWriteValue32", &h->write_value32, cudaEnableDefault, &q));
    if (q != cudaDriverEntryPointSuccess || !h->write_value32)
        return fail(h, AFMM_ENOTSUP, "cuStreamWriteValue32 unavailable");
    return AFMM_OK;
}
using WriteValueFn = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);

static constexpr int kMaxPieces = 64;
// input chunks of the streamed H2D: 8 up to 8 Mi bodies, then one per Mi bodies up to 16 (the first chunk's
// PCIe time is what the kernel's early tasks wait for; A/B on C2: 8 best, on C4 (16 Mi): 16 best, +2 %,
// profiles/r1_ab_input_chunks.txt, profiles/r2_ab_input_chunks_C4.txt)
static int in_chunks(long long n) { return (int)std::min<long long>(16, std::max<long long>(8, n >> 20)); }
static constexpr int kMaxChunks = 16;               // chunk masks ride in the high 16 bits of Task.piece
// First body of input chunk k of K (k = K: n).  Equal chunks up to 8 Mi bodies; above, quadratic boundaries
// n (k/K)^2 (small chunks first, large ones late: C4 host-to-host +0.9 %, C2 -2 %; a small first chunk followed
// by equal ones gains nothing; AFMM_E2E_UNIFORM=1 / 2 forces equal / quadratic; profiles/r2_ab_input_chunks_C4.txt)
static long long chunk_bound(int k, int K, long long n) {
    static const int force = [] { const char *e = getenv("AFMM_E2E_UNIFORM"); return e ? atoi(e) : 0; }();
    if (k >= K) return n;
    const bool quad = force == 2 || (force == 0 && n >= (8LL << 20));
    const long long b = quad ? n * k * k / ((long long)K * K) : (long long)k * ((n + K - 1) / K);
    return std::min<long long>(n, b & ~3LL);                    // multiples of 4: the packs' float4 path stays aligned
}

// Regroup this rank's tasks into P pieces of consecutive targets (equal modelled
// cost tgt_count * nsrc, cut in tgt_start order); inside a piece the tasks keep
// the work list's largest-cost-first order.  Per piece: the output body range and
// the prefix of bodies [0, need) its sources and targets lie in.
// Host copy of this rank's work list (tasks in work-list order and the segments
// they reference), whether it was built on the host or by the device ingest.
static afmm_status fetch_worklist(afmm_p2p *h, std::vector<afmm::Task> &t, std::vector<afmm::Seg> &sg) {
    const int nt = h->n_tasks;
    t.resize(nt);
    CUDA_TRY(h, cudaStreamSynchronize(h->stream));
    if (nt) CUDA_TRY(h, cudaMemcpy(t.data(), h->d_tasks, nt * sizeof(afmm::Task), cudaMemcpyDeviceToHost));
    int nseg = 0;
    for (const auto &x : t) nseg = std::max(nseg, x.seg_begin + x.seg_count);
    sg.resize(nseg);
    if (nseg) CUDA_TRY(h, cudaMemcpy(sg.data(), h->d_segs, nseg * sizeof(afmm::Seg), cudaMemcpyDeviceToHost));
    return AFMM_OK;
}

static afmm_status build_pipe(afmm_p2p *h, int P) {
    const int nt = h->n_tasks;
    std::vector<afmm::Task> t;
    std::vector<afmm::Seg> sg;
    if (afmm_status st0 = fetch_worklist(h, t, sg)) return st0;
    std::vector<int> ord(nt);
    for (int i = 0; i < nt; ++i) ord[i] = i;
    std::stable_sort(ord.begin(), ord.end(), [&](int a, int b) { return t[a].tgt_start < t[b].tgt_start; });
    double total = 0.0;
    for (const auto &x : t) total += (double)x.tgt_count * (double)std::max(x.nsrc, 1);
    std::vector<int> piece(nt, 0);
    double acc = 0.0;
    int p = 0;
    for (int r = 0; r < nt; ++r) {
        const afmm::Task &x = t[ord[r]];
        // a leaf's slices share tgt_start ranges that are disjoint; cut only between leaves' first slices
        while (p < P - 1 && acc >= total * (p + 1) / P && (r == 0 || x.self_start != t[ord[r - 1]].self_start)) ++p;
        piece[ord[r]] = p;
        acc += (double)x.tgt_count * (double)std::max(x.nsrc, 1);
    }
    h->pipe_off.assign(P + 1, 0);
    h->pipe_need.assign(P, 0);
    h->pipe_lo.assign(P, LLONG_MAX);
    h->pipe_hi.assign(P, 0);
    for (int i = 0; i < nt; ++i) {
        const int q = piece[i];
        h->pipe_off[q + 1]++;
        long long need = (long long)t[i].tgt_start + t[i].tgt_count;
        for (int j = 0; j < t[i].seg_count; ++j) {
            const afmm::Seg &z = sg[t[i].seg_begin + j];
            need = std::max(need, (long long)z.gstart + z.len);
        }
        h->pipe_need[q] = std::max(h->pipe_need[q], need);
        h->pipe_lo[q] = std::min(h->pipe_lo[q], (long long)t[i].tgt_start);
        h->pipe_hi[q] = std::max(h->pipe_hi[q], (long long)t[i].tgt_start + t[i].tgt_count);
    }
    for (int q = 0; q < P; ++q) {
        h->pipe_off[q + 1] += h->pipe_off[q];
        if (q > 0) h->pipe_need[q] = std::max(h->pipe_need[q], h->pipe_need[q - 1]);
        if (h->pipe_lo[q] > h->pipe_hi[q]) h->pipe_lo[q] = h->pipe_hi[q] = 0;   // empty piece
    }
    // Input chunks: the bodies in K Morton ranges (chunk_bound), copied and packed in order while
    // the kernel runs.  Task order: by the last input chunk the task needs (its sources
    // and targets), then by output piece, LPT kept inside -- so the kernel starts on the
    // first chunk and stays behind the copies, and every output piece's stragglers (leaves
    // whose U-lists reach far in Morton order) run as soon as the last chunk lands.
    const char *kenv = getenv("AFMM_E2E_CHUNKS");             // measurements only
    const int kin = kenv ? std::max(1, std::min(kMaxChunks, atoi(kenv))) : in_chunks(h->n);
    const int K = (int)std::min<long long>(kin, std::max<long long>(1, h->n / 4096));
    std::vector<int> need_chunk(nt, 0);
    for (int i = 0; i < nt; ++i) {
        long long need = (long long)t[i].tgt_start + t[i].tgt_count;
        for (int j = 0; j < t[i].seg_count; ++j) {
            const afmm::Seg &z = sg[t[i].seg_begin + j];
            need = std::max(need, (long long)z.gstart + z.len);
        }
        int c = 0;                                              // the chunk holding body need - 1
        while (c < K - 1 && chunk_bound(c + 1, K, h->n) < need) ++c;
        need_chunk[i] = c;
    }
    std::vector<int> ord2(nt);
    for (int i = 0; i < nt; ++i) ord2[i] = i;
    static const bool piece_major = [] {
        const char *e = getenv("AFMM_PIPE_ORDER");
        return !(e && e[0] == 'c');
    }();
    std::stable_sort(ord2.begin(), ord2.end(), [&](int a, int b) {
        if (piece_major)
            return piece[a] != piece[b] ? piece[a] < piece[b] : need_chunk[a] < need_chunk[b];
        return need_chunk[a] != need_chunk[b] ? need_chunk[a] < need_chunk[b] : piece[a] < piece[b];
    });
    std::vector<afmm::Task> grouped(std::max(nt, 1));
    for (int r = 0; r < nt; ++r) {                                              // stable: LPT kept
        afmm::Task x = t[ord2[r]];
        // need mask: chunks 0..need_chunk (they arrive in Morton order)
        x.piece = (int)((unsigned)piece[ord2[r]] | (((2u << need_chunk[ord2[r]]) - 1u) << 16));
        grouped[r] = x;
    }
    h->pipe_K = K;
    afmm_status st = ensure_device(h, &h->d_ptasks, h->ptasks_cap, grouped.size());
    if (st) return st;
    CUDA_TRY(h, cudaMemcpy(h->d_ptasks, grouped.data(), grouped.size() * sizeof(afmm::Task), cudaMemcpyHostToDevice));
    h->pipe_P = P;
    h->pipe_valid = true;
    return AFMM_OK;
}

extern "C" afmm_status afmm_p2p_eval_host_pipelined(afmm_p2p *h, long long n, const float *x, const float *y,
                                                    const float *z, const float *m, float *ax, float *ay,
                                                    float *az, float *phi, int n_pieces, afmm_p2p_stats *stats) {
    NvtxScope nvtx_("afmm.eval_host_pipelined");
    CHECK_HANDLE(h);
    if (h->cfg.law != AFMM_LAW_GRAVITY) return fail(h, AFMM_EINVAL, "eval_host_pipelined: gravity handles only");
    if (!h->have_tree || !h->d_bodies) return fail(h, AFMM_ESTATE, "eval_host_pipelined: set_bodies and set_tree first");
    if (n != h->n) return fail(h, AFMM_EINVAL, "eval_host_pipelined: n=%lld differs from the tree's %lld", n, h->n);
    if (!x || !y || !z || !m || !ax || !ay || !az || !phi)
        return fail(h, AFMM_EINVAL, "eval_host_pipelined: null pointer");
    if (n_pieces < 1 || n_pieces > kMaxPieces)
        return fail(h, AFMM_EINVAL, "eval_host_pipelined: n_pieces=%d outside [1, %d]", n_pieces, kMaxPieces);
    afmm_status st = set_device(h);
    if (st) return st;
    if (!h->s_in) {
        CUDA_TRY(h, cudaStreamCreateWithFlags(&h->s_in, cudaStreamNonBlocking));
        CUDA_TRY(h, cudaStreamCreateWithFlags(&h->s_out, cudaStreamNonBlocking));
        CUDA_TRY(h, cudaEventCreateWithFlags(&h->ev_start, cudaEventDisableTiming));
        CUDA_TRY(h, cudaEventCreateWithFlags(&h->ev_done, cudaEventDisableTiming));
        CUDA_TRY(h, cudaEventCreateWithFlags(&h->ev_in_done, cudaEventDisableTiming));
        for (int i = 0; i < kMaxPieces; ++i) {
            CUDA_TRY(h, cudaEventCreateWithFlags(&h->ev_in[i], cudaEventDisableTiming));
            CUDA_TRY(h, cudaEventCreateWithFlags(&h->ev_k[i], cudaEventDisableTiming));
        }
        CUDA_TRY(h, cudaMalloc(&h->d_pqueue, (kMaxPieces + 4) * sizeof(int)));
        CUDA_TRY(h, cudaMallocHost(&h->h_err, sizeof(int)));
    }
    if ((st = resolve_stream_ops(h))) return st;
    if (4 * n > h->soa_cap) {
        cudaFree(h->d_soa);
        h->d_soa = nullptr;
        h->soa_cap = 0;
        CUDA_TRY(h, cudaMalloc(&h->d_soa, (size_t)(4 * n) * sizeof(float)));
        h->soa_cap = 4 * n;
    }
    if (4 * n > h->out_cap) {
        cudaFree(h->d_out);
        h->d_out = nullptr;
        h->out_cap = 0;
        CUDA_TRY(h, cudaMalloc(&h->d_out, (size_t)(4 * n) * sizeof(float)));
        h->out_cap = 4 * n;
    }
    if (!h->pipe_valid || h->pipe_P != n_pieces)
        if ((st = build_pipe(h, n_pieces))) return st;
    const int P = n_pieces;
    float *dsoa[4] = {h->d_soa, h->d_soa + n, h->d_soa + 2 * n, h->d_soa + 3 * n};
    float *dout[4] = {h->d_out, h->d_out + n, h->d_out + 2 * n, h->d_out + 3 * n};
    const float *hin[4] = {x, y, z, m};
    float *hout[4] = {ax, ay, az, phi};
    // One launch over the piece-major task list: a piece's tail overlaps the
    // next piece; warps count finished tasks per piece (P2PParams.done) and the
    // copy-out stream waits on each counter (cuStreamWaitValue32) before copying
    // that piece's outputs back, while later pieces still run.  The inputs go in
    // first (sources of a piece may lie anywhere in the tree order).
    using WaitFn = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
    const WaitFn wait32 = reinterpret_cast<WaitFn>(h->wait_value32);
    using WriteFn = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
    const WriteFn write32 = reinterpret_cast<WriteFn>(h->write_value32);
    int *queue = h->d_pqueue, *done = h->d_pqueue + 1;
    unsigned *in_ready = reinterpret_cast<unsigned *>(h->d_pqueue + kMaxPieces + 1);
    int *in_err = h->d_pqueue + kMaxPieces + 2;
    unsigned *mass_bits = reinterpret_cast<unsigned *>(h->d_pqueue + kMaxPieces + 3);
    CUDA_TRY(h, cudaMemsetAsync(h->d_pqueue, 0, (kMaxPieces + 4) * sizeof(int), h->stream));
    // Zero-copy when all eight host arrays are page-locked and device-mapped (pinned
    // memory under unified addressing): the pack kernels read the inputs and the P2P
    // kernel's epilogue writes the outputs straight over PCIe -- no staging copies,
    // the output transfer spread over the whole kernel.  Else staged copies.
    const float *zin[4] = {nullptr, nullptr, nullptr, nullptr};
    float *zout[4] = {nullptr, nullptr, nullptr, nullptr};
    // (AFMM_E2E_ZEROCOPY: "0" off; "i" / "o" inputs / outputs only -- for measurements)
    const char *zenv = getenv("AFMM_E2E_ZEROCOPY");
    bool zc = !(zenv && zenv[0] == '0');
    for (int a = 0; a < 4 && zc; ++a) {
        void *d = nullptr;
        zc = host_mapped(hin[a], &d);
        zin[a] = static_cast<const float *>(d);
        zc = zc && host_mapped(hout[a], &d);
        zout[a] = static_cast<float *>(d);
    }
    const bool zc_in = zc && !(zenv && zenv[0] == 'o'), zc_out = zc && !(zenv && zenv[0] == 'i');
    h->last_zero_copy = zc;
    const float m0 = m[0];                          // equal-mass test of the streamed chunks
    h->bodies_pending = false;                      // every body comes from this call's host arrays
    h->deferred = false;
    h->last_chunked = false;
    CUDA_TRY(h, cudaMemsetAsync(mass_flag(h), 0xff, sizeof(int), h->stream));   // bodies replaced: flag "unequal"
    CUDA_TRY(h, cudaEventRecord(h->ev_start, h->stream));      // earlier readers of the bodies / outputs
    CUDA_TRY(h, cudaStreamWaitEvent(h->s_in, h->ev_start, 0));
    CUDA_TRY(h, cudaStreamWaitEvent(h->s_out, h->ev_start, 0));
    // inputs streamed in K Morton chunks: copy (4 SoA slices), pack, then publish the
    // chunk count in device memory (cuStreamWriteValue32 orders the packed bodies
    // before the flag); the kernel's warps wait per task for the chunk it needs.
    // The pack kernels run next to the persistent P2P kernel (128 threads, few
    // registers: they fit in what one P2P CTA leaves free on an SM).
    // The P2P launch is enqueued AFTER every input chunk's pack (host order): if the
    // copy stream and the compute stream share a hardware queue, a pack queued behind
    // the persistent kernel would never run (the kernel waits for it).  The kernel
    // does not wait for chunk 0 (its warps wait per task; m_0 comes from the host).
    int nlaunch = 0;
    auto launch = [&]() -> afmm_status {
        if (h->comm) {
            const afmm_status s0 = reset_tspan(h);
            if (s0) return s0;
        }
        const int ri = (int)(h->n_evals % afmm_p2p::kRing);
        h->ev0 = h->ring0[ri];
        h->ev1 = h->ring1[ri];
        CUDA_TRY(h, cudaEventRecord(h->ev0, h->stream));
        const int nt = h->pipe_off[P];
        if (nt > 0) {
            afmm::P2PParams prm;
            prm.bodies = h->d_bodies;
            prm.tasks = h->d_ptasks;
            prm.segs = h->d_segs;
            prm.n_tasks = nt;
            prm.queue = queue;
            prm.static_rounds = 0;                       // pieces complete in claim order
            for (int a = 0; a < 4; ++a) prm.out[0][a] = zc_out ? zout[a] : dout[a];
            prm.n_win = 1;
            prm.out_coalesce = zc_out ? 1 : 0;
            prm.mass_bits = (AFMM_EQMASS && h->cfg.law == AFMM_LAW_GRAVITY) ? mass_bits : nullptr;
            prm.eps2 = h->cfg.eps2;
            prm.G = (double)h->cfg.G;
            prm.mass_unequal = nullptr;                  // the flag is final only after the last chunk
            prm.done = zc_out ? nullptr : done;
            prm.in_ready = in_ready;
            prm.in_err = in_err;
            prm.wait_ns = wait_ns(h);
            prm.in_epoch = 0;                            // the flag word is zeroed per call (epoch 0)
            prm.m0 = m0;
            prm.m0_ptr = nullptr;
            prm.tspan = h->comm ? w_tspan(h) : nullptr;
            const int grid = std::max(1, std::min((nt + afmm::kWarps - 1) / afmm::kWarps, h->num_sms * h->blocks_per_sm));
            afmm::p2p_stream_kernel_t<afmm::Gravity><<<grid, afmm::kThreads, afmm::kDynSmem, h->stream>>>(prm);
            COUNT_LAUNCH(1);
            CUDA_TRY(h, cudaGetLastError());
            nlaunch = 1;
        }
        CUDA_TRY(h, cudaEventRecord(h->ev1, h->stream));
        return AFMM_OK;
    };
    const int K = h->pipe_K;
    // Without room for a pack block beside a P2P CTA (co_resident_pack) the chain
    // could not progress under the persistent kernel: pack every chunk first, then
    // launch (the kernel's chunk waits then pass at once).
    const bool streamed = h->co_resident_pack;
    h->last_streamed = streamed;
    // Enqueue the input chain: pack chunk k, then publish k + 1 (stream write).
    auto enqueue_inputs = [&](bool capturing) -> afmm_status {
        for (int k = 0; k < K; ++k) {
            const long long lo = chunk_bound(k, K, n), hi = chunk_bound(k + 1, K, n);
            if (hi > lo) {
                const float *src[4];
                for (int a = 0; a < 4; ++a) {
                    if (zc_in) {
                        src[a] = zin[a] + lo;
                    } else {
                        CUDA_TRY(h, cudaMemcpyAsync(dsoa[a] + lo, hin[a] + lo, (size_t)(hi - lo) * sizeof(float),
                                                    cudaMemcpyHostToDevice, h->s_in));
                        src[a] = dsoa[a] + lo;
                    }
                }
                const int threads = 128;
                const int blocks = (int)std::min<long long>((hi - lo + threads - 1) / threads, (long long)h->num_sms);
                afmm::pack_chunk_kernel<<<blocks, threads, 0, h->s_in>>>((int)(hi - lo), src[0], src[1], src[2],
                                                                        src[3], h->d_bodies + lo, m0, mass_bits, k);
                if (!capturing) COUNT_LAUNCH(1);          // a captured chain counts when its graph replays
                const cudaError_t le = cudaPeekAtLastError();
                if (le != cudaSuccess) {
                    if (capturing) return AFMM_ECUDA;
                    (void)cudaGetLastError();
                    return fail(h, AFMM_ECUDA, "eval_host_pipelined: pack launch failed: %s", cudaGetErrorString(le));
                }
            }
            // the delivered-chunk mask: chunks 0..k
            const CUresult r = write32((CUstream)h->s_in, (CUdeviceptr)in_ready, (cuuint32_t)((2u << k) - 1u), 0);
            if (r != CUDA_SUCCESS) {
                if (capturing) return AFMM_ECUDA;
                return fail(h, AFMM_ECUDA, "eval_host_pipelined: cuStreamWriteValue32 failed (%d)", (int)r);
            }
        }
        return AFMM_OK;
    };
    // Zero-copy: the chain is the same on every call with the same arrays, so it is
    // captured once into a graph and replayed by one launch (2K host API calls fewer
    // before the P2P launch).  AFMM_INPUT_GRAPH=0, or a failed capture: direct launches.
    const char *genv = getenv("AFMM_INPUT_GRAPH");
    bool use_graph = zc_in && !h->in_graph_off && !(genv && genv[0] == '0');
    if (use_graph) {
        unsigned m0bits;
        std::memcpy(&m0bits, &m0, sizeof m0bits);
        const bool same = h->in_graph && h->ig_n == n && h->ig_K == K && h->ig_m0 == m0bits &&
                          h->ig_bodies == h->d_bodies && h->ig_src[0] == zin[0] && h->ig_src[1] == zin[1] &&
                          h->ig_src[2] == zin[2] && h->ig_src[3] == zin[3];
        if (!same) {
            if (h->in_graph) cudaGraphExecDestroy(h->in_graph);
            h->in_graph = nullptr;
            cudaGraph_t g = nullptr;
            bool ok = cudaStreamBeginCapture(h->s_in, cudaStreamCaptureModeThreadLocal) == cudaSuccess;
            if (ok) {
                const afmm_status es = enqueue_inputs(true);
                const cudaError_t ee = cudaStreamEndCapture(h->s_in, &g);
                ok = es == AFMM_OK && ee == cudaSuccess && g != nullptr;
            }
            if (ok) ok = cudaGraphInstantiate(&h->in_graph, g, 0) == cudaSuccess;
            if (g) cudaGraphDestroy(g);
            if (!ok) {
                (void)cudaGetLastError();
                if (h->in_graph) cudaGraphExecDestroy(h->in_graph);
                h->in_graph = nullptr;
                h->in_graph_off = true;                  // do not try again on this handle
                use_graph = false;
            } else {
                h->ig_n = n;
                h->ig_K = K;
                h->ig_m0 = m0bits;
                h->ig_bodies = h->d_bodies;
                for (int a = 0; a < 4; ++a) h->ig_src[a] = zin[a];
            }
        }
        if (use_graph) {
            CUDA_TRY(h, cudaGraphLaunch(h->in_graph, h->s_in));
            COUNT_LAUNCH(K);
        }
    }
    h->last_input_graph = use_graph;
    if (!use_graph) {
        if ((st = enqueue_inputs(false))) return st;
    }
    if (!streamed) {                                  // serial fallback: inputs complete before the launch
        CUDA_TRY(h, cudaEventRecord(h->ev_in_done, h->s_in));
        CUDA_TRY(h, cudaStreamWaitEvent(h->stream, h->ev_in_done, 0));
    }
    if ((st = launch())) return st;
    // join the input chain into the handle's stream: the kernel waits only for the
    // chunks its own tasks reach (none at all for a rank without tasks or after a
    // wait timeout), so without this the call could return -- and the next call
    // reset the chunk flags -- while pack kernels still read the host inputs
    CUDA_TRY(h, cudaEventRecord(h->ev_in_done, h->s_in));
    CUDA_TRY(h, cudaStreamWaitEvent(h->stream, h->ev_in_done, 0));
    // the launch must be enqueued before the copy-out stream starts waiting on its counters
    for (int q = 0; q < P && !zc_out; ++q) {
        const long long lo = h->pipe_lo[q], hi = h->pipe_hi[q];
        const int cnt = h->pipe_off[q + 1] - h->pipe_off[q];
        if (hi <= lo || cnt == 0) continue;
        const CUresult r = wait32((CUstream)h->s_out, (CUdeviceptr)(done + q), (cuuint32_t)cnt, CU_STREAM_WAIT_VALUE_GEQ);
        if (r != CUDA_SUCCESS) return fail(h, AFMM_ECUDA, "eval_host_pipelined: cuStreamWaitValue32 failed (%d)", (int)r);
        for (int a = 0; a < 4; ++a)
            CUDA_TRY(h, cudaMemcpyAsync(hout[a] + lo, dout[a] + lo, (size_t)(hi - lo) * sizeof(float),
                                        cudaMemcpyDeviceToHost, h->s_out));
    }
    // safety net: nothing on s_out may outlive the kernel's stream order
    CUDA_TRY(h, cudaStreamWaitEvent(h->s_out, h->ev1, 0));
    CUDA_TRY(h, cudaEventRecord(h->ev_done, h->s_out));
    CUDA_TRY(h, cudaStreamWaitEvent(h->stream, h->ev_done, 0));
    h->n_evals++;
    h->evaluated = true;
    h->last.n_launches = nlaunch;
    // the wait-timeout flag rides on the stream into pinned memory: fill_stats'
    // synchronise covers it (no separate blocking copy)
    *h->h_err = 0;
    CUDA_TRY(h, cudaMemcpyAsync(h->h_err, in_err, sizeof(int), cudaMemcpyDeviceToHost, h->stream));
    if (h->comm && (st = comm_finish(h))) return st;
    if ((st = fill_stats(h, stats))) return st;
    if (*(volatile int *)h->h_err) return fail(h, AFMM_ECUDA, "eval_host_pipelined: input chunks never arrived (kernel wait timed out)");
    return AFMM_OK;
}

// ------------------------------------------------------------------ chunked body replication

// The delivery plan of the packed bodies (afmm_p2p_chunks) and the work list in
// delivery order: K <= 16 chunks of consecutive bodies; chunk c is owned by the
// rank whose body slice holds its first body; the delivery order deals the
// ranks' chunks round robin (every rank's first chunk among the first `world`
// deliveries, its k-th among the first k*world).  Every task gets the mask of the
// chunks its targets and source segments touch (high 16 bits of Task.piece) and
// the tasks are ordered by the delivery position of the last chunk they need
// (stable: the work list's largest-cost-first order inside each position), so
// the first tasks a warp claims are the ones the first chunks make runnable.
static afmm_status build_chunks(afmm_p2p *h) {
    std::vector<afmm::Task> t;
    std::vector<afmm::Seg> sg;
    afmm_status st = fetch_worklist(h, t, sg);
    if (st) return st;
    const long long n = h->n;
    const int K = (int)std::min<long long>(kMaxChunks, std::max<long long>(1, n / 4096));
    const int W = h->cfg.world;
    std::vector<long long> b(K + 1);
    for (int k = 0; k <= K; ++k) b[k] = n * k / K;
    auto chunk_of = [&](long long i) {            // chunk holding body i
        return (int)(std::upper_bound(b.begin(), b.end(), i) - b.begin()) - 1;
    };
    std::vector<std::vector<int>> owned(W);
    for (int k = 0; k < K; ++k) {
        int r = (int)(std::upper_bound(h->body_split.begin(), h->body_split.end(), b[k]) - h->body_split.begin()) - 1;
        r = std::max(0, std::min(W - 1, r));
        owned[r].push_back(k);
    }
    std::vector<int> order, pos(K);
    for (size_t j = 0; (int)order.size() < K; ++j)
        for (int r = 0; r < W; ++r)
            if (j < owned[r].size()) order.push_back(owned[r][j]);
    for (int j = 0; j < K; ++j) pos[order[j]] = j;
    const int nt = (int)t.size();
    std::vector<unsigned> mask(nt, 0);
    std::vector<int> ready(nt, 0);
    for (int i = 0; i < nt; ++i) {
        unsigned msk = 0;
        auto add = [&](long long lo, long long len) {
            if (len <= 0) return;
            for (int c = chunk_of(lo), e = chunk_of(lo + len - 1); c <= e; ++c) msk |= 1u << c;
        };
        add(t[i].tgt_start, t[i].tgt_count);
        for (int j = 0; j < t[i].seg_count; ++j) add(sg[t[i].seg_begin + j].gstart, sg[t[i].seg_begin + j].len);
        mask[i] = msk;
        int rd = 0;
        for (int c = 0; c < K; ++c)
            if (msk >> c & 1u) rd = std::max(rd, pos[c]);
        ready[i] = rd;
    }
    std::vector<int> ord(nt);
    std::iota(ord.begin(), ord.end(), 0);
    std::stable_sort(ord.begin(), ord.end(), [&](int a, int c) { return ready[a] < ready[c]; });
    std::vector<afmm::Task> out(std::max(nt, 1));
    for (int i = 0; i < nt; ++i) {
        out[i] = t[ord[i]];
        out[i].piece = (int)(mask[ord[i]] << 16);
    }
    if ((st = ensure_device(h, &h->d_ctasks, h->ctasks_cap, out.size()))) return st;
    CUDA_TRY(h, cudaMemcpy(h->d_ctasks, out.data(), out.size() * sizeof(afmm::Task), cudaMemcpyHostToDevice));
    h->chunk_K = K;
    h->chunk_bounds = b;
    h->chunk_order = order;
    h->chunk_valid = true;
    return AFMM_OK;
}

// The P2P kernel on the chunk-ordered work list, every task waiting for its
// chunks (epoch-tagged mask word, never reset).  deliver: the library
// communicator broadcasts the trailer, then the chunks in delivery order on
// s_comm, publishing the cumulative mask after each (cuStreamWriteValue32 orders
// the broadcast's writes before the flag); else the caller delivers and
// publishes (afmm_p2p_publish_chunks).  The kernel leaves comm_sms SMs free for
// the transport's kernels.
static afmm_status launch_chunked(afmm_p2p *h, float *ax, float *ay, float *az, float *phi, bool deliver) {
    afmm_status st;
    if (h->cfg.law != AFMM_LAW_GRAVITY) return fail(h, AFMM_ENOTSUP, "chunked replication: gravity handles only");
    if (!h->chunk_valid && (st = build_chunks(h))) return st;
    if ((st = resolve_stream_ops(h))) return st;
    const WriteValueFn write32 = reinterpret_cast<WriteValueFn>(h->write_value32);
    h->epoch = h->epoch % 0xffffu + 1u;                       // 1 .. 65535 (0: the pipelined path)
    const unsigned tag = h->epoch << 16;
    CUDA_TRY(h, cudaMemsetAsync(w_err(h), 0, sizeof(int), h->stream));
    CUDA_TRY(h, cudaMemsetAsync(h->d_queue, 0, sizeof(int), h->stream));
    if (h->comm && (st = reset_tspan(h))) return st;          // before the communication stream may start a kernel
    afmm::P2PParams p;
    p.bodies = h->d_bodies;
    p.tasks = h->d_ctasks;
    p.segs = h->d_segs;
    p.n_tasks = h->n_tasks;
    p.queue = h->d_queue;
    p.static_rounds = 0;                                       // claims follow the delivery order
    set_windows(h, p, ax, ay, az, phi);
    p.eps2 = h->cfg.eps2;
    p.G = (double)h->cfg.G;
    p.done = nullptr;
    p.in_ready = w_ready(h);
    p.in_err = w_err(h);
    p.wait_ns = wait_ns(h);
    p.in_epoch = h->epoch;
    p.mass_unequal = nullptr;
    p.mass_bits = (AFMM_EQMASS ? reinterpret_cast<const unsigned *>(mass_flag(h)) : nullptr);   // 0 or all bits
    p.m0 = 0.f;
    p.m0_ptr = reinterpret_cast<const float *>(mass_flag(h) + 1);                            // trailer word 1
    p.out_coalesce = 0;
    p.tspan = h->comm ? w_tspan(h) : nullptr;
    h->last_tail_ctas = 0;
    if (deliver) {
        const afmm::NcclApi &nc = afmm::nccl_api();
        CUDA_TRY(h, cudaEventRecord(h->ev_c0, h->stream));    // the root's pack, earlier readers of the bodies
        CUDA_TRY(h, cudaStreamWaitEvent(h->s_comm, h->ev_c0, 0));
        const bool defer = h->deferred;                        // root of set_bodies_deferred: pack per chunk here
        h->deferred = false;
        const int TH = 256;
        if (defer) {
            CUDA_TRY(h, cudaMemsetAsync(mass_flag(h), 0, sizeof(int), h->s_comm));
            mass_trailer_kernel<<<h->num_sms * 2, TH, 0, h->s_comm>>>(h->n, h->def_soa[3], mass_flag(h));
            COUNT_LAUNCH(1);
            CUDA_TRY(h, cudaGetLastError());
        }
        NCCL_TRY(h, nc.Broadcast(mass_flag(h), mass_flag(h), sizeof(float4), ncclChar, 0, h->comm, h->s_comm));
        unsigned cum = 0;
        for (int j = 0; j < h->chunk_K; ++j) {
            const int c = h->chunk_order[j];
            const long long lo = h->chunk_bounds[c], cnt = h->chunk_bounds[c + 1] - lo;
            if (defer && cnt > 0) {
                const int blocks = (int)std::min<long long>((cnt + TH - 1) / TH, (long long)h->num_sms * 4);
                pack_range_kernel<<<blocks, TH, 0, h->s_comm>>>(cnt, h->def_soa[0] + lo, h->def_soa[1] + lo,
                                                                h->def_soa[2] + lo, h->def_soa[3] + lo, h->d_bodies + lo);
                COUNT_LAUNCH(1);
                CUDA_TRY(h, cudaGetLastError());
            }
            if (cnt > 0)
                NCCL_TRY(h, nc.Broadcast(h->d_bodies + lo, h->d_bodies + lo, (size_t)cnt * sizeof(float4), ncclChar, 0,
                                         h->comm, h->s_comm));
            cum |= 1u << c;
            const CUresult r = write32((CUstream)h->s_comm, (CUdeviceptr)w_ready(h), (cuuint32_t)(tag | cum), 0);
            if (r != CUDA_SUCCESS) return fail(h, AFMM_ECUDA, "chunked eval: cuStreamWriteValue32 failed (%d)", (int)r);
        }
        // The SMs kept free for NCCL idle once the last chunk is out: a second, small grid of the same
        // kernel on the communication stream takes tasks from the same queue until it is empty (every
        // result is the same whichever CTA computes it).  AFMM_TAIL_KERNEL=0 disables it.
        const char *tenv = getenv("AFMM_TAIL_KERNEL");
        const int tail = std::min(comm_sms(h), (p.n_tasks + afmm::kWarps - 1) / afmm::kWarps);
        if (p.n_tasks > 0 && tail > 0 && !(tenv && tenv[0] == '0')) {
            afmm::p2p_stream_kernel_t<afmm::Gravity><<<tail, afmm::kThreads, afmm::kDynSmem, h->s_comm>>>(p);
            COUNT_LAUNCH(1);
            CUDA_TRY(h, cudaGetLastError());
            h->last_tail_ctas = tail;
        }
        CUDA_TRY(h, cudaEventRecord(h->ev_c1, h->s_comm));
    }
    h->last_zero_copy = false;
    h->last_input_graph = false;
    h->last_streamed = false;
    const int ri = (int)(h->n_evals % afmm_p2p::kRing);
    h->ev0 = h->ring0[ri];
    h->ev1 = h->ring1[ri];
    CUDA_TRY(h, cudaEventRecord(h->ev0, h->stream));
    int nlaunch = 0;
    if (p.n_tasks > 0) {
        const int room = std::max(1, h->num_sms * h->blocks_per_sm - comm_sms(h));
        const int grid = std::max(1, std::min((p.n_tasks + afmm::kWarps - 1) / afmm::kWarps, room));
        afmm::p2p_stream_kernel_t<afmm::Gravity><<<grid, afmm::kThreads, afmm::kDynSmem, h->stream>>>(p);
        COUNT_LAUNCH(1);
        CUDA_TRY(h, cudaGetLastError());
        nlaunch = 1 + (h->last_tail_ctas > 0);
    }
    CUDA_TRY(h, cudaEventRecord(h->ev1, h->stream));
    *h->h_cerr = 0;
    CUDA_TRY(h, cudaMemcpyAsync(h->h_cerr, w_err(h), sizeof(int), cudaMemcpyDeviceToHost, h->stream));
    if (deliver) CUDA_TRY(h, cudaStreamWaitEvent(h->stream, h->ev_c1, 0));   // the broadcast joins the stream
    h->n_evals++;
    h->evaluated = true;
    h->last_chunked = true;
    h->last.n_launches = nlaunch;
    return AFMM_OK;
}

// Library communicator, after every eval: the kernel's device-timer span (ms),
// all-reduced with MAX on s_comm -> *h_kms (the GPU time of PAPER L20 SVII.A).
// Every rank's contribution is enqueued after its own kernel, so when the
// all-reduce completes every rank's kernel -- and its fused-gather stores into
// the peer windows, fenced system-wide at kernel end -- has completed: the
// handle's stream waits for it.
static afmm_status comm_finish(afmm_p2p *h) {
    const afmm::NcclApi &nc = afmm::nccl_api();
    afmm::span_ms_kernel<<<1, 1, 0, h->stream>>>(w_tspan(h), w_kms(h));
    COUNT_LAUNCH(1);
    CUDA_TRY(h, cudaGetLastError());
    CUDA_TRY(h, cudaEventRecord(h->ev_c2, h->stream));
    CUDA_TRY(h, cudaStreamWaitEvent(h->s_comm, h->ev_c2, 0));
    NCCL_TRY(h, nc.AllReduce(w_kms(h), w_kms(h) + 1, 1, ncclFloat64, ncclMax, h->comm, h->s_comm));
    CUDA_TRY(h, cudaMemcpyAsync(h->h_kms, w_kms(h) + 1, sizeof(double), cudaMemcpyDeviceToHost, h->s_comm));
    CUDA_TRY(h, cudaEventRecord(h->ev_c3, h->s_comm));
    CUDA_TRY(h, cudaStreamWaitEvent(h->stream, h->ev_c3, 0));
    return AFMM_OK;
}

extern "C" afmm_status afmm_p2p_chunks(afmm_p2p *h, int *K, long long *bounds, int *order) {
    CHECK_HANDLE(h);
    if (!h->d_bodies || !h->have_tree) return fail(h, AFMM_ESTATE, "chunks: set_bodies and set_tree first");
    afmm_status st = set_device(h);
    if (st) return st;
    if (!h->chunk_valid && (st = build_chunks(h))) return st;
    if (K) *K = h->chunk_K;
    if (bounds) std::copy(h->chunk_bounds.begin(), h->chunk_bounds.end(), bounds);
    if (order) std::copy(h->chunk_order.begin(), h->chunk_order.end(), order);
    return AFMM_OK;
}

extern "C" afmm_status afmm_p2p_worklist(afmm_p2p *h, int *tasks, long long cap_tasks, long long *n_tasks, int *segs,
                                         long long cap_segs, long long *n_segs) {
    CHECK_HANDLE(h);
    if (!h->have_tree) return fail(h, AFMM_ESTATE, "worklist: set_tree first");
    afmm_status st = set_device(h);
    if (st) return st;
    std::vector<afmm::Task> t;
    std::vector<afmm::Seg> sg;
    if ((st = fetch_worklist(h, t, sg))) return st;
    static_assert(sizeof(afmm::Task) == 8 * sizeof(int) && sizeof(afmm::Seg) == 2 * sizeof(int), "layout");
    if (n_tasks) *n_tasks = (long long)t.size();
    if (n_segs) *n_segs = (long long)sg.size();
    if (tasks && cap_tasks >= (long long)t.size() && !t.empty()) std::memcpy(tasks, t.data(), t.size() * sizeof(afmm::Task));
    if (segs && cap_segs >= (long long)sg.size() && !sg.empty()) std::memcpy(segs, sg.data(), sg.size() * sizeof(afmm::Seg));
    return AFMM_OK;
}

extern "C" afmm_status afmm_p2p_eval_chunked(afmm_p2p *h, float *ax, float *ay, float *az, float *phi) {
    NvtxScope nvtx_("afmm.eval_chunked");
    CHECK_HANDLE(h);
    if (afmm_status st0 = flush_deferred(h)) return st0;
    if (!h->d_bodies || !h->have_tree) return fail(h, AFMM_ESTATE, "eval_chunked: set_bodies and set_tree first");
    if (!ax || !ay || !az || !phi) return fail(h, AFMM_EINVAL, "eval_chunked: null output pointer");
    afmm_status st = set_device(h);
    if (st) return st;
    if ((st = launch_chunked(h, ax, ay, az, phi, false))) return st;
    h->bodies_pending = false;
    return h->comm ? comm_finish(h) : AFMM_OK;
}

extern "C" afmm_status afmm_p2p_publish_chunks(afmm_p2p *h, int count, void *stream) {
    CHECK_HANDLE(h);
    if (!h->chunk_valid) return fail(h, AFMM_ESTATE, "publish_chunks: no chunk plan (call eval_chunked first)");
    if (count < 1 || count > h->chunk_K)
        return fail(h, AFMM_EINVAL, "publish_chunks: count %d outside [1, %d]", count, h->chunk_K);
    afmm_status st = set_device(h);
    if (st) return st;
    if ((st = resolve_stream_ops(h))) return st;
    unsigned cum = 0;
    for (int j = 0; j < count; ++j) cum |= 1u << h->chunk_order[j];
    const WriteValueFn write32 = reinterpret_cast<WriteValueFn>(h->write_value32);
    const CUresult r = write32((CUstream)(stream ? static_cast<cudaStream_t>(stream) : h->stream),
                               (CUdeviceptr)w_ready(h), (cuuint32_t)((h->epoch << 16) | cum), 0);
    if (r != CUDA_SUCCESS) return fail(h, AFMM_ECUDA, "publish_chunks: cuStreamWriteValue32 failed (%d)", (int)r);
    return AFMM_OK;
}

extern "C" afmm_status afmm_p2p_set_peer_windows(afmm_p2p *h, int count, float *const *ptrs) {
    if (!h) return AFMM_EINVAL;
    if (count < 0 || count > afmm::kMaxWin - 1)
        return fail(h, AFMM_EINVAL, "set_peer_windows: count %d outside [0, %d]", count, afmm::kMaxWin - 1);
    if (count > 0 && !ptrs) return fail(h, AFMM_EINVAL, "set_peer_windows: ptrs is null");
    for (int k = 0; k < 4 * count; ++k)
        if (!ptrs[k]) return fail(h, AFMM_EINVAL, "set_peer_windows: pointer %d is null", k);
    h->n_peers = count;
    for (int w = 0; w < afmm::kMaxWin - 1; ++w)
        for (int a = 0; a < 4; ++a) h->peers[w][a] = w < count ? ptrs[4 * w + a] : nullptr;
    return AFMM_OK;
}

namespace {
using RangeFn = CUresult (*)(CUdeviceptr *, size_t *, CUdeviceptr);
RangeFn address_range_fn() {
    static RangeFn fn = nullptr;
    if (!fn) {
        void *f = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = reinterpret_cast<RangeFn>(f);
    }
    return fn;
}
}  // namespace

extern "C" afmm_status afmm_ipc_export(const void *dev_ptr, afmm_ipc_handle *out) {
    if (!dev_ptr || !out) return AFMM_EINVAL;
    const RangeFn range = address_range_fn();
    if (!range) return AFMM_ENOTSUP;
    CUdeviceptr base = 0;
    size_t size = 0;
    if (range(&base, &size, (CUdeviceptr)dev_ptr) != CUDA_SUCCESS) return AFMM_EINVAL;
    cudaIpcMemHandle_t hd;
    if (cudaIpcGetMemHandle(&hd, (void *)base) != cudaSuccess) {
        cudaGetLastError();
        return AFMM_ECUDA;
    }
    static_assert(sizeof(hd) == sizeof(out->handle), "cudaIpcMemHandle_t is 64 bytes");
    std::memcpy(out->handle, &hd, sizeof(hd));
    out->offset = (long long)((CUdeviceptr)dev_ptr - base);
    return AFMM_OK;
}

extern "C" afmm_status afmm_ipc_import(const afmm_ipc_handle *in, void **dev_ptr, void **base) {
    if (!in || !dev_ptr || !base || in->offset < 0) return AFMM_EINVAL;
    cudaIpcMemHandle_t hd;
    std::memcpy(&hd, in->handle, sizeof(hd));
    void *b = nullptr;
    if (cudaIpcOpenMemHandle(&b, hd, cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
        cudaGetLastError();
        return AFMM_ECUDA;
    }
    *base = b;
    *dev_ptr = (char *)b + in->offset;
    return AFMM_OK;
}

extern "C" afmm_status afmm_ipc_close(void *base) {
    if (!base) return AFMM_EINVAL;
    if (cudaIpcCloseMemHandle(base) != cudaSuccess) {
        cudaGetLastError();
        return AFMM_ECUDA;
    }
    return AFMM_OK;
}

extern "C" long long afmm_launch_count(void) { return g_launches.load(std::memory_order_relaxed); }

extern "C" afmm_status afmm_p2p_stats_get(afmm_p2p *h, afmm_p2p_stats *stats) {
    NvtxScope nvtx_("afmm.stats_get");
    CHECK_HANDLE(h);
    if (!h->evaluated) return fail(h, AFMM_ESTATE, "stats_get: no eval yet");
    afmm_status st = set_device(h);
    if (st) return st;
    return fill_stats(h, stats);
}

#if AFMM_PROF
// tuning builds only (-DAFMM_PROF=1): the per-warp cycle breakdown of the last P2P launch
extern "C" int afmm_p2p_prof_read(unsigned long long *host, int n) {
    const int cap = 148 * 32 * afmm::kProfSlots;
    n = n < cap ? n : cap;
    if (cudaMemcpyFromSymbol(host, afmm::afmm_prof_buf, (size_t)n * 8) != cudaSuccess) return -1;
    return n;
}
#endif
extern "C" int afmm_p2p_kernel_times(afmm_p2p *h, int max_count, double *ms) {
    if (!h || h->poisoned || max_count < 0 || (max_count > 0 && !ms)) return AFMM_EINVAL;
    if (set_device(h)) return AFMM_ECUDA;
    if (cudaStreamSynchronize(h->stream) != cudaSuccess) {
        fail(h, AFMM_ECUDA, "kernel_times: stream sync failed");
        return AFMM_ECUDA;
    }
    long long avail = std::min<long long>(h->n_evals, afmm_p2p::kRing);
    const int cnt = (int)std::min<long long>(avail, max_count);
    for (int i = 0; i < cnt; ++i) {
        const long long ev = h->n_evals - cnt + i;      // oldest first
        const int ri = (int)(ev % afmm_p2p::kRing);
        float f = 0.f;
        if (cudaEventElapsedTime(&f, h->ring0[ri], h->ring1[ri]) != cudaSuccess) {
            fail(h, AFMM_ECUDA, "kernel_times: cudaEventElapsedTime failed");
            return AFMM_ECUDA;
        }
        ms[i] = f;
    }
    return cnt;
}
