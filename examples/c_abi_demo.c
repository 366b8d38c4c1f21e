/*
 * c_abi_demo.c -- the library from plain C, no Python: GPU octree + U-lists
 * (afmm_tree_*), then the near-field P2P through the host-pointer entry points
 * (afmm_p2p_set_bodies_host / set_tree / eval_host), and a check of sampled
 * bodies against a direct fp64 sum over their U-lists (the definition of the
 * near-field sum, PAPER L12 SI.C; reading R16's per-body bound on phi).
 *
 *   make demo            (gcc, links libafmm_p2p.so and libcudart)
 *   examples/c_abi_demo [n] [S]     -> prints stats, exit status 0 if within 1e-5
 */
#include <math.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#include <cuda_runtime_api.h>

#include "afmm_p2p.h"
#include "afmm_tree.h"

#define CHECK(call)                                                                                \
    do {                                                                                           \
        afmm_status s_ = (call);                                                                   \
        if (s_ != AFMM_OK) {                                                                       \
            fprintf(stderr, "%s -> %d\n", #call, (int)s_);                                        \
            return 2;                                                                              \
        }                                                                                          \
    } while (0)

static uint64_t rng = 88172645463325252ull;
static float urand(void) {               /* xorshift64 -> [0, 1) */
    rng ^= rng << 13;
    rng ^= rng >> 7;
    rng ^= rng << 17;
    return (float)((rng >> 40) * (1.0 / 16777216.0));
}

int main(int argc, char **argv) {
    const long long n = argc > 1 ? atoll(argv[1]) : 200000;
    const int S = argc > 2 ? atoi(argv[2]) : 64;
    const float eps2 = 1e-6f;
    float *h[4], *d[3];
    for (int a = 0; a < 4; ++a) h[a] = (float *)malloc(n * sizeof(float));
    for (long long i = 0; i < n; ++i) {
        h[0][i] = urand();
        h[1][i] = urand();
        h[2][i] = urand();
        h[3][i] = 1.0f / (float)n;
    }
    for (int a = 0; a < 3; ++a) {
        if (cudaMalloc((void **)&d[a], n * sizeof(float)) != cudaSuccess) return 2;
        cudaMemcpy(d[a], h[a], n * sizeof(float), cudaMemcpyHostToDevice);
    }
    /* 1. tree on the GPU, copied to host arrays */
    afmm_tree *t = NULL;
    CHECK(afmm_tree_create(0, NULL, &t));
    CHECK(afmm_tree_build(t, n, d[0], d[1], d[2], S, 0, NULL, 0));
    int L = 0;
    long long nnz = 0;
    CHECK(afmm_tree_info(t, &L, &nnz, NULL, NULL, NULL, NULL));
    int *perm = malloc(n * sizeof(int)), *ls = malloc(L * sizeof(int)), *lc = malloc(L * sizeof(int));
    long long *uo = malloc((L + 1) * sizeof(long long));
    int *ui = malloc(nnz * sizeof(int));
    CHECK(afmm_tree_copy_out(t, perm, ls, lc, NULL, NULL, uo, ui));
    /* bodies in tree (Morton) order */
    float *b[4];
    for (int a = 0; a < 4; ++a) {
        b[a] = malloc(n * sizeof(float));
        for (long long i = 0; i < n; ++i) b[a][i] = h[a][perm[i]];
    }
    /* 2. P2P through the C ABI, host pointers in and out */
    afmm_p2p_config cfg;
    CHECK(afmm_p2p_config_init(&cfg));
    cfg.eps2 = eps2;
    afmm_p2p *p = NULL;
    CHECK(afmm_p2p_create(&cfg, &p));
    CHECK(afmm_p2p_set_bodies_host(p, n, b[0], b[1], b[2], b[3]));
    CHECK(afmm_p2p_set_tree(p, L, ls, lc, uo, ui));
    float *o[4];
    for (int a = 0; a < 4; ++a) o[a] = malloc(n * sizeof(float));
    afmm_p2p_stats st;
    CHECK(afmm_p2p_eval_host(p, o[0], o[1], o[2], o[3], &st));
    /* 3. check sampled target leaves against a direct fp64 sum over U(t) */
    double worst = 0.0;
    for (int k = 0; k < 64; ++k) {
        const int tl = (int)((long long)k * (L - 1) / 63);
        for (int i = ls[tl]; i < ls[tl] + lc[tl]; ++i) {
            double phi = 0.0;
            for (long long e = uo[tl]; e < uo[tl + 1]; ++e) {
                const int s = ui[e];
                for (int j = ls[s]; j < ls[s] + lc[s]; ++j) {
                    if (j == i) continue;
                    const double dx = (double)b[0][j] - b[0][i], dy = (double)b[1][j] - b[1][i],
                                 dz = (double)b[2][j] - b[2][i];
                    phi -= (double)b[3][j] / sqrt(dx * dx + dy * dy + dz * dz + (double)eps2);
                }
            }
            const double rel = phi != 0.0 ? fabs(o[3][i] - phi) / fabs(phi) : fabs((double)o[3][i]);
            if (rel > worst) worst = rel;
        }
    }
    printf("n=%lld S=%d leaves=%d nnz=%lld interactions=%lld kernel_ms=%.4f phi_max_rel(64 leaves)=%.3e %s\n", n, S,
           L, nnz, st.interactions_total, st.kernel_ms, worst, afmm_version());
    afmm_p2p_destroy(p);
    afmm_tree_destroy(t);
    for (int a = 0; a < 3; ++a) cudaFree(d[a]);
    return worst <= 1e-5 ? 0 : 1;
}
