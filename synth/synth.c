/*
 * synth.c -- seeded, integer-only synthetic INPUT generators.
 *
 * This module is shared by the CPU oracle (oracle/) and the CUDA path
 * (paper_conf_isca_muthukrishnannl21_b200/).  It holds NONE of the method's
 * arithmetic (no stencil, no PageRank/SSSP math, no PROACT protocol): it only
 * produces the inputs both sides consume, so that both see byte-identical data.
 *
 * Why synthetic: PAPER.md Sec. IV-C (L265-L269) runs on the Wikipedia and HV15R
 * datasets which are not available here; BASELINE.json configs 3-4 replace
 * them with RMAT scale-24, edge factor 16.  The Jacobi grid init and the
 * microbenchmark seed follow SURVEY.md Sec. 8(c) (c-table).
 *
 * Everything is counter based (splitmix64 of seed ^ counter), so any element
 * can be regenerated independently, in any thread order, in any language.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* splitmix64 output function (Steele, Lea, Flood 2014): one step from state x. */
uint64_t synth_splitmix64(uint64_t x)
{
    uint64_t z = x + 0x9E3779B97F4A7C15ULL;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

/* Jacobi initial grid: x0[i][j] = 1 + (splitmix64(seed ^ (i*N+j)) >> 41) * 2^-23,
 * an exact fp32 value in [1, 2).  Rows [row0, row0+nrows) of an N-wide grid are written to out. */
void synth_jacobi_init(float *out, int64_t N, int64_t row0, int64_t nrows, uint64_t seed)
{
#pragma omp parallel for schedule(static)
    for (int64_t r = 0; r < nrows; ++r) {
        int64_t i = row0 + r;
        for (int64_t j = 0; j < N; ++j) {
            uint64_t m = synth_splitmix64(seed ^ (uint64_t)(i * N + j)) >> 41; /* 23 bits */
            out[r * N + j] = 1.0f + (float)m * (1.0f / 8388608.0f);
        }
    }
}

/* Graph500-style RMAT quadrant thresholds A, A+B, A+B+C (A,B,C = .57,.19,.19) as 32-bit integers. */
#define RMAT_TA 2448131358u   /* floor(0.57 * 2^32) */
#define RMAT_TB 3264175144u   /* floor(0.76 * 2^32) */
#define RMAT_TC 4080218931u   /* floor(0.95 * 2^32) */

/* level-l draw of edge e: base = splitmix64(seed ^ e); r = splitmix64(base ^ (l >> 1)); the even
 * level takes the low 32 bits, the odd level the high 32 bits (two draws per splitmix64 call). */
static uint32_t rmat_draw(uint64_t base, int level)
{
    uint64_t r = synth_splitmix64(base ^ (uint64_t)(level >> 1));
    return (level & 1) ? (uint32_t)(r >> 32) : (uint32_t)r;
}

/* Fisher-Yates permutation of [0, V) driven by splitmix64(perm_seed ^ i). */
void synth_permutation(uint32_t *perm, int64_t V, uint64_t perm_seed)
{
    for (int64_t i = 0; i < V; ++i) perm[i] = (uint32_t)i;
    for (int64_t i = V - 1; i > 0; --i) {
        uint64_t j = synth_splitmix64(perm_seed ^ (uint64_t)i) % (uint64_t)(i + 1);
        uint32_t t = perm[i]; perm[i] = perm[j]; perm[j] = t;
    }
}

/*
 * RMAT edge list: E0 = V * edge_factor raw edges, V = 2^scale.  Edge e picks one quadrant per
 * level (MSB first) by comparing rmat_draw(seed, e, level) against the thresholds; endpoints are
 * then relabelled by the seeded permutation; self loops are dropped, duplicates kept, generation
 * order preserved.  src/dst must hold E0 entries; returns the number of edges kept.
 */
int64_t synth_rmat(uint32_t *src, uint32_t *dst, int scale, int64_t edge_factor,
                   uint64_t seed, uint64_t perm_seed)
{
    int64_t V = (int64_t)1 << scale;
    int64_t E0 = V * edge_factor;
    uint32_t *perm = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)V);
    if (!perm) return -1;
    synth_permutation(perm, V, perm_seed);
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < E0; ++e) {
        uint32_t u = 0, v = 0;
        uint64_t base = synth_splitmix64(seed ^ (uint64_t)e);
        for (int l = 0; l < scale; ++l) {
            uint32_t r = rmat_draw(base, l);
            uint32_t ubit = r >= RMAT_TB;                          /* quadrants C, D */
            uint32_t vbit = (r >= RMAT_TA && r < RMAT_TB) || r >= RMAT_TC; /* B, D */
            u = (u << 1) | ubit;
            v = (v << 1) | vbit;
        }
        src[e] = perm[u];
        dst[e] = perm[v];
    }
    free(perm);
    /* stable compaction: drop self loops */
    int64_t k = 0;
    for (int64_t e = 0; e < E0; ++e) {
        if (src[e] != dst[e]) { src[k] = src[e]; dst[k] = dst[e]; ++k; }
    }
    return k;
}

/* SSSP edge weights: w(e) = 1 + splitmix64(seed ^ e) % 255, in [1, 255]. */
void synth_weights(int32_t *w, int64_t E, uint64_t seed)
{
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < E; ++e)
        w[e] = 1 + (int32_t)(synth_splitmix64(seed ^ (uint64_t)e) % 255u);
}

/* Banded system for the paper's Jacobi solver (Sec. IV-C: "Jacobi solver for
 * banded matrices").  DIA layout: a[(o + w) * N + i] = A[i][i + o], o in [-w, w];
 * off-diagonals -(1 + u) / (4w) with u = (splitmix64(seed ^ ((o+w)*N + i)) >> 41) * 2^-23 in
 * [0, 1), entries outside the matrix (i + o not in [0, N)) are 0; diagonal 2 (strictly dominant:
 * sum |off| <= 1); b[i] = 1 + (splitmix64(~seed ^ i) >> 41) * 2^-23. */
void synth_banded(float *a, float *b, int64_t N, int64_t w, uint64_t seed)
{
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < N; ++i) {
        for (int64_t o = -w; o <= w; ++o) {
            float v;
            if (o == 0) v = 2.0f;
            else if (i + o < 0 || i + o >= N) v = 0.0f;
            else {
                uint64_t m = synth_splitmix64(seed ^ (uint64_t)((o + w) * N + i)) >> 41;
                v = -(1.0f + (float)m * (1.0f / 8388608.0f)) / (float)(4 * w);
            }
            a[(o + w) * N + i] = v;
        }
        b[i] = 1.0f + (float)(synth_splitmix64(~seed ^ (uint64_t)i) >> 41) * (1.0f / 8388608.0f);
    }
}
