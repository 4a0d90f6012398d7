/*
 * oracle.c -- plain, slow, obviously-correct CPU reference for the PROACT hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Nothing on the product path may import, call, link or execute
 * anything under oracle/: only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs do.  It shares no code with the CUDA path (no headers, helpers or
 * tables); the only common module is synth/ (seeded input generators, no method arithmetic).
 *
 * Source of truth: /root/reference/PAPER.md (ISCA'21 PROACT), cited as PAPER.md:L<line>.
 * PROACT only changes WHEN bytes move between GPUs (Sec. III-B: "all the local writes to
 * a PROACT-enabled region are sent to the remote GPUs"), so each workload's oracle is the plain
 * single-array definition, iterated phase by phase (O-math below).  The protocol itself is
 * pinned by a separate multi-threaded simulator (O-proto, oracle_proto_*), which checks the
 * paper's invariants under random interleavings.
 *
 * Floating point: compiled with -ffp-contract=off; fp32 where the method is fp32 (Jacobi,
 * DESIGN.md reading R10), fp64 accumulation where the paper is silent (PageRank, reading R12).
 *
 * Pins (tests/test_oracle_*.py): MurmurHash3 published vectors (fmix32), harmonic fixed points
 * and closed-form sine-mode decay (Jacobi), dense linear solve (PageRank), Dijkstra and dense
 * min-plus brute force (SSSP), invariants (mass, symmetry, monotonicity).
 */
#define _GNU_SOURCE
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <stdatomic.h>
#include <pthread.h>
#include <sched.h>
#include <omp.h>
#include <time.h>

static double now_s(void)
{
    struct timespec t;
    clock_gettime(CLOCK_MONOTONIC, &t);
    return (double)t.tv_sec + 1e-9 * (double)t.tv_nsec;
}

/* OpenMP thread count (results never depend on it: every parallel loop writes disjoint cells). */
void oracle_set_threads(int n) { if (n > 0) omp_set_num_threads(n); }
int oracle_get_threads(void) { return omp_get_max_threads(); }

/* ------------------------------------------------------------------------------------------ */
/* Microbenchmark (Sec. IV-C: a synthetic compute kernel on the source GPU
 * generating data needed in its entirety by the destination GPUs; Sec. V-A: each source
 * thread block generates 4KB).  Word k of phase p is a chain of K MurmurHash3 finalisers
 * (reading R14): v = fmix32(k ^ (p * 0x9E3779B9) ^ seed), then K-1 more fmix32(v). */

uint32_t oracle_fmix32(uint32_t h)
{
    h ^= h >> 16;
    h *= 0x85EBCA6Bu;
    h ^= h >> 13;
    h *= 0xC2B2AE35u;
    h ^= h >> 16;
    return h;
}

uint32_t oracle_micro_word(uint64_t k, uint32_t phase, uint32_t seed, int K)
{
    uint32_t v = oracle_fmix32((uint32_t)k ^ (phase * 0x9E3779B9u) ^ seed);
    for (int i = 1; i < K; ++i) v = oracle_fmix32(v);
    return v;
}

/* The full region (W words) after phase `phase`: every replica must equal this. */
void oracle_micro_phase(uint32_t *out, int64_t W, uint32_t phase, uint32_t seed, int K)
{
#pragma omp parallel for schedule(static)
    for (int64_t k = 0; k < W; ++k) out[k] = oracle_micro_word((uint64_t)k, phase, seed, K);
}

/* ------------------------------------------------------------------------------------------ */
/* Jacobi (Sec. IV-C: "iteratively computes the solution vector using Jacobi's
 * method"; BASELINE.json configs 1-2: 2D 5-point stencil, fp32).  Reading R9/R10:
 * Laplace equation, Dirichlet boundary (boundary cells copied through every iteration), fixed
 * association x' = 0.25 * ((up + down) + (left + right)), fp32 round-to-nearest, no FMA. */

void oracle_jacobi_step(const float *in, float *out, int64_t N)
{
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < N; ++i) {
        for (int64_t j = 0; j < N; ++j) {
            int64_t c = i * N + j;
            if (i == 0 || j == 0 || i == N - 1 || j == N - 1) {
                out[c] = in[c];
            } else {
                float vert = in[c - N] + in[c + N];
                float horz = in[c - 1] + in[c + 1];
                out[c] = 0.25f * (vert + horz);
            }
        }
    }
}

/* x holds x^0 on entry and x^iters on return. */
int oracle_jacobi(float *x, int64_t N, int iters)
{
    float *tmp = (float *)malloc(sizeof(float) * (size_t)(N * N));
    if (!tmp) return -1;
    float *a = x, *b = tmp;
    for (int k = 0; k < iters; ++k) {
        oracle_jacobi_step(a, b, N);
        float *t = a; a = b; b = t;
    }
    if (a != x) memcpy(x, a, sizeof(float) * (size_t)(N * N));
    free(tmp);
    return 0;
}

/* ------------------------------------------------------------------------------------------ */
/* PageRank (Sec. IV-C: "assigns a 'Page-rank score' to web pages based on their
 * importance").  Reading R11/R12: r^0 = 1/V; r^{k+1}[v] = (1-d)/V + d * sum_{u->v} r^k[u]/out(u),
 * d = 0.85, out(u) counts multi-edges, dangling mass not redistributed; the per-vertex sum is
 * accumulated in fp64 over in-edges in CSC order (edges stably sorted by destination) and the
 * result rounded to fp32 once per iteration (r is fp32 between iterations). */

int oracle_pagerank(int64_t V, int64_t E, const uint32_t *src, const uint32_t *dst,
                    int iters, double d, float *r_out, double *iter_seconds)
{
    int64_t *outdeg = (int64_t *)calloc((size_t)V + 1, sizeof(int64_t));
    int64_t *colptr = (int64_t *)calloc((size_t)V + 1, sizeof(int64_t));
    uint32_t *rowidx = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)(E ? E : 1));
    float *r = (float *)malloc(sizeof(float) * (size_t)(V ? V : 1));
    float *rn = (float *)malloc(sizeof(float) * (size_t)(V ? V : 1));
    if (!outdeg || !colptr || !rowidx || !r || !rn) return -1;
    /* CSC: stable counting sort of the edge list by destination */
    for (int64_t e = 0; e < E; ++e) { outdeg[src[e]]++; colptr[dst[e] + 1]++; }
    for (int64_t v = 0; v < V; ++v) colptr[v + 1] += colptr[v];
    {
        int64_t *cur = (int64_t *)malloc(sizeof(int64_t) * (size_t)(V ? V : 1));
        if (!cur) return -1;
        memcpy(cur, colptr, sizeof(int64_t) * (size_t)V);
        for (int64_t e = 0; e < E; ++e) rowidx[cur[dst[e]]++] = src[e];
        free(cur);
    }
    for (int64_t v = 0; v < V; ++v) r[v] = (float)(1.0 / (double)V);
    const double base = (1.0 - d) / (double)V;
    const double t0 = now_s();   /* iterations only (the CSC build above is input preparation) */
    for (int k = 0; k < iters; ++k) {
#pragma omp parallel for schedule(dynamic, 4096)
        for (int64_t v = 0; v < V; ++v) {
            double sum = 0.0;
            for (int64_t p = colptr[v]; p < colptr[v + 1]; ++p) {
                uint32_t u = rowidx[p];
                sum += (double)r[u] / (double)outdeg[u];
            }
            rn[v] = (float)(base + d * sum);
        }
        float *t = r; r = rn; rn = t;
    }
    if (iter_seconds) *iter_seconds = now_s() - t0;
    memcpy(r_out, r, sizeof(float) * (size_t)V);
    free(outdeg); free(colptr); free(rowidx); free(r); free(rn);
    return 0;
}

/* ------------------------------------------------------------------------------------------ */
/* SSSP (Sec. IV-C: "In each iteration, every vertex computes its shortest
 * distance from the source vertex using the Bellman-Ford algorithm").  Reading R13: int32
 * distances, INF = INT32_MAX, synchronous rounds d^{k+1}[v] = min(d^k[v],
 * min_{u->v, d^k[u] != INF} d^k[u] + w(u->v)); stop after the first round that changes nothing
 * (that round is counted) or after V rounds.  Also records, per round, how many vertices
 * changed (used by the roofline accounting).  Written as the paper says it -- every vertex
 * computes its own distance -- i.e. a pull over each vertex's in-edges (CSC, edges stably sorted
 * by destination), one vertex per loop iteration, OpenMP over vertices: a min over a fixed set
 * is order independent, so the result does not depend on the thread count. */

int oracle_sssp(int64_t V, int64_t E, const uint32_t *src, const uint32_t *dst,
                const int32_t *w, int64_t s, int max_rounds, int32_t *d_out,
                int *rounds_out, int64_t *changed_per_round, double *iter_seconds)
{
    int32_t *dk = (int32_t *)malloc(sizeof(int32_t) * (size_t)(V ? V : 1));
    int32_t *dn = (int32_t *)malloc(sizeof(int32_t) * (size_t)(V ? V : 1));
    int64_t *colptr = (int64_t *)calloc((size_t)V + 1, sizeof(int64_t));
    uint32_t *rowidx = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)(E ? E : 1));
    int32_t *wt = (int32_t *)malloc(sizeof(int32_t) * (size_t)(E ? E : 1));
    if (!dk || !dn || !colptr || !rowidx || !wt) return -1;
    /* CSC: stable counting sort of the edges by destination (input preparation) */
    for (int64_t e = 0; e < E; ++e) colptr[dst[e] + 1]++;
    for (int64_t v = 0; v < V; ++v) colptr[v + 1] += colptr[v];
    {
        int64_t *cur = (int64_t *)malloc(sizeof(int64_t) * (size_t)(V ? V : 1));
        if (!cur) return -1;
        memcpy(cur, colptr, sizeof(int64_t) * (size_t)V);
        for (int64_t e = 0; e < E; ++e) {
            const int64_t q = cur[dst[e]]++;
            rowidx[q] = src[e];
            wt[q] = w[e];
        }
        free(cur);
    }
    for (int64_t v = 0; v < V; ++v) dk[v] = INT32_MAX;
    if (V > 0) dk[s] = 0;
    if (max_rounds <= 0 || max_rounds > V) max_rounds = (int)(V > 0 ? V : 1);
    int rounds = 0;
    const double t0 = now_s();
    for (int k = 0; k < max_rounds; ++k) {
        int64_t changed = 0;
#pragma omp parallel for schedule(dynamic, 4096) reduction(+ : changed)
        for (int64_t v = 0; v < V; ++v) {
            int32_t best = dk[v];
            for (int64_t p = colptr[v]; p < colptr[v + 1]; ++p) {
                const int32_t du = dk[rowidx[p]];
                if (du == INT32_MAX) continue;
                const int64_t cand = (int64_t)du + (int64_t)wt[p];
                if (cand < best) best = (int32_t)cand;
            }
            dn[v] = best;
            changed += best != dk[v];
        }
        if (changed_per_round) changed_per_round[k] = changed;
        int32_t *t = dk; dk = dn; dn = t;
        rounds = k + 1;
        if (changed == 0) break;
    }
    if (iter_seconds) *iter_seconds = now_s() - t0;
    memcpy(d_out, dk, sizeof(int32_t) * (size_t)V);
    *rounds_out = rounds;
    free(dk); free(dn); free(colptr); free(rowidx); free(wt);
    return 0;
}

/* ------------------------------------------------------------------------------------------ */
/* O-proto: a protocol simulator.  G simulated GPUs are threads groups: per rank, P producer
 * threads ("CTAs") and A agent threads, all std C11 atomics, with random yields.  It follows
 * PAPER.md Sec. III-B/C step by step:
 *   - producers write ONLY the local copy of a PROACT-enabled region (L123, Fig. 5) and, per
 *     tile, bump the chunk's counter (L127-L129; reading R1: counting bytes up to `expected`);
 *   - an agent polls the counters (L137 "Polling"), and a ready chunk is pushed to every peer
 *     replica at the same offset (1:1 correspondence, L123), then an arrival flag is raised
 *     (reading R5; the paper's global barrier L125 is the BARRIER mode);
 *   - credits: before overwriting peer p's replica with generation-e data the agent waits for
 *     p to have finished phase e-1 (reading R6).
 * Workload: the microbenchmark (all-gather shape, reading R14) or tiny Jacobi (halo waits on
 * the flags).  Invariants checked every phase:
 *   I1 each (chunk, dest) delivered exactly once; I2 counter observed at claim == expected;
 *   I3 after the phase every flag carries the phase's generation; I4 replica bytes == producer
 *   bytes (checked at the end against O-math by the caller).
 * Returns 0, or a negative code identifying the violated invariant. */

#define PROTO_MAXG 8

typedef struct {
    int G, P, A, workload;   /* workload 0 = micro, 1 = jacobi */
    int64_t N;               /* jacobi: grid N; micro: words W */
    int64_t chunk_words;     /* chunk size in 4-byte words */
    int phases;
    uint32_t seed;
    int K;
    uint64_t rng_seed;
    /* replicas: rep[g][buf] full extent, buf = 2 for ping-pong */
    uint32_t *rep[PROTO_MAXG][2];
    int64_t own0[PROTO_MAXG + 1];     /* owned word ranges, rank-ordered concatenation */
    int64_t tile_words;
    /* per rank per buf per chunk */
    _Atomic int64_t *counter[PROTO_MAXG];
    int64_t *expected[PROTO_MAXG];
    _Atomic int32_t *deliv[PROTO_MAXG];      /* [chunk_global * G + dest] deliveries this phase */
    _Atomic uint32_t *arrive[PROTO_MAXG];    /* consumer side, [buf][chunk_global] */
    _Atomic uint32_t done[PROTO_MAXG][PROTO_MAXG]; /* done[at rank][from rank] */
    _Atomic int32_t tile_next[PROTO_MAXG];
    _Atomic int32_t producers_left[PROTO_MAXG];
    _Atomic int err;
    int64_t nchunks_total;
    int64_t chunk0[PROTO_MAXG + 1];   /* global chunk index of rank's first chunk */
} proto_t;

typedef struct { proto_t *S; int g, id; uint64_t rng; int phase; } proto_thr;

static uint64_t xs(uint64_t *s) { uint64_t x = *s; x ^= x << 13; x ^= x >> 7; x ^= x << 17; *s = x; return x; }
static void maybe_yield(uint64_t *rng) { if ((xs(rng) & 7) == 0) sched_yield(); }

static void proto_fail(proto_t *S, int code) { int z = 0; atomic_compare_exchange_strong(&S->err, &z, code); }

static int64_t proto_chunk_of(proto_t *S, int g, int64_t word)   /* owned-local chunk index */
{ return (word - S->own0[g]) / S->chunk_words; }

static float as_f(uint32_t u) { float f; memcpy(&f, &u, 4); return f; }
static uint32_t as_u(float f) { uint32_t u; memcpy(&u, &f, 4); return u; }

/* producer thread: tiles of the owned range, instrumented stores, per-tile commit */
static void *proto_producer(void *arg)
{
    proto_thr *T = (proto_thr *)arg; proto_t *S = T->S; int g = T->g; int e = T->phase;
    int inb = e & 1, outb = inb ^ 1;
    int64_t lo = S->own0[g], hi = S->own0[g + 1];
    int64_t ntiles = (hi - lo + S->tile_words - 1) / S->tile_words;
    for (;;) {
        int32_t t = atomic_fetch_add(&S->tile_next[g], 1);
        if (t >= ntiles || atomic_load(&S->err)) break;
        int64_t w0 = lo + (int64_t)t * S->tile_words, w1 = w0 + S->tile_words;
        if (w1 > hi) w1 = hi;
        /* consumer wait (reading R5): Jacobi reads neighbour rows produced remotely */
        if (S->workload == 1 && e > 0) {
            int64_t N = S->N;
            int64_t r0 = w0 / N, r1 = (w1 - 1) / N;
            int64_t need[2] = { (r0 - 1) * N, (r1 + 1) * N };
            for (int q = 0; q < 2; ++q) {
                int64_t wq = need[q];
                if (wq < 0 || wq >= N * N || (wq >= lo && wq < hi)) continue;
                for (int64_t x = wq; x < wq + N; x += 1) {   /* every chunk covering the row */
                    int owner = 0; while (!(x >= S->own0[owner] && x < S->own0[owner + 1])) ++owner;
                    int64_t gc = S->chunk0[owner] + proto_chunk_of(S, owner, x);
                    while (atomic_load_explicit(&S->arrive[g][inb * S->nchunks_total + gc],
                                                memory_order_acquire) < (uint32_t)e) {
                        if (atomic_load(&S->err)) return NULL;
                        sched_yield();
                    }
                }
            }
        }
        /* compute + instrumented store into the LOCAL replica (L123), with per-tile tally */
        int64_t tally_c = -1, tally_b = 0;
        for (int64_t k = w0; k < w1; ++k) {
            uint32_t v;
            if (S->workload == 0) {
                v = oracle_micro_word((uint64_t)k, (uint32_t)e, S->seed, S->K);
            } else {
                int64_t N = S->N, i = k / N, j = k % N;
                const uint32_t *in = S->rep[g][inb];
                if (i == 0 || j == 0 || i == N - 1 || j == N - 1) v = in[k];
                else {
                    float vert = as_f(in[k - N]) + as_f(in[k + N]);
                    float horz = as_f(in[k - 1]) + as_f(in[k + 1]);
                    v = as_u(0.25f * (vert + horz));
                }
            }
            S->rep[g][outb][k] = v;
            int64_t c = proto_chunk_of(S, g, k);
            if (c != tally_c) {
                if (tally_c >= 0) {
                    int64_t old = atomic_fetch_add_explicit(&S->counter[g][tally_c], tally_b,
                                                            memory_order_release);
                    if (old + tally_b > S->expected[g][tally_c]) proto_fail(S, -2);
                }
                tally_c = c; tally_b = 0;
            }
            tally_b += 4;
            maybe_yield(&T->rng);
        }
        if (tally_c >= 0) {
            int64_t old = atomic_fetch_add_explicit(&S->counter[g][tally_c], tally_b, memory_order_release);
            if (old + tally_b > S->expected[g][tally_c]) proto_fail(S, -2);
        }
    }
    atomic_fetch_sub(&S->producers_left[g], 1);
    return NULL;
}

/* agent thread: polls counters, pushes ready chunks to every peer, raises flags */
static void *proto_agent(void *arg)
{
    proto_thr *T = (proto_thr *)arg; proto_t *S = T->S; int g = T->g; int e = T->phase;
    int outb = (e & 1) ^ 1;
    int64_t nown = S->chunk0[g + 1] - S->chunk0[g];
    /* static ownership: agent id handles chunks c with c % A == id (reading R4) */
    for (int64_t c = T->id; c < nown; c += S->A) {
        int64_t v;
        while ((v = atomic_load_explicit(&S->counter[g][c], memory_order_acquire)) != S->expected[g][c]) {
            if (v > S->expected[g][c]) { proto_fail(S, -2); return NULL; }
            if (atomic_load(&S->err)) return NULL;
            sched_yield();
        }
        atomic_store_explicit(&S->counter[g][c], 0, memory_order_relaxed); /* reset for next phase */
        int64_t gc = S->chunk0[g] + c;
        int64_t w0 = S->own0[g] + c * S->chunk_words, w1 = w0 + S->chunk_words;
        if (w1 > S->own0[g + 1]) w1 = S->own0[g + 1];
        for (int p = 0; p < S->G; ++p) {
            if (p == g) continue;
            /* credit: p must have finished phase e-1 before its buffer is overwritten (R6) */
            while (atomic_load_explicit(&S->done[g][p], memory_order_acquire) < (uint32_t)e) {
                if (atomic_load(&S->err)) return NULL;
                sched_yield();
            }
            memcpy(S->rep[p][outb] + w0, S->rep[g][outb] + w0, sizeof(uint32_t) * (size_t)(w1 - w0));
            atomic_fetch_add(&S->deliv[g][gc * S->G + p], 1);
            atomic_store_explicit(&S->arrive[p][outb * S->nchunks_total + gc], (uint32_t)(e + 1),
                                  memory_order_release);
            maybe_yield(&T->rng);
        }
    }
    return NULL;
}

typedef struct { proto_t *S; int g; } proto_rank_arg;

static void *proto_rank(void *arg)
{
    proto_rank_arg *R = (proto_rank_arg *)arg; proto_t *S = R->S; int g = R->g;
    pthread_t th[64]; proto_thr ta[64];
    for (int e = 0; e < S->phases && !atomic_load(&S->err); ++e) {
        atomic_store(&S->tile_next[g], 0);
        atomic_store(&S->producers_left[g], S->P);
        int n = 0;
        for (int i = 0; i < S->P + S->A; ++i) {
            ta[n].S = S; ta[n].g = g; ta[n].id = i < S->P ? i : i - S->P; ta[n].phase = e;
            ta[n].rng = S->rng_seed * 0x9E3779B97F4A7C15ULL + (uint64_t)(g * 1000 + e * 64 + i + 1);
            pthread_create(&th[n], NULL, i < S->P ? proto_producer : proto_agent, &ta[n]);
            ++n;
        }
        for (int i = 0; i < n; ++i) pthread_join(th[i], NULL);  /* kernel boundary */
        /* I1: every (owned chunk, dest) delivered exactly once this phase; then reset */
        for (int64_t c = S->chunk0[g]; c < S->chunk0[g + 1]; ++c)
            for (int p = 0; p < S->G; ++p) {
                int32_t want = p == g ? 0 : 1;
                if (atomic_exchange(&S->deliv[g][c * S->G + p], 0) != want) proto_fail(S, -1);
            }
        /* phase sync: credit done = e+1 to every peer (reading R6, L125 barrier semantics) */
        for (int p = 0; p < S->G; ++p)
            atomic_store_explicit(&S->done[p][g], (uint32_t)(e + 1), memory_order_release);
    }
    return NULL;
}

/* Runs the simulation.  init (workload words, full extent) seeds every replica's buffer 0
 * (identical initial replicas, reading R16).  out receives rank r's final buffer for r = 0..G-1
 * concatenated (G * words).  Returns 0 or a negative invariant code. */
int oracle_proto_run(int G, int P, int A, int workload, int64_t N_or_W, int64_t chunk_words,
                     int64_t tile_words, int phases, uint32_t seed, int K, uint64_t rng_seed,
                     const uint32_t *init, uint32_t *out)
{
    if (G < 1 || G > PROTO_MAXG || P < 1 || A < 1 || P + A > 64 || chunk_words < 1) return -10;
    proto_t *S = (proto_t *)calloc(1, sizeof(proto_t));
    if (!S) return -11;
    S->G = G; S->P = P; S->A = A; S->workload = workload; S->N = N_or_W;
    S->chunk_words = chunk_words; S->tile_words = tile_words; S->phases = phases;
    S->seed = seed; S->K = K; S->rng_seed = rng_seed;
    int64_t W = workload == 1 ? N_or_W * N_or_W : N_or_W;
    /* ownership: Jacobi rows split evenly (ragged last), micro words split evenly */
    for (int g = 0; g <= G; ++g) {
        if (workload == 1) S->own0[g] = ((N_or_W * g) / G) * N_or_W;
        else S->own0[g] = (W * g) / G;
    }
    S->chunk0[0] = 0;
    for (int g = 0; g < G; ++g) {
        int64_t len = S->own0[g + 1] - S->own0[g];
        S->chunk0[g + 1] = S->chunk0[g] + (len + chunk_words - 1) / chunk_words;
    }
    S->nchunks_total = S->chunk0[G];
    int rc = 0;
    for (int g = 0; g < G; ++g) {
        for (int b = 0; b < 2; ++b) {
            S->rep[g][b] = (uint32_t *)malloc(sizeof(uint32_t) * (size_t)(W ? W : 1));
            if (init) memcpy(S->rep[g][b], init, sizeof(uint32_t) * (size_t)W);
            else memset(S->rep[g][b], 0, sizeof(uint32_t) * (size_t)W);
        }
        int64_t nown = S->chunk0[g + 1] - S->chunk0[g];
        S->counter[g] = (_Atomic int64_t *)calloc((size_t)(nown ? nown : 1), sizeof(int64_t));
        S->expected[g] = (int64_t *)calloc((size_t)(nown ? nown : 1), sizeof(int64_t));
        for (int64_t c = 0; c < nown; ++c) {
            int64_t w0 = S->own0[g] + c * chunk_words, w1 = w0 + chunk_words;
            if (w1 > S->own0[g + 1]) w1 = S->own0[g + 1];
            S->expected[g][c] = 4 * (w1 - w0);
        }
        S->deliv[g] = (_Atomic int32_t *)calloc((size_t)(S->nchunks_total * G + 1), sizeof(int32_t));
        S->arrive[g] = (_Atomic uint32_t *)calloc((size_t)(2 * S->nchunks_total + 1), sizeof(uint32_t));
    }
    pthread_t rt[PROTO_MAXG]; proto_rank_arg ra[PROTO_MAXG];
    for (int g = 0; g < G; ++g) { ra[g].S = S; ra[g].g = g; pthread_create(&rt[g], NULL, proto_rank, &ra[g]); }
    for (int g = 0; g < G; ++g) pthread_join(rt[g], NULL);
    rc = atomic_load(&S->err);
    if (rc == 0) {
        /* I2: counters back to zero (every chunk reached expected and was reset exactly once) */
        for (int g = 0; g < G; ++g)
            for (int64_t c = 0; c < S->chunk0[g + 1] - S->chunk0[g]; ++c)
                if (atomic_load(&S->counter[g][c]) != 0) rc = -2;
        /* I3: every flag of the last written buffer carries the last generation */
        int lastb = (phases & 1);
        for (int g = 0; g < G && rc == 0; ++g)
            for (int p = 0; p < G; ++p) {
                if (p == g || phases == 0) continue;
                for (int64_t gc = S->chunk0[p]; gc < S->chunk0[p + 1]; ++gc)
                    if (atomic_load(&S->arrive[g][lastb * S->nchunks_total + gc]) != (uint32_t)phases) rc = -3;
            }
    }
    if (out) {
        int lastb = phases & 1;
        for (int g = 0; g < G; ++g) memcpy(out + (size_t)g * (size_t)W, S->rep[g][lastb], sizeof(uint32_t) * (size_t)W);
    }
    for (int g = 0; g < G; ++g) {
        free(S->rep[g][0]); free(S->rep[g][1]); free((void *)S->counter[g]); free(S->expected[g]);
        free((void *)S->deliv[g]); free((void *)S->arrive[g]);
    }
    free(S);
    return rc;
}

/* ------------------------------------------------------------------------------------------ */
/* Banded Jacobi (Sec. IV-C: "the Jacobi solver for banded matrices ... iteratively
 * computes the solution vector using Jacobi's method").  A in DIA layout
 * a[(o+w)*N + i] = A[i][i+o].  Reading R19: fp32, the off-diagonal sum accumulated in the order
 * o = -w .. w (o != 0, 0 <= i+o < N), each term a*x rounded then added (no FMA), then
 * x'[i] = (b[i] - sum) / A[i][i] (IEEE division).  x holds x^0 on entry and x^iters on return. */
int oracle_banded_jacobi(const float *a, const float *b, float *x, int64_t N, int64_t w, int iters)
{
    float *t = (float *)malloc(sizeof(float) * (size_t)(N ? N : 1));
    if (!t) return -1;
    float *cur = x, *nxt = t;
    for (int k = 0; k < iters; ++k) {
#pragma omp parallel for schedule(static)
        for (int64_t i = 0; i < N; ++i) {
            float sum = 0.0f;
            for (int64_t o = -w; o <= w; ++o) {
                if (o == 0 || i + o < 0 || i + o >= N) continue;
                float term = a[(o + w) * N + i] * cur[i + o];
                sum = sum + term;
            }
            nxt[i] = (b[i] - sum) / a[w * N + i];
        }
        float *s = cur; cur = nxt; nxt = s;
    }
    if (cur != x) memcpy(x, cur, sizeof(float) * (size_t)N);
    free(t);
    return 0;
}
