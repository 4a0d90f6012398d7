// graph.cu -- graph workloads of the PROACT hot path: PageRank (config 3) and SSSP (config 4).
//
// PAPER.md Sec. IV-C: PageRank "assigns a 'Page-rank score' to web pages based on their
// importance" (L265); SSSP: "In each iteration, every vertex computes its shortest distance from
// the source vertex using the Bellman-Ford algorithm" (L267).  Both are destination-partitioned:
// rank g owns a contiguous, chunk-aligned, in-edge-balanced vertex range and pulls over the
// in-edges (CSC) of its vertices, reading the replicated vertex vector of the previous phase
// (waited for with proact::wait_all) and writing its slice of the next one through proact::put
// with one release commit per 4 KiB tile (a2, a3).
//   PageRank (readings R11/R12): the replicated vector is contrib[u] = r[u] / out(u) (fp32,
//     0 for dangling u); r'[v] = (float)((1-d)/V + d * sum_{u->v} contrib[u]) with the sum in
//     fp64; each vertex also keeps r'[v] locally.
//   SSSP (reading R13): int32 distances, synchronous Bellman-Ford; the region is SPARSE: a
//     source u is relaxed only if its chunk changed in the previous phase (arrival flag bit /
//     local changed stamp), a chunk is pushed only if it changed now or in the previous phase.
// Hubs (in-degree > HEAVY) are reduced by the whole CTA after the tile's light vertices.
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <cstdio>
#include <vector>

#include "proact.h"
#include "proact_device.cuh"
#include "proact_workloads.h"

using proact::launch_ctx;
using proact::region_dev;

namespace {

constexpr int GB = 256;            // threads per CTA
constexpr int GT = 1024;           // vertices per tile (4 KiB of output, the paper's L279)
constexpr int GL = 8;              // lanes per light vertex
constexpr uint32_t HEAVY = 2048;   // in-degree above which the whole CTA reduces a vertex
constexpr int MAXHEAVY = 64;       // per-tile hub list (overflow: the group does it itself)

struct GraphDev {
    const uint32_t *colptr;   // [nv + 1]
    const uint32_t *rowidx;   // [E_own] source vertex ids
    const int32_t *w;         // [E_own] weights (SSSP) or nullptr
    const uint32_t *outdeg;   // [V] global out-degree (multi-edges counted)
    float *r_own;             // [nv] PageRank values of my vertices
    uint32_t V, v0, nv, pad;
};

struct Graph {
    bool used = false;
    uint32_t V = 0, v0 = 0, nv = 0;
    uint64_t E_own = 0;
    uint32_t *colptr = nullptr, *rowidx = nullptr, *outdeg = nullptr;
    int32_t *w = nullptr;
    float *r_own = nullptr;
};
constexpr int MAXGRAPH = 4;
thread_local Graph graphs[MAXGRAPH];

#define GCK(call)                                                                        \
    do {                                                                                 \
        cudaError_t e_ = (call);                                                         \
        if (e_ != cudaSuccess) {                                                         \
            fprintf(stderr, "[proact] %s: %s (%s:%d)\n", #call, cudaGetErrorString(e_), \
                    __FILE__, __LINE__);                                                 \
            return PROACT_ERR_CUDA;                                                      \
        }                                                                                \
    } while (0)

// ------------------------------------------------------------------ CSC construction kernels
__global__ void count_kernel(const uint32_t *src, const uint32_t *dst, uint64_t E, uint32_t v0, uint32_t v1,
                             uint32_t *indeg, uint32_t *outdeg)
{
    for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < E; e += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t d = dst[e];
        if (indeg && d >= v0 && d < v1) atomicAdd(&indeg[d - v0], 1u);
        if (outdeg) atomicAdd(&outdeg[src[e]], 1u);
    }
}

// exclusive scan, 3 passes: per-block scan of 4096 items (+ block totals), scan of totals,
// add offsets.  n <= 2^26.
constexpr int SB = 1024, SI = 4;
__global__ void scan_blocks(const uint32_t *in, uint32_t *out, uint32_t *tot, uint64_t n)
{
    __shared__ uint32_t s[SB];
    const uint64_t base = (uint64_t)blockIdx.x * SB * SI + (uint64_t)threadIdx.x * SI;
    uint32_t v[SI], sum = 0;
    for (int k = 0; k < SI; ++k) {
        v[k] = base + k < n ? in[base + k] : 0u;
        sum += v[k];
    }
    s[threadIdx.x] = sum;
    __syncthreads();
    for (int off = 1; off < SB; off <<= 1) {   // Hillis-Steele inclusive scan of thread sums
        const uint32_t x = threadIdx.x >= (unsigned)off ? s[threadIdx.x - off] : 0u;
        __syncthreads();
        s[threadIdx.x] += x;
        __syncthreads();
    }
    uint32_t run = s[threadIdx.x] - sum;
    for (int k = 0; k < SI; ++k) {
        if (base + k < n) out[base + k] = run;
        run += v[k];
    }
    if (threadIdx.x == SB - 1) tot[blockIdx.x] = s[SB - 1];
}
__global__ void scan_totals(uint32_t *tot, uint32_t nb)
{
    __shared__ uint32_t s[SB];
    const uint32_t per = (nb + SB - 1) / SB;
    uint32_t sum = 0;
    for (uint32_t k = 0; k < per; ++k) {
        const uint32_t i = threadIdx.x * per + k;
        if (i < nb) sum += tot[i];
    }
    s[threadIdx.x] = sum;
    __syncthreads();
    for (int off = 1; off < SB; off <<= 1) {
        const uint32_t x = threadIdx.x >= (unsigned)off ? s[threadIdx.x - off] : 0u;
        __syncthreads();
        s[threadIdx.x] += x;
        __syncthreads();
    }
    uint32_t run = s[threadIdx.x] - sum;
    for (uint32_t k = 0; k < per; ++k) {
        const uint32_t i = threadIdx.x * per + k;
        if (i < nb) {
            const uint32_t t = tot[i];
            tot[i] = run;
            run += t;
        }
    }
}
__global__ void scan_add(uint32_t *out, const uint32_t *tot, uint64_t n)
{
    const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
    if (i < n) out[i] += tot[i / (SB * SI)];
}

int exclusive_scan(const uint32_t *in, uint32_t *out, uint64_t n, cudaStream_t s)
{
    if (n == 0) return PROACT_OK;
    const uint32_t nb = (uint32_t)((n + SB * SI - 1) / (SB * SI));
    uint32_t *tot = nullptr;
    GCK(cudaMallocAsync((void **)&tot, 4 * (size_t)nb, s));
    scan_blocks<<<nb, SB, 0, s>>>(in, out, tot, n);
    scan_totals<<<1, SB, 0, s>>>(tot, nb);
    scan_add<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(out, tot, n);
    GCK(cudaGetLastError());
    GCK(cudaFreeAsync(tot, s));
    return PROACT_OK;
}

__global__ void scatter_kernel(const uint32_t *src, const uint32_t *dst, const int32_t *wsrc, uint64_t E,
                               uint32_t v0, uint32_t v1, uint32_t *cursor, uint32_t *rowidx, int32_t *w)
{
    for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < E; e += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t d = dst[e];
        if (d >= v0 && d < v1) {
            const uint32_t pos = atomicAdd(&cursor[d - v0], 1u);
            rowidx[pos] = src[e];
            if (w) w[pos] = wsrc[e];
        }
    }
}

// ------------------------------------------------------------------ phase kernels
struct PrParams {
    GraphDev g;
    int region_in, region_out;
    double d, base;   // damping, (1-d)/V
};
struct SsspParams {
    GraphDev g;
    int region_in, region_out;
    int first;        // phase 0: every source is "changed"
    int pad;
};

// L2 policies: the CSC stream (read once per phase) is evict-first, the gathered vertex vector
// (64 MiB at RMAT-24, fits the 126 MB L2) evict-last.
__device__ __forceinline__ uint64_t pol_first()
{
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t pol_last()
{
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint32_t ld_stream_u(const uint32_t *p, uint64_t pol)
{
    uint32_t v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ int32_t ld_stream_i(const int32_t *p, uint64_t pol)
{
    int32_t v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
}
// The gathered vector: written by peers' agents during the previous phase (all arrived: the CTA
// waited with wait_all before its first load, and nothing rewrites it this phase), so the
// read-only path is coherent here.
__device__ __forceinline__ float ld_gather_f(const float *p, uint64_t pol)
{
    float v;
    asm volatile("ld.global.nc.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ int32_t ld_gather_i(const int32_t *p, uint64_t pol)
{
    int32_t v;
    asm volatile("ld.global.nc.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ uint32_t ld_nc_u(const uint32_t *p)
{
    uint32_t v;
    asm volatile("ld.global.nc.u32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}

__device__ __forceinline__ void pr_finish(const launch_ctx &lc, const PrParams &p, uint32_t v, double s)
{
    const float r = (float)(p.base + p.d * s);
    p.g.r_own[v - p.g.v0] = r;
    const uint32_t od = p.g.outdeg[v];
    const float c = od ? __fdiv_rn(r, (float)od) : 0.f;
    proact::put(lc, p.region_out, (uint64_t)v * 4, c);
}

__device__ __forceinline__ double block_sum_f64(double x, double *red)
{
    for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xFFFFFFFFu, x, o);
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = x;
    __syncthreads();
    double t = 0.0;
    if (threadIdx.x < 32) {
        t = threadIdx.x < (GB / 32) ? red[threadIdx.x] : 0.0;
        for (int o = 16; o > 0; o >>= 1) t += __shfl_xor_sync(0xFFFFFFFFu, t, o);
    }
    __syncthreads();
    return t;   // valid in thread 0
}

// sum over edges [e0, e1) with stride `step` starting at `first`, 4 gathers in flight per lane
__device__ __forceinline__ double pr_sum(const uint32_t *rowidx, const float *cin, uint32_t first, uint32_t e1,
                                         uint32_t step, uint64_t pf, uint64_t pl)
{
    double s = 0.0;
    uint32_t e = first;
    for (; e + 3 * step < e1; e += 4 * step) {
        const uint32_t u0 = ld_stream_u(rowidx + e, pf), u1 = ld_stream_u(rowidx + e + step, pf);
        const uint32_t u2 = ld_stream_u(rowidx + e + 2 * step, pf), u3 = ld_stream_u(rowidx + e + 3 * step, pf);
        const float c0 = ld_gather_f(cin + u0, pl), c1 = ld_gather_f(cin + u1, pl);
        const float c2 = ld_gather_f(cin + u2, pl), c3 = ld_gather_f(cin + u3, pl);
        s += (double)c0;
        s += (double)c1;
        s += (double)c2;
        s += (double)c3;
    }
    for (; e < e1; e += step) s += (double)ld_gather_f(cin + ld_stream_u(rowidx + e, pf), pl);
    return s;
}

// Light vertices of a tile are fetched dynamically by 8-lane groups (balances skewed degrees);
// hubs are queued and reduced by the whole CTA afterwards.
__global__ void __launch_bounds__(GB, 6) pagerank_kernel(launch_ctx lc, PrParams p)
{
    if (proact::agent_dispatch(lc)) return;
    __shared__ uint32_t heavy[MAXHEAVY];
    __shared__ uint32_t nheavy, next;
    __shared__ double red[GB / 32];
    const float *cin = reinterpret_cast<const float *>(lc.ctx->region[p.region_in].base);
    const uint32_t ntiles = (p.g.nv + GT - 1) / GT;
    const uint32_t sub = threadIdx.x % GL, lead = (threadIdx.x & 31) & ~(GL - 1);
    const uint32_t gmask = 0xFFu << lead;
    const uint64_t pf = pol_first(), pl = pol_last();
    bool waited = false;
    for (uint32_t t = proact::producer_block(lc); t < ntiles; t += proact::producer_grid(lc)) {
        if (!waited) {   // (a7) every chunk of the previous generation is in my replica
            if (threadIdx.x == 0) proact::wait_all(lc, p.region_in);
            waited = true;
        }
        if (threadIdx.x == 0) {
            nheavy = 0;
            next = 0;
        }
        __syncthreads();
        const uint32_t lo = p.g.v0 + t * GT, hi = min(lo + GT, p.g.v0 + p.g.nv);
        for (;;) {   // a warp takes 4 vertices (one per 8-lane group); control flow stays converged
            uint32_t k4 = 0;
            if ((threadIdx.x & 31) == 0) k4 = atomicAdd(&next, 4u);
            k4 = __shfl_sync(0xFFFFFFFFu, k4, 0);
            if (lo + k4 >= hi) break;
            const uint32_t v = lo + k4 + ((threadIdx.x & 31) >> 3);
            uint32_t e0 = 0, e1 = 0;
            if (v < hi) {
                e0 = p.g.colptr[v - p.g.v0];
                e1 = p.g.colptr[v - p.g.v0 + 1];
            }
            bool queued = false;
            if (sub == 0 && e1 - e0 > HEAVY) {
                const uint32_t h = atomicAdd(&nheavy, 1u);
                if (h < MAXHEAVY) { heavy[h] = v; queued = true; }
            }
            queued = __shfl_sync(0xFFFFFFFFu, queued, lead);
            if (queued) e1 = e0;   // the hub is reduced by the whole CTA below
            const uint32_t maxd = __reduce_max_sync(0xFFFFFFFFu, e1 - e0);
            double s = 0.0;
            for (uint32_t b = sub; b < maxd; b += 4 * GL) {
                uint32_t u[4];
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const uint32_t e = e0 + b + q * GL;
                    u[q] = e < e1 ? ld_stream_u(p.g.rowidx + e, pf) : 0xFFFFFFFFu;
                }
#pragma unroll
                for (int q = 0; q < 4; ++q)
                    if (u[q] != 0xFFFFFFFFu) s += (double)ld_gather_f(cin + u[q], pl);
            }
            for (int o = GL / 2; o > 0; o >>= 1) s += __shfl_xor_sync(0xFFFFFFFFu, s, o);
            if (sub == 0 && v < hi && !queued) pr_finish(lc, p, v, s);
        }
        __syncthreads();
        const uint32_t nh = min(nheavy, (uint32_t)MAXHEAVY);
        for (uint32_t h = 0; h < nh; ++h) {   // hubs: the whole CTA, fp64 tree reduction
            const uint32_t v = heavy[h];
            const uint32_t e0 = p.g.colptr[v - p.g.v0], e1 = p.g.colptr[v - p.g.v0 + 1];
            double s = pr_sum(p.g.rowidx, cin, e0 + threadIdx.x, e1, GB, pf, pl);
            s = block_sum_f64(s, red);
            if (threadIdx.x == 0) pr_finish(lc, p, v, s);
        }
        __syncthreads();
        if (threadIdx.x == 0) proact::commit_span(lc, p.region_out, (uint64_t)lo * 4, (uint64_t)(hi - lo) * 4);
    }
}

// relax edges [first, e1) stride `step` into best; sources filtered by the changed-chunk bitmap
__device__ __forceinline__ int32_t sssp_relax(const SsspParams &p, const uint32_t *chg, uint32_t cshift,
                                              uint32_t cdiv, const int32_t *din, uint32_t first, uint32_t e1,
                                              uint32_t step, int32_t best, uint64_t pf, uint64_t pl)
{
    for (uint32_t e = first; e < e1; e += 2 * step) {
        const bool has1 = e + step < e1;
        const uint32_t u0 = ld_stream_u(p.g.rowidx + e, pf);
        const uint32_t u1 = has1 ? ld_stream_u(p.g.rowidx + e + step, pf) : 0u;
        const uint32_t g0 = cdiv ? u0 / cdiv : u0 >> cshift, g1 = cdiv ? u1 / cdiv : u1 >> cshift;
        const bool a0 = p.first || (chg[g0 >> 5] >> (g0 & 31) & 1u);
        const bool a1 = has1 && (p.first || (chg[g1 >> 5] >> (g1 & 31) & 1u));
        if (a0) {
            const int32_t du = ld_gather_i(din + u0, pl);
            if (du != INT32_MAX) {
                const int64_t cand = (int64_t)du + (int64_t)ld_stream_i(p.g.w + e, pf);
                if (cand < (int64_t)best) best = (int32_t)cand;
            }
        }
        if (a1) {
            const int32_t du = ld_gather_i(din + u1, pl);
            if (du != INT32_MAX) {
                const int64_t cand = (int64_t)du + (int64_t)ld_stream_i(p.g.w + e + step, pf);
                if (cand < (int64_t)best) best = (int32_t)cand;
            }
        }
    }
    return best;
}

__device__ __forceinline__ int32_t block_min_i32(int32_t x, int32_t *red)
{
    for (int o = 16; o > 0; o >>= 1) x = min(x, __shfl_xor_sync(0xFFFFFFFFu, x, o));
    if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = x;
    __syncthreads();
    int32_t t = INT32_MAX;
    if (threadIdx.x < 32) {
        t = threadIdx.x < (GB / 32) ? red[threadIdx.x] : INT32_MAX;
        for (int o = 16; o > 0; o >>= 1) t = min(t, __shfl_xor_sync(0xFFFFFFFFu, t, o));
    }
    __syncthreads();
    return t;
}

constexpr uint32_t CHG_WORDS = 4096;   // changed-chunk bitmap in shared memory (<= 131072 chunks)

__global__ void __launch_bounds__(GB, 6) sssp_kernel(launch_ctx lc, SsspParams p)
{
    if (proact::agent_dispatch(lc)) return;
    __shared__ uint32_t heavy[MAXHEAVY];
    __shared__ uint32_t nheavy, next;
    __shared__ int32_t red[GB / 32];
    __shared__ uint32_t chg[CHG_WORDS];
    const region_dev &Ri = lc.ctx->region[p.region_in];
    const int32_t *din = reinterpret_cast<const int32_t *>(Ri.base);
    const uint32_t ntiles = (p.g.nv + GT - 1) / GT;
    const uint32_t sub = threadIdx.x % GL, lead = (threadIdx.x & 31) & ~(GL - 1);
    const uint32_t gmask = 0xFFu << lead;
    const uint64_t pf = pol_first(), pl = pol_last();
    // source vertex -> global chunk id: rank slices are chunk-aligned, so it is u*4/chunk_bytes
    const uint32_t cv = Ri.chunk_bytes / 4;   // vertices per chunk
    const uint32_t cshift = __popc(cv) == 1 ? (uint32_t)(__ffs(cv) - 1) : 0u, cdiv = __popc(cv) == 1 ? 0u : cv;
    bool ready = false;
    for (uint32_t t = proact::producer_block(lc); t < ntiles; t += proact::producer_grid(lc)) {
        if (!ready) {   // (a7) wait for the previous generation, then snapshot its changed bits
            if (threadIdx.x == 0) proact::wait_all(lc, p.region_in);
            __syncthreads();
            const uint32_t gen = lc.gen[p.region_in];
            const bool agent = proact::uses_agent(lc);
            for (uint32_t wi = threadIdx.x; wi < CHG_WORDS && wi * 32 < Ri.n_total; wi += GB) {
                uint32_t bits = 0;
                for (uint32_t b = 0; b < 32; ++b) {
                    const uint32_t g = wi * 32 + b;
                    if (g >= Ri.n_total) break;
                    bool c;
                    if (g >= Ri.chunk0 && g < Ri.chunk0 + Ri.n_own) c = Ri.changed_gen[g - Ri.chunk0] == gen;
                    else c = !agent || (ld_nc_u(Ri.arrive + g) & 1u);   // no flags without the agent
                    bits |= (uint32_t)c << b;
                }
                chg[wi] = bits;
            }
            ready = true;
        }
        if (threadIdx.x == 0) {
            nheavy = 0;
            next = 0;
        }
        __syncthreads();
        const uint32_t lo = p.g.v0 + t * GT, hi = min(lo + GT, p.g.v0 + p.g.nv);
        bool changed = false;
        for (;;) {   // a warp takes 4 vertices (one per 8-lane group); control flow stays converged
            uint32_t k4 = 0;
            if ((threadIdx.x & 31) == 0) k4 = atomicAdd(&next, 4u);
            k4 = __shfl_sync(0xFFFFFFFFu, k4, 0);
            if (lo + k4 >= hi) break;
            const uint32_t v = lo + k4 + ((threadIdx.x & 31) >> 3);
            uint32_t e0 = 0, e1 = 0;
            int32_t old = INT32_MAX;
            if (v < hi) {
                e0 = p.g.colptr[v - p.g.v0];
                e1 = p.g.colptr[v - p.g.v0 + 1];
                old = din[v];
            }
            bool queued = false;
            if (sub == 0 && e1 - e0 > HEAVY) {
                const uint32_t h = atomicAdd(&nheavy, 1u);
                if (h < MAXHEAVY) { heavy[h] = v; queued = true; }
            }
            queued = __shfl_sync(0xFFFFFFFFu, queued, lead);
            if (queued) e1 = e0;
            const uint32_t maxd = __reduce_max_sync(0xFFFFFFFFu, e1 - e0);
            int32_t best = old;
            for (uint32_t b = sub; b < maxd; b += 2 * GL)
                best = sssp_relax(p, chg, cshift, cdiv, din, e0 + b, min(e1, e0 + b + 2 * GL), GL, best, pf, pl);
            for (int o = GL / 2; o > 0; o >>= 1) best = min(best, __shfl_xor_sync(0xFFFFFFFFu, best, o));
            if (sub == 0 && v < hi && !queued) {
                proact::put(lc, p.region_out, (uint64_t)v * 4, best);
                changed |= best != old;
            }
        }
        __syncthreads();
        const uint32_t nh = min(nheavy, (uint32_t)MAXHEAVY);
        for (uint32_t h = 0; h < nh; ++h) {
            const uint32_t v = heavy[h];
            const uint32_t e0 = p.g.colptr[v - p.g.v0], e1 = p.g.colptr[v - p.g.v0 + 1];
            const int32_t old = din[v];
            int32_t best = sssp_relax(p, chg, cshift, cdiv, din, e0 + threadIdx.x, e1, GB, INT32_MAX, pf, pl);
            best = min(block_min_i32(best, red), old);
            if (threadIdx.x == 0) {
                proact::put(lc, p.region_out, (uint64_t)v * 4, best);
                changed |= best != old;
            }
        }
        // per-tile chunk state (SPARSE region): changed now -> flag bit + vote; push if changed
        // now or in the previous phase (the peers' ping-pong copy holds d^{k-1}, reading R13)
        const int any = __syncthreads_or(changed);
        if (threadIdx.x == 0) {
            const uint64_t off = (uint64_t)lo * 4;
            const bool prev = !p.first && proact::local_changed(lc, p.region_in, off);
            if (any) {
                proact::mark_changed(lc, p.region_out, off);
                proact::vote(lc);
            }
            if (any || prev) proact::mark_push(lc, p.region_out, off);
            proact::commit_span(lc, p.region_out, off, (uint64_t)(hi - lo) * 4);
        }
    }
}

__global__ void pr_init_kernel(float *contrib, const uint32_t *outdeg, uint32_t V, float r0)
{
    for (uint32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < V; u += gridDim.x * blockDim.x)
        contrib[u] = outdeg[u] ? __fdiv_rn(r0, (float)outdeg[u]) : 0.f;
}

int graph_dev(int id, GraphDev *g)
{
    if (id < 0 || id >= MAXGRAPH || !graphs[id].used) return PROACT_ERR_INVALID;
    const Graph &G = graphs[id];
    g->colptr = G.colptr;
    g->rowidx = G.rowidx;
    g->w = G.w;
    g->outdeg = G.outdeg;
    g->r_own = G.r_own;
    g->V = G.V;
    g->v0 = G.v0;
    g->nv = G.nv;
    g->pad = 0;
    return PROACT_OK;
}

}  // namespace

// ================================================================ C entry points
extern "C" {

int proact_graph_partition(const uint32_t *d_dst, unsigned long long E, unsigned V, int G, unsigned align,
                           unsigned *bounds, void *stream)
{
    if (!d_dst || !bounds || G < 1 || align == 0 || V == 0) return PROACT_ERR_INVALID;
    cudaStream_t s = (cudaStream_t)stream;
    uint32_t *indeg = nullptr;
    GCK(cudaMalloc((void **)&indeg, 4 * (size_t)V));
    GCK(cudaMemsetAsync(indeg, 0, 4 * (size_t)V, s));
    if (E) count_kernel<<<1184, 256, 0, s>>>(d_dst, d_dst, E, 0, V, indeg, nullptr);
    GCK(cudaGetLastError());
    std::vector<uint32_t> h(V);
    GCK(cudaMemcpyAsync(h.data(), indeg, 4 * (size_t)V, cudaMemcpyDeviceToHost, s));
    GCK(cudaStreamSynchronize(s));
    GCK(cudaFree(indeg));
    return proact_partition_bounds(h.data(), V, G, align, bounds);
}

int proact_partition_bounds(const uint32_t *indeg, unsigned V, int G, unsigned align, unsigned *bounds)
{
    if (!indeg || !bounds || G < 1 || align == 0) return PROACT_ERR_INVALID;
    // bounds[g]: the align-multiple vertex whose in-edge prefix is closest to g*E/G (monotone)
    std::vector<uint64_t> cum((size_t)V + 1, 0);
    for (uint32_t v = 0; v < V; ++v) cum[v + 1] = cum[v] + indeg[v];
    auto dist = [&](uint64_t x, uint64_t t) { return cum[x] > t ? cum[x] - t : t - cum[x]; };
    bounds[0] = 0;
    for (int g = 1; g < G; ++g) {
        const uint64_t target = cum[V] * (uint64_t)g / (uint64_t)G;
        const uint64_t v = (uint64_t)(std::lower_bound(cum.begin(), cum.end(), target) - cum.begin());
        const uint64_t a = v / align * align, b = std::min<uint64_t>(a + align, V);
        const uint32_t pick = (uint32_t)(dist(a, target) <= dist(b, target) ? a : b);
        bounds[g] = std::min<unsigned>(V, std::max<unsigned>(pick, bounds[g - 1]));
    }
    bounds[G] = V;
    return PROACT_OK;
}

int proact_graph_build(const uint32_t *d_src, const uint32_t *d_dst, const int32_t *d_w, unsigned long long E,
                       unsigned V, unsigned v0, unsigned v1, void *stream)
{
    if (!d_src || !d_dst || v1 < v0 || v1 > V) return PROACT_ERR_INVALID;
    int id = -1;
    for (int k = 0; k < MAXGRAPH; ++k)
        if (!graphs[k].used) { id = k; break; }
    if (id < 0) return PROACT_ERR_NOMEM;
    cudaStream_t s = (cudaStream_t)stream;
    Graph G;
    G.V = V;
    G.v0 = v0;
    G.nv = v1 - v0;
    uint32_t *indeg = nullptr;
    GCK(cudaMalloc((void **)&indeg, 4 * ((size_t)G.nv + 1)));
    GCK(cudaMalloc((void **)&G.colptr, 4 * ((size_t)G.nv + 1)));
    GCK(cudaMalloc((void **)&G.outdeg, 4 * (size_t)V));
    GCK(cudaMalloc((void **)&G.r_own, 4 * ((size_t)G.nv + 1)));
    GCK(cudaMemsetAsync(indeg, 0, 4 * ((size_t)G.nv + 1), s));
    GCK(cudaMemsetAsync(G.outdeg, 0, 4 * (size_t)V, s));
    if (E) count_kernel<<<1184, 256, 0, s>>>(d_src, d_dst, E, v0, v1, indeg, G.outdeg);
    GCK(cudaGetLastError());
    int rc = exclusive_scan(indeg, G.colptr, (uint64_t)G.nv + 1, s);
    if (rc) return rc;
    uint32_t e_own = 0;
    GCK(cudaMemcpyAsync(&e_own, G.colptr + G.nv, 4, cudaMemcpyDeviceToHost, s));
    GCK(cudaStreamSynchronize(s));
    G.E_own = e_own;
    GCK(cudaMalloc((void **)&G.rowidx, 4 * ((size_t)e_own + 1)));
    if (d_w) GCK(cudaMalloc((void **)&G.w, 4 * ((size_t)e_own + 1)));
    GCK(cudaMemcpyAsync(indeg, G.colptr, 4 * ((size_t)G.nv + 1), cudaMemcpyDeviceToDevice, s));   // cursors
    if (E) scatter_kernel<<<1184, 256, 0, s>>>(d_src, d_dst, d_w, E, v0, v1, indeg, G.rowidx, G.w);
    GCK(cudaGetLastError());
    GCK(cudaFreeAsync(indeg, s));
    GCK(cudaStreamSynchronize(s));
    G.used = true;
    graphs[id] = G;
    return id;
}

int proact_graph_free(int id)
{
    if (id < 0 || id >= MAXGRAPH || !graphs[id].used) return PROACT_ERR_INVALID;
    Graph &G = graphs[id];
    cudaFree(G.colptr);
    cudaFree(G.rowidx);
    cudaFree(G.outdeg);
    cudaFree(G.r_own);
    if (G.w) cudaFree(G.w);
    G = Graph();
    return PROACT_OK;
}

int proact_graph_info(int id, unsigned long long *e_own, unsigned *v0, unsigned *nv)
{
    if (id < 0 || id >= MAXGRAPH || !graphs[id].used) return PROACT_ERR_INVALID;
    if (e_own) *e_own = graphs[id].E_own;
    if (v0) *v0 = graphs[id].v0;
    if (nv) *nv = graphs[id].nv;
    return PROACT_OK;
}

int proact_pagerank_init(int graph, int region, void *stream)
{
    GraphDev g;
    int rc = graph_dev(graph, &g);
    if (rc) return rc;
    proact_region_info ri;
    rc = proact_region_info_get(region, &ri);
    if (rc) return rc;
    if (ri.total_bytes != 4ull * g.V) return PROACT_ERR_INVALID;
    pr_init_kernel<<<1184, 256, 0, (cudaStream_t)stream>>>((float *)ri.replica_base, g.outdeg, g.V,
                                                           (float)(1.0 / (double)g.V));
    GCK(cudaGetLastError());
    return PROACT_OK;
}

int proact_pagerank_phase(int graph, int region_in, int region_out, double damping, void *stream)
{
    PrParams p;
    int rc = graph_dev(graph, &p.g);
    if (rc) return rc;
    proact_region_info ro;
    rc = proact_region_info_get(region_out, &ro);
    if (rc) return rc;
    if (ro.total_bytes != 4ull * p.g.V || ro.own_offset != 4ull * p.g.v0 || ro.own_bytes != 4ull * p.g.nv)
        return PROACT_ERR_INVALID;
    p.region_in = region_in;
    p.region_out = region_out;
    p.d = damping;
    p.base = (1.0 - damping) / (double)p.g.V;
    launch_ctx lc;
    void *args[2] = {&lc, &p};
    int regs[1] = {region_out};
    return proact_launch(regs, 1, (const void *)pagerank_kernel, 0, GB, args, 0, stream);
}

int proact_pagerank_ranks(int graph, float *d_out, void *stream)
{
    if (graph < 0 || graph >= MAXGRAPH || !graphs[graph].used) return PROACT_ERR_INVALID;
    if (graphs[graph].nv == 0) return PROACT_OK;   // empty slice: nothing to copy
    if (!d_out) return PROACT_ERR_INVALID;
    GCK(cudaMemcpyAsync(d_out, graphs[graph].r_own, 4 * (size_t)graphs[graph].nv, cudaMemcpyDeviceToDevice,
                        (cudaStream_t)stream));
    return PROACT_OK;
}

int proact_sssp_phase(int graph, int region_in, int region_out, int first, void *stream)
{
    SsspParams p;
    int rc = graph_dev(graph, &p.g);
    if (rc) return rc;
    if (!p.g.w) return PROACT_ERR_INVALID;
    proact_region_info ro;
    rc = proact_region_info_get(region_out, &ro);
    if (rc) return rc;
    if (ro.total_bytes != 4ull * p.g.V || ro.own_offset != 4ull * p.g.v0 || ro.own_bytes != 4ull * p.g.nv ||
        ro.chunk_bytes % 4096 || ro.n_total_chunks > 32u * CHG_WORDS)
        return PROACT_ERR_INVALID;
    p.region_in = region_in;
    p.region_out = region_out;
    p.first = first ? 1 : 0;
    p.pad = 0;
    launch_ctx lc;
    void *args[2] = {&lc, &p};
    int regs[1] = {region_out};
    return proact_launch(regs, 1, (const void *)sssp_kernel, 0, GB, args, 0, stream);
}

}  // extern "C"
