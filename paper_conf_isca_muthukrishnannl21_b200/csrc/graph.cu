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
#include <cstdlib>
#include <cstring>
#include <vector>

#include "proact.h"
#include "proact_device.cuh"
#include "proact_workloads.h"

using proact::launch_ctx;
using proact::region_dev;

namespace {

#ifndef PROACT_GB
#define PROACT_GB 256
#endif
constexpr int GB = PROACT_GB;      // threads per CTA
#ifndef PROACT_GT   // 512: PageRank 1.035 vs 1.065 ms at 1024 (smaller per-group accumulators leave
#define PROACT_GT 512 // more L1 as landing space for the gathers), SSSP unchanged
#endif
constexpr int GT = PROACT_GT;      // vertices per tile (2 KiB of output)
// consecutive in-edges per thread per round (merge path) and CTAs per SM, measured on B200
// (tools/sweep_graph.py): PageRank 4 / 8 (1.65 ms at RMAT-24; 8 / 6: 2.2 ms), SSSP 2 / 6
#ifndef PROACT_PR_RUN
#define PROACT_PR_RUN 4
#endif
#ifndef PROACT_PR_MINB
#define PROACT_PR_MINB 8
#endif
#ifndef PROACT_SSSP_RUN
#define PROACT_SSSP_RUN 2
#endif
#ifndef PROACT_SSSP_MINB
#define PROACT_SSSP_MINB 6
#endif
constexpr uint32_t SPLIT = 32768;  // max in-edges per work item: bigger tiles are split

// Work item = (vertex tile, in-edge sub-range).  Tiles whose in-edges exceed SPLIT (hubs) are
// split over several items (processed by different CTAs, split items first); their partial
// sums meet in a per-split-tile global accumulator and the last item to arrive finishes the
// tile.  Every item then carries about the same number of edges: the CTAs stay balanced on a
// power-law graph.
struct Item {
    uint32_t tile, e0, e1;   // edges [e0, e1) (local CSC indices)
    uint32_t nsplit;         // items of this tile (1 = unsplit)
    uint32_t slot;           // split-tile accumulator slot
    uint32_t run_pr;         // first entry of this item in runv_pr (PageRank runs of PR_RUN edges)
    uint32_t run_ss;         // first entry of this item in runv_ss (SSSP runs of SSSP_RUN edges)
    uint32_t run_ph;         // first entry of this item in runv_ph (hot-kernel runs of PRH_RUN edges)
    uint32_t run_p8;         // first entry of this item in runv_p8 (PageRank hot runs of PRH_RUN_PR edges)
};

struct GraphDev {
    const uint32_t *colptr;   // [nv + 1]
    const uint32_t *rowidx;   // [E_own] source vertex ids
    const int32_t *w;         // [E_own] weights (SSSP) or nullptr
    const uint32_t *outdeg;   // [V] global out-degree (multi-edges counted)
    float *r_own;             // [nv] PageRank values of my vertices
    const Item *items;        // [nitems]
    unsigned long long *acc_f;   // [nslot * GT] split-tile fixed-point sums (PageRank), zero between launches
    int32_t *acc_i;           // [nslot * GT] split-tile minima (SSSP), INT32_MAX between launches
    uint32_t *acc_cnt;        // [nslot] arrivals of a split tile's items
    const uint16_t *runv_pr;  // per PageRank run (RUN consecutive in-edges of an item): tile-local
    const uint16_t *runv_ss;  //   vertex of its first edge (the merge-path search, done once at build)
    const uint16_t *runv_ph;
    const uint16_t *runv_p8;
    const uint32_t *rowidx_h; // [E_own] rowidx with hot sources encoded as HOT_BIT | slot (nhot > 0)
    const uint32_t *hot_ids;  // [nhot] the hot sources (highest out-degree), ascending ids
    uint32_t V, v0, nv, nitems, nhot;
};

struct Graph {
    bool used = false;
    uint32_t V = 0, v0 = 0, nv = 0;
    uint64_t E_own = 0;
    uint32_t *colptr = nullptr, *rowidx = nullptr, *outdeg = nullptr;
    int32_t *w = nullptr;
    float *r_own = nullptr;
    Item *items = nullptr;
    uint32_t nitems = 0, nslot = 0;
    unsigned long long *acc_f = nullptr;
    int32_t *acc_i = nullptr;
    uint32_t *acc_cnt = nullptr;
    uint16_t *runv_pr = nullptr, *runv_ss = nullptr, *runv_ph = nullptr, *runv_p8 = nullptr;
    uint32_t *rowidx_h = nullptr, *hot_ids = nullptr;
    uint32_t nhot = 0;
    uint64_t e_hot = 0;   // my in-edges whose source is hot
    // SSSP push rounds (weighted graphs): my in-edges grouped by SOURCE, the private copy of the
    // previous round's input, the round's relaxation minima, the frontier's heavy sources
    uint64_t E_all = 0;                    // global edge count (the build's E)
    uint32_t *prp = nullptr;               // [V + 1] row pointers over global source ids
    uint32_t *pcol = nullptr;              // [E_own] local destination v - v0
    int32_t *pwt = nullptr;                // [E_own] weight
    int32_t *dprev = nullptr;              // [V] previous round's input distances
    int32_t *ptmp = nullptr;               // [nv] minima of the round, INT32_MAX between rounds
    uint32_t *ptouch = nullptr;            // [nv / 1024] a frontier edge reached the 4 KiB block
    uint2 *heavy = nullptr;                // [nheavy_max] pieces (source, first edge) of heavy frontier sources
    uint32_t nheavy_max = 0;
    uint32_t *pctl = nullptr;              // [4]: heavy pieces, barrier arrivals, barrier generation, claims
    unsigned long long *dcnt = nullptr;    // [2] per round parity: out-degree sum of my changed vertices
    unsigned long long *hcnt = nullptr;    // pinned: the last round's sum (read for the next decision)
    uint32_t round = 0;
    bool tracked = false;                  // the last round left dprev = its input
    int last_mode = 0;                     // 0 pull, 1 push (last launched round)
};
constexpr int MAXGRAPH = 4;

// Hot-source table (pagerank_hot_kernel): the nhot sources with the highest out-degree carry
// 23 % of RMAT-24's edges at nhot = 8192 (44 % at 45056).  Their contributions are staged once per
// launch in shared memory, where a warp's 32 random reads cost ~3-4 bank wavefronts instead of the
// 32 L1TEX wavefronts of a global gather (profiles/r01b_ncu_pagerank.md).  The default keeps two
// 1024-thread CTAs per SM: one CTA with the 45056-entry table halves the warps in flight and runs
// 2.4x slower (the gathers are latency-bound, tools/sweep_pagerank.py).
constexpr uint32_t HOT_BIT = 0x80000000u;
constexpr uint32_t HOT_MAX = 65536;   // 16-bit slots; above HOT_SLICE the table spans a cluster
#ifndef PROACT_HOT_SLICE_LOG2
#define PROACT_HOT_SLICE_LOG2 13
#endif
constexpr uint32_t HOT_SHIFT = PROACT_HOT_SLICE_LOG2;
constexpr uint32_t HOT_SLICE = 1u << HOT_SHIFT;  // entries one CTA holds (8192: 32 KiB; 2 CTAs of 1024 threads per SM)
#ifndef PROACT_GRAPH_HOT_DEFAULT
#define PROACT_GRAPH_HOT_DEFAULT 8192
#endif
constexpr uint32_t HOT_DEFAULT = PROACT_GRAPH_HOT_DEFAULT;

// Hot tables larger than one CTA's slice live in the distributed shared memory of a thread-block
// cluster (CL CTAs): CTA rank q of the cluster stages slots [q * HOT_SLICE, (q + 1) * HOT_SLICE)
// and a lookup of slot s reads CTA (s >> HOT_SHIFT)'s slice -- its own shared memory, or a peer's
// through DSMEM (mapa + ld.shared::cluster).  A lookup that leaves the SM goes over the cluster's
// SM-to-SM network instead of the L1 -> L2 request path the remaining gathers saturate, and the
// table covers (RMAT-24) 30 % of the in-edges at 2 CTAs, 37 % at 4, 48 % at 8 instead of 22 %.
__device__ __forceinline__ uint32_t cluster_rank()
{
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync_all()
{
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
template <int CL, class T>
__device__ __forceinline__ T hot_lookup(const T *hot, uint32_t hot_s, uint32_t my, uint32_t s)
{
    if (CL == 1) return hot[s];
    const uint32_t o = s >> HOT_SHIFT, li = s & (HOT_SLICE - 1u);
    if (o == my) return hot[li];
    uint32_t ra;
    asm("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(hot_s + 4u * li), "r"(o));
    uint32_t v;
    asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(ra) : "memory");
    T out;
    memcpy(&out, &v, 4);
    return out;
}
#ifndef PROACT_PRH_PG
#define PROACT_PRH_PG 4
#endif
#ifndef PROACT_PRH_RUN_PR   // pagerank_hot_kernel: consecutive in-edges per thread and run (4 or 8;
#define PROACT_PRH_RUN_PR 4  // 16-byte index loads from a 4-edge-aligned base, RUN/4 of them)
#endif
#ifndef PROACT_PRH_RUN
#define PROACT_PRH_RUN 4
#endif
#ifndef PROACT_PRH_SEGRED   // warp segmented reduction instead of per-run atomics: measured slower
#define PROACT_PRH_SEGRED 0   // (1.31 vs 1.20 ms at RMAT-24; the shared atomics are not the bound)
#endif
#ifndef PROACT_PRH_MINB      // pagerank_hot_kernel CTAs per SM (64 / 32 registers per thread at 1 / 2):
#define PROACT_PRH_MINB 2     // 1.153 ms at 2 vs 1.176 ms at 1 (RMAT-24, hot = 8192)
#endif
#ifndef PROACT_SSH_MINB      // sssp_hot_kernel CTAs per SM
#define PROACT_SSH_MINB 2
#endif
#ifndef PROACT_PRH_VEC       // pagerank_hot_kernel: 16-byte index loads from a 4-edge-aligned base
#define PROACT_PRH_VEC 1
#endif
#ifndef PROACT_SSH_VEC       // sssp_hot_kernel: runs of 4 edges, 16-byte index / weight loads (runv_ph)
#define PROACT_SSH_VEC 1
#endif
#ifndef PROACT_PRH_PIPE
#define PROACT_PRH_PIPE 1
#endif
constexpr int PG = PROACT_PRH_PG;     // item groups (of GB threads) per hot-kernel CTA
constexpr uint32_t CPS = GT + 4;      // words per group colptr window (GT + 1, padded)
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

__global__ void hot_slot_kernel(const uint32_t *hot_ids, uint32_t nhot, uint32_t *slot)
{
    for (uint32_t s = blockIdx.x * blockDim.x + threadIdx.x; s < nhot; s += gridDim.x * blockDim.x)
        slot[hot_ids[s]] = s;
}
__global__ void hot_encode_kernel(const uint32_t *rowidx, uint64_t E, const uint32_t *slot, uint32_t *out,
                                  unsigned long long *nhot_edges)
{
    uint32_t n = 0;
    for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < E; e += (uint64_t)gridDim.x * blockDim.x) {
        const uint32_t u = rowidx[e], k = slot[u];
        out[e] = k != 0xFFFFFFFFu ? (HOT_BIT | k) : u;
        n += k != 0xFFFFFFFFu;
    }
    atomicAdd(nhot_edges, (unsigned long long)n);
}

// ------------------------------------------------------------------ phase kernels
struct PrParams {
    GraphDev g;
    int region_in, region_out;
    double d, base;   // damping, (1-d)/V
};
// SSSP push rounds (direction-optimised Bellman-Ford, reading R24): device pointers of the Graph's
// push arrays; track = keep dprev current (every round, pull or push), par = round parity
struct PushDev {
    const uint32_t *prp, *pcol;
    const int32_t *pwt;
    int32_t *dprev, *ptmp;
    uint32_t *ptouch;
    uint2 *heavy;
    uint32_t *pctl;
    unsigned long long *dcnt;
    uint32_t track, par;   // track: pull kernels keep dprev current this round
    uint32_t skip, pad;    // push round: mark the blocks frontier edges reach, skip the others
};
struct SsspParams {
    GraphDev g;
    int region_in, region_out;
    int first;        // phase 0: every source is "changed"
    int pad;
    PushDev q;
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
__device__ __forceinline__ uint32_t ld_stream_u16(const uint16_t *p, uint64_t pol)
{
    uint16_t v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.u16 %0, [%1], %2;" : "=h"(v) : "l"(p), "l"(pol));
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
#ifndef PROACT_GATHER_MODE   // 0: .nc; 1: .nc + L1::no_allocate; 2: .cg (L2 only).  1 and 2: -2 %
#define PROACT_GATHER_MODE 1  // PageRank, -6 % SSSP at RMAT-24 (tools/sweep_pagerank.py, sweep_graph.py)
#endif
#if PROACT_GATHER_MODE == 1
#define GATHER_OP "ld.global.nc.L1::no_allocate.L2::cache_hint"
#elif PROACT_GATHER_MODE == 2
#define GATHER_OP "ld.global.cg.L2::cache_hint"
#else
#define GATHER_OP "ld.global.nc.L2::cache_hint"
#endif
__device__ __forceinline__ float ld_gather_f(const float *p, uint64_t pol)
{
    float v;
    asm volatile(GATHER_OP ".f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ int32_t ld_gather_i(const int32_t *p, uint64_t pol)
{
    int32_t v;
    asm volatile(GATHER_OP ".s32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
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
    {   // r' is only read back at the end: keep it out of the L2 working set
        const uint64_t pf = pol_first();
        asm volatile("st.global.L2::cache_hint.f32 [%0], %1, %2;" ::"l"(p.g.r_own + (v - p.g.v0)), "f"(r), "l"(pf)
                     : "memory");
    }
    const uint32_t od = ld_stream_u(p.g.outdeg + v, pol_first());
    const float c = od ? __fdiv_rn(r, (float)od) : 0.f;
    proact::put(lc, p.region_out, (uint64_t)v * 4, c);
}

// Local vertex index i (0..nv_tile-1) of edge e of the tile: the last i with cp[i] <= e (cp in
// shared memory, cp[nv_tile] = end of the tile's edges; zero-degree vertices are skipped).
__device__ __forceinline__ uint32_t vertex_of(const uint32_t *cp, uint32_t nvt, uint32_t e)
{
    uint32_t lo = 0, hi = nvt;
    while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        if (cp[mid] <= e) lo = mid;
        else hi = mid;
    }
    return lo;
}

// Build-time merge-path search: for every run of RUN consecutive in-edges of every item, the
// tile-local index of the vertex owning the run's first edge (vertex_of on the global colptr).
// One CTA per item.  The kernels read these 2-byte entries instead of searching shared memory.
__global__ void runv_kernel(const Item *items, const uint32_t *colptr, uint32_t nv, uint32_t RUN, int which,
                            uint16_t *runv)
{
    const Item it = items[blockIdx.x];
    const uint32_t lo = it.tile * GT, nvt = min(lo + GT, nv) - lo;
    // hot-kernel runs (which == 2, PRH_VEC) start at the 4-edge-aligned base below e0
    const uint32_t b0 = which >= 2 && PROACT_PRH_VEC ? (it.e0 & ~3u) : it.e0;
    const uint32_t nrun = (it.e1 - b0 + RUN - 1) / RUN;
    const uint32_t off = which == 3 ? it.run_p8 : which == 2 ? it.run_ph : which ? it.run_ss : it.run_pr;
    for (uint32_t j = threadIdx.x; j < nrun; j += blockDim.x)
        runv[off + j] = (uint16_t)vertex_of(colptr + lo, nvt, max(it.e0, b0 + j * RUN));
}

// Tile prologue: colptr of the tile into shared memory (+ the accumulator init by the caller).
__device__ __forceinline__ uint32_t load_tile(const GraphDev &g, uint32_t tile, uint32_t *cp, uint32_t &lo)
{
    lo = g.v0 + tile * GT;
    const uint32_t hi = min(lo + GT, g.v0 + g.nv), nvt = hi - lo;
    const uint64_t pf = pol_first();
    for (uint32_t i = threadIdx.x; i <= nvt; i += GB) cp[i] = ld_stream_u(g.colptr + (lo - g.v0 + i), pf);
    return nvt;
}

// Split tiles: the last item to arrive (after its global atomics) finishes the tile.
__device__ __forceinline__ bool split_arrive(const GraphDev &g, const Item &it, uint32_t *flag)
{
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        const uint32_t old = atomicAdd(&g.acc_cnt[it.slot], 1u);
        __threadfence();
        *flag = old + 1 == it.nsplit;
    }
    __syncthreads();
    return *flag != 0;
}

// PageRank: merge-path over the item's in-edges (RUN consecutive edges per thread, RUN gathers
// in flight).  Per-vertex sums are accumulated EXACTLY in 2^-62 fixed point (64-bit integer
// shared-memory atomics; every contribution is < 1 and a vertex's sum <= 1/d < 2^1, so it never
// overflows): each term is rounded once (absolute error <= 2^-63, relative to the smallest
// contribution ~1e-10 below 1e-9), the sum itself is exact and order independent, so results are
// bit-reproducible for any schedule; r' = (float)((1-d)/V + d * sum) as in the oracle (R12).
constexpr double FIX = 4611686018427387904.0;          // 2^62
constexpr double UNFIX = 1.0 / 4611686018427387904.0;  // 2^-62
// the fixed-point value of one fp32 contribution: round(g * 2^62), ties to even (an integer-only
// variant from the float's bits measured no faster, profiles/r02p_pagerank_fix62_int.log)
__device__ __forceinline__ unsigned long long fix62(float g)
{
    return (unsigned long long)__double2ll_rn((double)g * FIX);
}

__global__ void __launch_bounds__(GB, PROACT_PR_MINB) pagerank_kernel(launch_ctx lc, PrParams p)
{
    constexpr int RUN = PROACT_PR_RUN;
    if (proact::agent_dispatch(lc)) return;
    __shared__ uint32_t acc_lo[GT], acc_hi[GT];   // 64-bit fixed point as two native 32-bit halves
    __shared__ uint32_t cp[GT + 1];
    __shared__ uint32_t last;
    const float *cin = reinterpret_cast<const float *>(lc.ctx->region[p.region_in].base);
    const uint64_t pl = pol_last(), pf = pol_first();
    // 64-bit shared-memory atomicAdd is a CAS loop on sm_100; two 32-bit adds + carry are native
    auto acc_add = [&](uint32_t i, unsigned long long x) {
        const uint32_t xl = (uint32_t)x, old = atomicAdd(&acc_lo[i], xl);
        const uint32_t carry = old + xl < old ? 1u : 0u;
        const uint32_t xh = (uint32_t)(x >> 32) + carry;
        if (xh) atomicAdd(&acc_hi[i], xh);
    };
    auto acc_get = [&](uint32_t i) { return ((unsigned long long)acc_hi[i] << 32) | acc_lo[i]; };
    __shared__ uint32_t kclaim;
    bool waited = false;
    for (;;) {
        if (threadIdx.x == 0) {
            if (!waited) proact::wait_all(lc, p.region_in);   // (a7) previous generation is here
            kclaim = proact::claim_tile(lc, p.g.nitems);       // items dealt dynamically
        }
        waited = true;
        __syncthreads();
        const uint32_t k = kclaim;
        if (k >= p.g.nitems) break;
        const Item it = p.g.items[k];
        uint32_t lo;
        const uint32_t nvt = load_tile(p.g, it.tile, cp, lo);
        for (uint32_t i = threadIdx.x; i < nvt; i += GB) acc_lo[i] = acc_hi[i] = 0u;
        __syncthreads();
        // Runs are dealt to lanes in a 4 x 8 transposed order (lane l takes run 8*(l&3)... see
        // lrun): a warp still covers 32 consecutive runs (coalesced index loads), but lanes that
        // issue the same atomic instruction sit RUN*8 edges apart, so light vertices rarely
        // collide on one shared-memory address.  A warp whose 32 runs all lie inside one vertex
        // (hub in-edges) reduces in registers and issues a single atomic.
        const uint32_t lane = threadIdx.x & 31u;
        const uint32_t lrun = (threadIdx.x & ~31u) + ((lane & 3u) << 3) + (lane >> 2);
        for (uint32_t base = it.e0; base < it.e1; base += GB * RUN) {
            const uint32_t r0 = base + lrun * RUN;
            const bool act = r0 < it.e1;
            uint32_t i = 0xFFFFFFFFu;
            unsigned long long sum = 0ull;
            bool single = false;
            if (act) {
                const uint32_t r1 = min(r0 + RUN, it.e1);
                float g[RUN];
                i = ld_stream_u16(p.g.runv_pr + it.run_pr + (r0 - it.e0) / RUN, pf);
#pragma unroll
                for (int q = 0; q < RUN; ++q)
                    g[q] = r0 + q < r1 ? ld_gather_f(cin + ld_stream_u(p.g.rowidx + r0 + q, pf), pl) : 0.f;
                uint32_t nxt = cp[i + 1];
                single = r1 <= nxt;   // the whole run belongs to vertex i
#pragma unroll
                for (int q = 0; q < RUN; ++q) {
                    if (r0 + q >= r1) break;
                    while (r0 + q >= nxt) {
                        if (sum) acc_add(i, sum);
                        sum = 0ull;
                        nxt = cp[++i + 1];
                    }
                    sum += fix62(g[q]);
                }
            }
            // hub fast path: every lane active, single-vertex runs, the same vertex
            const uint32_t i0 = __shfl_sync(0xFFFFFFFFu, i, 0);
            if (__all_sync(0xFFFFFFFFu, act && single && i == i0)) {
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) sum += __shfl_xor_sync(0xFFFFFFFFu, sum, o);
                if (lane == 0 && sum) acc_add(i0, sum);
            } else if (act && sum) {
                acc_add(i, sum);
            }
        }
        __syncthreads();
        bool fin = true;
        if (it.nsplit > 1) {   // hub tile: sums meet in the global accumulator
            unsigned long long *ga = p.g.acc_f + (size_t)it.slot * GT;
            for (uint32_t i = threadIdx.x; i < nvt; i += GB)
                if (acc_get(i)) atomicAdd(&ga[i], acc_get(i));
            fin = split_arrive(p.g, it, &last);
            if (fin) {
                for (uint32_t i = threadIdx.x; i < nvt; i += GB) {
                    const unsigned long long v = __ldcg(&ga[i]);
                    acc_lo[i] = (uint32_t)v;
                    acc_hi[i] = (uint32_t)(v >> 32);
                    ga[i] = 0ull;   // ready for the next launch
                }
                if (threadIdx.x == 0) p.g.acc_cnt[it.slot] = 0;
                __syncthreads();
            }
        }
        if (fin) {
            for (uint32_t i = threadIdx.x; i < nvt; i += GB) pr_finish(lc, p, lo + i, (double)acc_get(i) * UNFIX);
            __syncthreads();
            if (threadIdx.x == 0) proact::commit_span(lc, p.region_out, (uint64_t)lo * 4, (uint64_t)nvt * 4);
        }
        __syncthreads();
    }
}

// ---- PageRank with a shared-memory hot-source table (the default when the graph has one).
// One CTA per SM of PG independent item groups (GB threads each, own named barrier, own
// accumulator / colptr arrays) around one table: hot[s] = contrib[hot_ids[s]], staged after the
// arrival wait.  An in-edge whose source is hot (rowidx_h = HOT_BIT | s) reads the table; the
// others gather from the replica as in pagerank_kernel.  Same exact fixed-point sums, so the
// result is bit-identical to pagerank_kernel's.
__device__ __forceinline__ void grp_bar(uint32_t grp)
{
    asm volatile("bar.sync %0, %1;" ::"r"(grp + 1u), "r"((uint32_t)GB) : "memory");
}

// claim_tile for PG claimers per CTA: the CTA counts out (and the last CTA re-arms the launch's
// counters) when its last group has seen the end of the work list.
__device__ __forceinline__ uint32_t claim_group(const launch_ctx &lc, uint32_t n, uint32_t *nout)
{
    uint32_t *S = lc.ctx->sched;
    const uint32_t t = atomicAdd(&S[0], 1u);
    if (t >= n && atomicAdd(nout, 1u) + 1u == (uint32_t)PG) {
        const uint32_t P = gridDim.x - lc.agent_ctas;
        if (atomicAdd(&S[1], 1u) + 1u == P) {
            S[0] = 0u;
            S[1] = 0u;
        }
    }
    return t;
}

template <int CL>
__global__ void __launch_bounds__(GB * PG, PROACT_PRH_MINB) pagerank_hot_kernel(launch_ctx lc, PrParams p)
{
    constexpr int RUN = PROACT_PRH_RUN_PR;
    if (proact::agent_dispatch(lc)) return;
    extern __shared__ uint32_t dyn[];   // [PG][CPS] colptr windows, then the hot table
    __shared__ uint32_t acc_lo_a[PG][GT], acc_hi_a[PG][GT];
    __shared__ uint32_t kclaim_a[PG], last_a[PG], nout;
    const uint32_t grp = threadIdx.x / GB, t = threadIdx.x % GB;
    uint32_t *acc_lo = acc_lo_a[grp], *acc_hi = acc_hi_a[grp], *cp = dyn + grp * CPS;
    float *hot = reinterpret_cast<float *>(dyn + PG * CPS);
    const float *cin = reinterpret_cast<const float *>(lc.ctx->region[p.region_in].base);
    const uint64_t pl = pol_last(), pf = pol_first();
    auto acc_add = [&](uint32_t i, unsigned long long x) {
        const uint32_t xl = (uint32_t)x, old = atomicAdd(&acc_lo[i], xl);
        const uint32_t carry = old + xl < old ? 1u : 0u;
        const uint32_t xh = (uint32_t)(x >> 32) + carry;
        if (xh) atomicAdd(&acc_hi[i], xh);
    };
    auto acc_get = [&](uint32_t i) { return ((unsigned long long)acc_hi[i] << 32) | acc_lo[i]; };
    auto acc_set = [&](uint32_t i, unsigned long long v) {
        acc_lo[i] = (uint32_t)v;
        acc_hi[i] = (uint32_t)(v >> 32);
    };
    if (threadIdx.x == 0) {
        proact::wait_all(lc, p.region_in);   // (a7) previous generation is here
        nout = 0u;
    }
    __syncthreads();
    const uint32_t my = CL > 1 ? cluster_rank() : 0u;
    const uint32_t hot_s = (uint32_t)__cvta_generic_to_shared(hot);
    {   // my slice of the hot table (all of it without a cluster)
        const uint32_t s0 = my * HOT_SLICE;
        const uint32_t ns = CL == 1 ? p.g.nhot : (p.g.nhot > s0 ? min(HOT_SLICE, p.g.nhot - s0) : 0u);
        for (uint32_t s = threadIdx.x; s < ns; s += blockDim.x) hot[s] = ld_gather_f(cin + __ldg(p.g.hot_ids + s0 + s), pl);
    }
    __syncthreads();
    if (CL > 1) cluster_sync_all();   // every slice staged before any peer reads it
    const uint32_t lane = t & 31u;
#if PROACT_PRH_SEGRED
    const uint32_t lrun = t;   // natural order: a warp's lanes hold 32 consecutive runs
#else
    const uint32_t lrun = (t & ~31u) + ((lane & 3u) << 3) + (lane >> 2);   // as in pagerank_kernel
#endif
    for (;;) {
        if (t == 0) kclaim_a[grp] = claim_group(lc, p.g.nitems, &nout);
        grp_bar(grp);
        const uint32_t k = kclaim_a[grp];
        if (k >= p.g.nitems) break;
        const Item it = p.g.items[k];
        const uint32_t lo = p.g.v0 + it.tile * GT, nvt = min(lo + GT, p.g.v0 + p.g.nv) - lo;
        for (uint32_t i = t; i <= nvt; i += GB) cp[i] = ld_stream_u(p.g.colptr + (lo - p.g.v0 + i), pf);
        for (uint32_t i = t; i < nvt; i += GB) acc_set(i, 0ull);
        grp_bar(grp);
        // index stream software-pipelined one round ahead (PRH_PIPE): the next round's rowidx /
        // run entries are in flight while this round's gathers are, so a round costs one L2 round
        // trip instead of two
        uint32_t xn[RUN], in_ = 0;
#if PROACT_PRH_VEC
        static_assert(RUN % 4 == 0, "PRH_VEC loads a run as RUN / 4 16-byte vectors");
        const uint32_t abase = it.e0 & ~3u;   // runs start 16-byte aligned; edges < e0 are masked
        auto load_idx = [&](uint32_t base) {
            const uint32_t r0 = base + lrun * RUN;
            if (r0 < it.e1) {
#pragma unroll
                for (int v = 0; v < RUN / 4; ++v) {
                    uint32_t v0, v1, v2, v3;
                    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                                 : "=r"(v0), "=r"(v1), "=r"(v2), "=r"(v3) : "l"(p.g.rowidx_h + r0 + 4 * v), "l"(pf));
                    xn[4 * v] = v0;
                    xn[4 * v + 1] = v1;
                    xn[4 * v + 2] = v2;
                    xn[4 * v + 3] = v3;
                }
#pragma unroll
                for (int q = 0; q < RUN; ++q)
                    if (r0 + q >= it.e1 || r0 + q < it.e0) xn[q] = HOT_BIT;   // not this item's edge
                in_ = ld_stream_u16(p.g.runv_p8 + it.run_p8 + (r0 - abase) / RUN, pf);
            } else {
#pragma unroll
                for (int q = 0; q < RUN; ++q) xn[q] = HOT_BIT;
                in_ = 0u;
            }
        };
#else
        const uint32_t abase = it.e0;
        auto load_idx = [&](uint32_t base) {
            const uint32_t r0 = base + lrun * RUN;
#pragma unroll
            for (int q = 0; q < RUN; ++q) xn[q] = r0 + q < it.e1 ? ld_stream_u(p.g.rowidx_h + r0 + q, pf) : HOT_BIT;
            in_ = r0 < it.e1 ? ld_stream_u16(p.g.runv_p8 + it.run_p8 + (r0 - it.e0) / RUN, pf) : 0u;
        };
#endif
        if (PROACT_PRH_PIPE) load_idx(abase);
        for (uint32_t base = abase; base < it.e1; base += GB * RUN) {
            const uint32_t r0 = base + lrun * RUN;
            const bool act = r0 < it.e1;
            if (!PROACT_PRH_PIPE) load_idx(base);
            uint32_t x[RUN];
#pragma unroll
            for (int q = 0; q < RUN; ++q) x[q] = xn[q];
            uint32_t i = act ? in_ : 0xFFFFFFFFu;
            if (PROACT_PRH_PIPE && base + GB * RUN < it.e1) load_idx(base + GB * RUN);
#if PROACT_PRH_SEGRED
            // Per-lane segments in edge order: the first (kin, vin), the last (kout, vout); segments
            // strictly inside the run are flushed at once.  A warp-wide segmented scan then joins
            // the chains that cross lanes, so every vertex a warp touches costs ONE shared atomic
            // per round (shared atomics cost ~2 cycles per active lane, B300_MICROARCH.md).
            uint32_t kin = 0xFFFFFFFFu, kout = 0xFFFFFFFFu;
            unsigned long long vin = 0ull, vout = 0ull;
            bool multi = false;
            if (act) {
                const uint32_t r1 = min(r0 + RUN, it.e1);
                float g[RUN];
#pragma unroll
                for (int q = 0; q < RUN; ++q) {
                    const bool h = x[q] & HOT_BIT;
                    g[q] = h ? hot_lookup<CL>(hot, hot_s, my, x[q] & ~HOT_BIT & 0xFFFFu) : 0.f;
                    if (!h) g[q] = ld_gather_f(cin + x[q], pl);
                }
                uint32_t nxt = cp[i + 1];
                unsigned long long sum = 0ull;
#pragma unroll
                for (int q = 0; q < RUN; ++q) {
                    if (r0 + q >= r1) break;
                    if (r0 + q < it.e0) continue;   // PRH_VEC: the aligned run starts before the item
                    while (r0 + q >= nxt) {   // vertex i closes before edge r0 + q
                        if (!multi) {
                            kin = i;
                            vin = sum;
                            multi = true;
                        } else if (sum) {
                            acc_add(i, sum);
                        }
                        sum = 0ull;
                        nxt = cp[++i + 1];
                    }
                    sum += fix62(g[q]);
                }
                if (!multi) {
                    kin = i;
                    vin = sum;
                }
                kout = i;
                vout = sum;
            }
            const uint32_t kprev = __shfl_up_sync(0xFFFFFFFFu, kout, 1);
            const uint32_t knext = __shfl_down_sync(0xFFFFFFFFu, kin, 1);
            // chain value ending at my last segment: inclusive segmented scan, a segment starts
            // at every lane that does not wholly continue the previous lane's last vertex
            unsigned long long T = vout;
            bool st = !(lane > 0 && !multi && kin == kprev);
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const unsigned long long Tu = __shfl_up_sync(0xFFFFFFFFu, T, d);
                const bool su = __shfl_up_sync(0xFFFFFFFFu, st, d);
                if (lane >= (uint32_t)d && !st) {
                    T += Tu;
                    st = su;
                }
            }
            const unsigned long long Tprev = __shfl_up_sync(0xFFFFFFFFu, T, 1);
            if (act) {
                if (multi) {   // my first vertex, joined with the chain arriving from the left
                    const unsigned long long hv = vin + (lane > 0 && kin == kprev ? Tprev : 0ull);
                    if (hv) acc_add(kin, hv);
                }
                if ((lane == 31 || knext != kout) && T) acc_add(kout, T);   // my chain ends here
            }
        }
#else
            unsigned long long sum = 0ull;
            bool single = false;
            if (act) {
                const uint32_t r1 = min(r0 + RUN, it.e1);
                float g[RUN];
#pragma unroll
                for (int q = 0; q < RUN; ++q) {
                    const bool h = x[q] & HOT_BIT;
                    g[q] = h ? hot_lookup<CL>(hot, hot_s, my, x[q] & ~HOT_BIT & 0xFFFFu) : 0.f;
                    if (!h) g[q] = ld_gather_f(cin + x[q], pl);
                }
                uint32_t nxt = cp[i + 1];
                single = r1 <= nxt;
#pragma unroll
                for (int q = 0; q < RUN; ++q) {
                    if (r0 + q >= r1) break;
                    if (r0 + q < it.e0) continue;   // PRH_VEC: the aligned run starts before the item
                    while (r0 + q >= nxt) {
                        if (sum) acc_add(i, sum);
                        sum = 0ull;
                        nxt = cp[++i + 1];
                    }
                    sum += fix62(g[q]);
                }
            }
            const uint32_t i0 = __shfl_sync(0xFFFFFFFFu, i, 0);
            if (__all_sync(0xFFFFFFFFu, act && single && i == i0)) {
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) sum += __shfl_xor_sync(0xFFFFFFFFu, sum, o);
                if (lane == 0 && sum) acc_add(i0, sum);
            } else if (act && sum) {
                acc_add(i, sum);
            }
        }
#endif
        grp_bar(grp);
        bool fin = true;
        if (it.nsplit > 1) {   // hub tile: sums meet in the global accumulator
            unsigned long long *ga = p.g.acc_f + (size_t)it.slot * GT;
            for (uint32_t i = t; i < nvt; i += GB)
                if (acc_get(i)) atomicAdd(&ga[i], acc_get(i));
            grp_bar(grp);
            if (t == 0) {
                __threadfence();
                const uint32_t old = atomicAdd(&p.g.acc_cnt[it.slot], 1u);
                __threadfence();
                last_a[grp] = old + 1 == it.nsplit;
            }
            grp_bar(grp);
            fin = last_a[grp] != 0;
            if (fin) {
                for (uint32_t i = t; i < nvt; i += GB) {
                    acc_set(i, __ldcg(&ga[i]));
                    ga[i] = 0ull;   // ready for the next launch
                }
                if (t == 0) p.g.acc_cnt[it.slot] = 0;
                grp_bar(grp);
            }
        }
        if (fin) {
            for (uint32_t i = t; i < nvt; i += GB) pr_finish(lc, p, lo + i, (double)acc_get(i) * UNFIX);
            grp_bar(grp);
            if (t == 0) proact::commit_span(lc, p.region_out, (uint64_t)lo * 4, (uint64_t)nvt * 4);
        }
        grp_bar(grp);
    }
    if (CL > 1) cluster_sync_all();   // my slice stays readable until every peer is done
}

// Helpers of the SSSP push rounds (reading R24; see sssp_push_kernel) shared with the pull kernels.
constexpr uint32_t PUSH_HEAVY = 1024;   // frontier sources with more edges here: queued as pieces
constexpr uint32_t PUSH_PIECE = 4096;   // edges per heavy piece (one CTA claims a piece)
constexpr uint32_t PB = 256;            // threads per push-round CTA (x 4 vertices = one 4 KiB block)

__device__ __forceinline__ int32_t ld_cg_i(const int32_t *p)
{
    int32_t v;
    asm volatile("ld.global.cg.s32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}
// Grid-wide barrier of the producer CTAs (all co-resident: proact_launch caps the persistent grid
// at the co-resident capacity).  ctl[1] arrivals, ctl[2] generation; watchdog-guarded.
__device__ __forceinline__ bool grid_barrier(const launch_ctx &lc, uint32_t *ctl)
{
    __shared__ uint32_t gb_bad;
    __syncthreads();
    if (threadIdx.x == 0) {
        gb_bad = 0u;
        const uint32_t gen = proact::ld_acquire_gpu(&ctl[2]);   // before arriving
        __threadfence();
        if (atomicAdd(&ctl[1], 1u) + 1u == proact::producer_grid(lc)) {
            ctl[1] = 0u;            // re-armed before the release
            __threadfence();
            atomicAdd(&ctl[2], 1u);
        } else {
            const uint64_t t0 = proact::globaltimer();
            uint32_t it = 0;
            while (proact::ld_acquire_gpu(&ctl[2]) == gen)
                if (proact::spin_step(lc.ctx, t0, it, proact::SITE_GRID_BARRIER)) { gb_bad = 1u; break; }
        }
        __threadfence();
    }
    __syncthreads();
    return gb_bad == 0u;
}
// dprev := the arrived input (pull rounds; the push kernel does it while finding the frontier):
// 16-byte vectors, two in flight per thread (the loop is latency-bound otherwise)
__device__ __forceinline__ void track_input(const launch_ctx &lc, const SsspParams &p, const int32_t *din)
{
    if (!p.q.track) return;
    const uint64_t n4 = p.g.V / 4, stride = (uint64_t)proact::producer_grid(lc) * blockDim.x;
    const int4 *a = reinterpret_cast<const int4 *>(din);
    int4 *b = reinterpret_cast<int4 *>(p.q.dprev);
    for (uint64_t i = (uint64_t)proact::producer_block(lc) * blockDim.x + threadIdx.x; i < n4; i += 2 * stride) {
        const bool two = i + stride < n4;
        const int4 x0 = a[i], y0 = b[i];
        int4 x1 = x0, y1 = y0;
        if (two) {
            x1 = a[i + stride];
            y1 = b[i + stride];
        }
        if (x0.x != y0.x || x0.y != y0.y || x0.z != y0.z || x0.w != y0.w) b[i] = x0;
        if (two && (x1.x != y1.x || x1.y != y1.y || x1.z != y1.z || x1.w != y1.w)) b[i + stride] = x1;
    }
    if (proact::producer_block(lc) == 0)
        for (uint64_t u = n4 * 4 + threadIdx.x; u < p.g.V; u += blockDim.x) p.q.dprev[u] = din[u];
}
// out-degree sum of my changed vertices, for the next round's pull / push decision (host): warp
// sums meet in the CTA's shared accumulator (one global atomic per CTA, count_flush at the end --
// a global atomic per warp and tile serialises on one address)
__device__ __forceinline__ void count_changed(const SsspParams &p, unsigned long long cs, unsigned long long *cta)
{
    if (!p.q.dcnt) return;   // (callers accumulate in 32 bits: a thread's vertices' out-degrees)
    for (int o = 16; o > 0; o >>= 1) cs += __shfl_xor_sync(0xFFFFFFFFu, cs, o);
    if ((threadIdx.x & 31u) == 0u && cs) atomicAdd(cta, cs);
}
__device__ __forceinline__ void count_flush(const SsspParams &p, const unsigned long long *cta)
{
    if (!p.q.dcnt) return;
    __syncthreads();
    if (threadIdx.x == 0 && *cta) atomicAdd(&p.q.dcnt[p.q.par], *cta);
}
// relax edge e (source distance du) into my vertex pcol[e]: a fire-and-forget atomicMin (RED)
__device__ __forceinline__ void push_relax(const SsspParams &p, uint32_t e, int32_t du)
{
    const uint32_t v = __ldg(p.q.pcol + e);
    const int64_t c = (int64_t)du + (int64_t)__ldg(p.q.pwt + e);
    const int32_t cand = c < (int64_t)INT32_MAX ? (int32_t)c : INT32_MAX;
    atomicMin(p.q.ptmp + v, cand);
    if (p.q.skip) p.q.ptouch[v >> 10] = 1u;   // the block's minima need a look in step 3
}

constexpr uint32_t CHG_WORDS = 4096;   // changed-chunk bitmap in shared memory (<= 131072 chunks)

// SSSP: merge-path over the item's in-edges; a source is relaxed only if its chunk changed in
// the previous round (bitmap snapshot); per-vertex minima via shared-memory atomicMin.
__global__ void __launch_bounds__(GB, PROACT_SSSP_MINB) sssp_kernel(launch_ctx lc, SsspParams p)
{
    constexpr int RUN = PROACT_SSSP_RUN;
    if (proact::agent_dispatch(lc)) return;
    __shared__ int32_t acc[GT];
    __shared__ uint32_t cp[GT + 1];
    __shared__ uint32_t chg[CHG_WORDS];
    __shared__ uint32_t last;
    const region_dev &Ri = lc.ctx->region[p.region_in];
    const int32_t *din = reinterpret_cast<const int32_t *>(Ri.base);
    const uint64_t pf = pol_first(), pl = pol_last();
    // source vertex -> global chunk id: rank slices are chunk-aligned, so it is u*4/chunk_bytes
    const uint32_t cv = Ri.chunk_bytes / 4;
    const uint32_t cshift = __popc(cv) == 1 ? (uint32_t)(__ffs(cv) - 1) : 0u, cdiv = __popc(cv) == 1 ? 0u : cv;
    __shared__ uint32_t kclaim;
    __shared__ unsigned long long cs_cta;
    bool ready = false;
    if (p.q.dcnt) {   // every CTA keeps its share of dprev current (if asked), items or not
        if (threadIdx.x == 0) {
            cs_cta = 0ull;
            proact::wait_all(lc, p.region_in);
            if (proact::producer_block(lc) == 0) p.q.dcnt[p.q.par ^ 1u] = 0ull;
        }
        __syncthreads();
        track_input(lc, p, din);
    }
    for (;;) {
        if (threadIdx.x == 0) kclaim = proact::claim_tile(lc, p.g.nitems);   // items dealt dynamically
        __syncthreads();
        const uint32_t k = kclaim;
        if (k >= p.g.nitems) break;
        if (!ready) {   // (a7) wait for the previous generation, then snapshot its changed bits
            if (threadIdx.x == 0) proact::wait_all(lc, p.region_in);
            __syncthreads();
            const uint32_t gen = lc.gen[p.region_in];
            const uint32_t pm = lc.gen_mech[p.region_in];   // how the input was produced
            const bool agent = pm == PROACT_MECH_FUSED || pm == PROACT_MECH_ELIDE;
            for (uint32_t wi = threadIdx.x; wi < CHG_WORDS && wi * 32 < Ri.n_total; wi += GB) {
                uint32_t bits = 0;
                for (uint32_t bb = 0; bb < 32; ++bb) {
                    const uint32_t g = wi * 32 + bb;
                    if (g >= Ri.n_total) break;
                    bool c;
                    if (g >= Ri.chunk0 && g < Ri.chunk0 + Ri.n_own) c = Ri.changed_gen[g - Ri.chunk0] == gen;
                    else c = !agent || (ld_nc_u(Ri.arrive + g) & 1u);   // no flags without the agent
                    bits |= (uint32_t)c << bb;
                }
                chg[wi] = bits;
            }
            ready = true;
        }
        const Item it = p.g.items[k];
        uint32_t lo;
        const uint32_t nvt = load_tile(p.g, it.tile, cp, lo);
        for (uint32_t i = threadIdx.x; i < nvt; i += GB) acc[i] = INT32_MAX;
        __syncthreads();
        // lane order and hub fast path as in pagerank_kernel
        const uint32_t lane = threadIdx.x & 31u;
        const uint32_t lrun = (threadIdx.x & ~31u) + ((lane & 3u) << 3) + (lane >> 2);
        for (uint32_t base = it.e0; base < it.e1; base += GB * RUN) {
            const uint32_t r0 = base + lrun * RUN;
            const bool act = r0 < it.e1;
            uint32_t i = 0xFFFFFFFFu;
            int32_t best = INT32_MAX;
            bool single = false;
            if (act) {
                const uint32_t r1 = min(r0 + RUN, it.e1);
                int32_t c[RUN];
#pragma unroll
                for (int q = 0; q < RUN; ++q) {
                    c[q] = INT32_MAX;
                    if (r0 + q < r1) {
                        const uint32_t u = ld_stream_u(p.g.rowidx + r0 + q, pf);
                        const uint32_t g = cdiv ? u / cdiv : u >> cshift;
                        if (p.first || (chg[g >> 5] >> (g & 31) & 1u)) {
                            const int32_t du = ld_gather_i(din + u, pl);
                            if (du != INT32_MAX) {
                                const int64_t cand = (int64_t)du + (int64_t)ld_stream_i(p.g.w + r0 + q, pf);
                                c[q] = cand < (int64_t)INT32_MAX ? (int32_t)cand : INT32_MAX;
                            }
                        }
                    }
                }
                i = ld_stream_u16(p.g.runv_ss + it.run_ss + (r0 - it.e0) / RUN, pf);
                uint32_t nxt = cp[i + 1];
                single = r1 <= nxt;
#pragma unroll
                for (int q = 0; q < RUN; ++q) {
                    if (r0 + q >= r1) break;
                    while (r0 + q >= nxt) {
                        if (best != INT32_MAX) atomicMin(&acc[i], best);
                        best = INT32_MAX;
                        nxt = cp[++i + 1];
                    }
                    best = min(best, c[q]);
                }
            }
            const uint32_t i0 = __shfl_sync(0xFFFFFFFFu, i, 0);
            if (__all_sync(0xFFFFFFFFu, act && single && i == i0)) {
                best = __reduce_min_sync(0xFFFFFFFFu, best);
                if (lane == 0 && best != INT32_MAX) atomicMin(&acc[i0], best);
            } else if (act && best != INT32_MAX) {
                atomicMin(&acc[i], best);
            }
        }
        __syncthreads();
        bool fin = true;
        if (it.nsplit > 1) {
            int32_t *ga = p.g.acc_i + (size_t)it.slot * GT;
            for (uint32_t i = threadIdx.x; i < nvt; i += GB)
                if (acc[i] != INT32_MAX) atomicMin(&ga[i], acc[i]);
            fin = split_arrive(p.g, it, &last);
            if (fin) {
                for (uint32_t i = threadIdx.x; i < nvt; i += GB) {
                    acc[i] = __ldcg(&ga[i]);
                    ga[i] = INT32_MAX;
                }
                if (threadIdx.x == 0) p.g.acc_cnt[it.slot] = 0;
                __syncthreads();
            }
        }
        if (fin) {
            bool changed = false;
            uint32_t cs = 0;   // out-degree sum of the tile's changed vertices (push decision, R24)
            for (uint32_t i = threadIdx.x; i < nvt; i += GB) {
                const uint32_t v = lo + i;
                const int32_t old = din[v];
                const int32_t best = min(old, acc[i]);
                proact::put(lc, p.region_out, (uint64_t)v * 4, best);
                changed |= best != old;
                if (best != old) cs += __ldg(p.g.outdeg + v);
            }
            count_changed(p, cs, &cs_cta);
            // per-tile chunk state (SPARSE region): changed now -> flag bit + vote; push if
            // changed now or in the previous round (the peers' ping-pong copy holds d^{k-1})
            const int any = __syncthreads_or(changed);
            if (threadIdx.x == 0) {
                const uint64_t off = (uint64_t)lo * 4;
                const bool prev = !p.first && proact::local_changed(lc, p.region_in, off);
                if (any) {
                    proact::mark_changed(lc, p.region_out, off);
                    proact::vote(lc);
                }
                if (any || prev) proact::mark_push(lc, p.region_out, off);
                proact::commit_span(lc, p.region_out, off, (uint64_t)nvt * 4);
            }
        }
        __syncthreads();
    }
    count_flush(p, &cs_cta);
}

// ---- SSSP with the hot-source table and the pipelined index stream (as pagerank_hot_kernel).
// hot[s] = d[hot_ids[s]] if that source's chunk changed in the previous round (or first round),
// else INT32_MAX, so a hot in-edge needs neither the bitmap test nor the global gather.
template <int CL>
__global__ void __launch_bounds__(GB * PG, PROACT_SSH_MINB) sssp_hot_kernel(launch_ctx lc, SsspParams p)
{
#if PROACT_SSH_VEC
    static_assert(PROACT_PRH_VEC && PROACT_PRH_RUN == 4, "SSH_VEC shares the aligned 4-edge runs of runv_ph");
    constexpr int RUN = 4;
#else
    constexpr int RUN = PROACT_SSSP_RUN;   // shares runv_ss with sssp_kernel
#endif
    if (proact::agent_dispatch(lc)) return;
    extern __shared__ uint32_t dyn[];   // [PG][CPS] colptr windows, then the hot table
    __shared__ int32_t acc_a[PG][GT];
    __shared__ uint32_t chg[CHG_WORDS];
    __shared__ uint32_t kclaim_a[PG], last_a[PG], any_a[PG], nout;
    const uint32_t grp = threadIdx.x / GB, t = threadIdx.x % GB;
    int32_t *acc = acc_a[grp];
    uint32_t *cp = dyn + grp * CPS;
    int32_t *hot = reinterpret_cast<int32_t *>(dyn + PG * CPS);
    const region_dev &Ri = lc.ctx->region[p.region_in];
    const int32_t *din = reinterpret_cast<const int32_t *>(Ri.base);
    const uint64_t pf = pol_first(), pl = pol_last();
    const uint32_t cv = Ri.chunk_bytes / 4;
    const uint32_t cshift = __popc(cv) == 1 ? (uint32_t)(__ffs(cv) - 1) : 0u, cdiv = __popc(cv) == 1 ? 0u : cv;
    auto changed_src = [&](uint32_t u) {
        const uint32_t g = cdiv ? u / cdiv : u >> cshift;
        return p.first || (chg[g >> 5] >> (g & 31) & 1u);
    };
    // (a7) wait for the previous generation, snapshot its changed bits, stage the hot table
    __shared__ unsigned long long cs_cta;
    if (threadIdx.x == 0) {
        proact::wait_all(lc, p.region_in);
        nout = 0u;
        cs_cta = 0ull;
        if (p.q.dcnt && proact::producer_block(lc) == 0) p.q.dcnt[p.q.par ^ 1u] = 0ull;
    }
    __syncthreads();
    track_input(lc, p, din);   // dprev := this round's input (push rounds, reading R24)
    {
        const uint32_t gen = lc.gen[p.region_in];
        const uint32_t pm = lc.gen_mech[p.region_in];
        const bool agent = pm == PROACT_MECH_FUSED || pm == PROACT_MECH_ELIDE;
        for (uint32_t wi = threadIdx.x; wi < CHG_WORDS && wi * 32 < Ri.n_total; wi += blockDim.x) {
            uint32_t bits = 0;
            for (uint32_t bb = 0; bb < 32; ++bb) {
                const uint32_t g = wi * 32 + bb;
                if (g >= Ri.n_total) break;
                bool c;
                if (g >= Ri.chunk0 && g < Ri.chunk0 + Ri.n_own) c = Ri.changed_gen[g - Ri.chunk0] == gen;
                else c = !agent || (ld_nc_u(Ri.arrive + g) & 1u);
                bits |= (uint32_t)c << bb;
            }
            chg[wi] = bits;
        }
    }
    __syncthreads();
    const uint32_t my = CL > 1 ? cluster_rank() : 0u;
    const uint32_t hot_s = (uint32_t)__cvta_generic_to_shared(hot);
    {   // my slice of the hot table (all of it without a cluster)
        const uint32_t s0 = my * HOT_SLICE;
        const uint32_t ns = CL == 1 ? p.g.nhot : (p.g.nhot > s0 ? min(HOT_SLICE, p.g.nhot - s0) : 0u);
        for (uint32_t s = threadIdx.x; s < ns; s += blockDim.x) {
            const uint32_t u = __ldg(p.g.hot_ids + s0 + s);
            hot[s] = changed_src(u) ? ld_gather_i(din + u, pl) : INT32_MAX;
        }
    }
    __syncthreads();
    if (CL > 1) cluster_sync_all();
    const uint32_t lane = t & 31u;
    const uint32_t lrun = (t & ~31u) + ((lane & 3u) << 3) + (lane >> 2);   // as in sssp_kernel
    for (;;) {
        if (t == 0) kclaim_a[grp] = claim_group(lc, p.g.nitems, &nout);
        grp_bar(grp);
        const uint32_t k = kclaim_a[grp];
        if (k >= p.g.nitems) break;
        const Item it = p.g.items[k];
        const uint32_t lo = p.g.v0 + it.tile * GT, nvt = min(lo + GT, p.g.v0 + p.g.nv) - lo;
        for (uint32_t i = t; i <= nvt; i += GB) cp[i] = ld_stream_u(p.g.colptr + (lo - p.g.v0 + i), pf);
        for (uint32_t i = t; i < nvt; i += GB) acc[i] = INT32_MAX;
        grp_bar(grp);
        uint32_t xn[RUN], in_ = 0;
#if PROACT_SSH_VEC
        const uint32_t abase = it.e0 & ~3u;   // as in pagerank_hot_kernel (PRH_VEC)
        auto load_idx = [&](uint32_t base) {
            const uint32_t r0 = base + lrun * RUN;
            if (r0 < it.e1) {
                uint32_t v0, v1, v2, v3;
                asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
                             : "=r"(v0), "=r"(v1), "=r"(v2), "=r"(v3) : "l"(p.g.rowidx_h + r0), "l"(pf));
                xn[0] = v0;
                xn[1] = v1;
                xn[2] = v2;
                xn[3] = v3;
                in_ = ld_stream_u16(p.g.runv_ph + it.run_ph + (r0 - abase) / RUN, pf);
            } else {
                in_ = 0u;
            }
        };
#else
        const uint32_t abase = it.e0;
        auto load_idx = [&](uint32_t base) {
            const uint32_t r0 = base + lrun * RUN;
#pragma unroll
            for (int q = 0; q < RUN; ++q) xn[q] = r0 + q < it.e1 ? ld_stream_u(p.g.rowidx_h + r0 + q, pf) : HOT_BIT;
            in_ = r0 < it.e1 ? ld_stream_u16(p.g.runv_ss + it.run_ss + (r0 - it.e0) / RUN, pf) : 0u;
        };
#endif
        load_idx(abase);
        for (uint32_t base = abase; base < it.e1; base += GB * RUN) {
            const uint32_t r0 = base + lrun * RUN;
            const bool act = r0 < it.e1;
            uint32_t x[RUN];
#pragma unroll
            for (int q = 0; q < RUN; ++q) x[q] = xn[q];
            uint32_t i = act ? in_ : 0xFFFFFFFFu;
            if (base + GB * RUN < it.e1) load_idx(base + GB * RUN);
            int32_t best = INT32_MAX;
            bool single = false;
            if (act) {
                const uint32_t r1 = min(r0 + RUN, it.e1);
                int32_t c[RUN];
#pragma unroll
                for (int q = 0; q < RUN; ++q) {
                    int32_t du = INT32_MAX;
                    if (r0 + q < r1 && r0 + q >= it.e0) {
                        if (x[q] & HOT_BIT) du = hot_lookup<CL>(hot, hot_s, my, x[q] & ~HOT_BIT & 0xFFFFu);
                        else if (changed_src(x[q])) du = ld_gather_i(din + x[q], pl);
                    }
                    c[q] = du;
                }
#if PROACT_SSH_VEC
                bool anyc = false;
#pragma unroll
                for (int q = 0; q < RUN; ++q) anyc |= c[q] != INT32_MAX;
                if (anyc) {   // one 16-byte weight load for the run
                    int32_t wv[4];
                    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.s32 {%0,%1,%2,%3}, [%4], %5;"
                                 : "=r"(wv[0]), "=r"(wv[1]), "=r"(wv[2]), "=r"(wv[3]) : "l"(p.g.w + r0), "l"(pf));
#pragma unroll
                    for (int q = 0; q < RUN; ++q)
                        if (c[q] != INT32_MAX) {
                            const int64_t cand = (int64_t)c[q] + (int64_t)wv[q];
                            c[q] = cand < (int64_t)INT32_MAX ? (int32_t)cand : INT32_MAX;
                        }
                }
#else
#pragma unroll
                for (int q = 0; q < RUN; ++q)
                    if (c[q] != INT32_MAX) {
                        const int64_t cand = (int64_t)c[q] + (int64_t)ld_stream_i(p.g.w + r0 + q, pf);
                        c[q] = cand < (int64_t)INT32_MAX ? (int32_t)cand : INT32_MAX;
                    }
#endif
                uint32_t nxt = cp[i + 1];
                single = r1 <= nxt;
#pragma unroll
                for (int q = 0; q < RUN; ++q) {
                    if (r0 + q >= r1) break;
                    if (r0 + q < it.e0) continue;   // SSH_VEC: the aligned run starts before the item
                    while (r0 + q >= nxt) {
                        if (best != INT32_MAX) atomicMin(&acc[i], best);
                        best = INT32_MAX;
                        nxt = cp[++i + 1];
                    }
                    best = min(best, c[q]);
                }
            }
            const uint32_t i0 = __shfl_sync(0xFFFFFFFFu, i, 0);
            if (__all_sync(0xFFFFFFFFu, act && single && i == i0)) {
                best = __reduce_min_sync(0xFFFFFFFFu, best);
                if (lane == 0 && best != INT32_MAX) atomicMin(&acc[i0], best);
            } else if (act && best != INT32_MAX) {
                atomicMin(&acc[i], best);
            }
        }
        grp_bar(grp);
        bool fin = true;
        if (it.nsplit > 1) {
            int32_t *ga = p.g.acc_i + (size_t)it.slot * GT;
            for (uint32_t i = t; i < nvt; i += GB)
                if (acc[i] != INT32_MAX) atomicMin(&ga[i], acc[i]);
            grp_bar(grp);
            if (t == 0) {
                __threadfence();
                const uint32_t old = atomicAdd(&p.g.acc_cnt[it.slot], 1u);
                __threadfence();
                last_a[grp] = old + 1 == it.nsplit;
            }
            grp_bar(grp);
            fin = last_a[grp] != 0;
            if (fin) {
                for (uint32_t i = t; i < nvt; i += GB) {
                    acc[i] = __ldcg(&ga[i]);
                    ga[i] = INT32_MAX;
                }
                if (t == 0) p.g.acc_cnt[it.slot] = 0;
                grp_bar(grp);
            }
        }
        if (fin) {
            if (t == 0) any_a[grp] = 0u;
            grp_bar(grp);
            bool changed = false;
            uint32_t cs = 0;   // out-degree sum of the tile's changed vertices (push decision, R24)
            for (uint32_t i = t; i < nvt; i += GB) {
                const uint32_t v = lo + i;
                const int32_t old = din[v];
                const int32_t best = min(old, acc[i]);
                proact::put(lc, p.region_out, (uint64_t)v * 4, best);
                changed |= best != old;
                if (best != old) cs += __ldg(p.g.outdeg + v);
            }
            count_changed(p, cs, &cs_cta);
            if (__any_sync(0xFFFFFFFFu, changed) && lane == 0) any_a[grp] = 1u;
            grp_bar(grp);   // orders the group's puts before the commit (a3)
            if (t == 0) {   // chunk state as in sssp_kernel
                const uint64_t off = (uint64_t)lo * 4;
                const bool any = any_a[grp] != 0u;
                const bool prev = !p.first && proact::local_changed(lc, p.region_in, off);
                if (any) {
                    proact::mark_changed(lc, p.region_out, off);
                    proact::vote(lc);
                }
                if (any || prev) proact::mark_push(lc, p.region_out, off);
                proact::commit_span(lc, p.region_out, off, (uint64_t)nvt * 4);
            }
        }
        grp_bar(grp);
    }
    count_flush(p, &cs_cta);
    if (CL > 1) cluster_sync_all();   // my slice stays readable until every peer is done
}

// ---- SSSP push rounds (reading R24: direction-optimised Bellman-Ford).  PAPER.md L267 fixes the
// result -- "every vertex computes its shortest distance ... using the Bellman-Ford algorithm" --
// d^{k+1}[v] = min(d^k[v], min_{u->v} d^k[u] + w); a source u with d^k[u] = d^{k-1}[u] was already
// relaxed into v in round k, so only the FRONTIER (sources whose distance changed in round k)
// matters.  When the frontier's out-edges are few (late rounds), the rank pushes from them over
// its in-edges grouped by source (prp / pcol / pwt) with atomicMin into a private array, instead
// of pulling over every in-edge; the same d^{k+1}, bit for bit (min is order independent).  The
// frontier is found by comparing the arrived input with a PRIVATE copy of the previous input
// (dprev, kept current in every round): the output replica itself cannot serve, peers' agents
// already write this round's chunks into it.
#ifndef PROACT_PUSH_MINB
#define PROACT_PUSH_MINB 6   // push-round CTAs per SM (r02s sweep: 6 > 4 > 8, latency-bound loops)
#endif
__global__ void __launch_bounds__(PB, PROACT_PUSH_MINB) sssp_push_kernel(launch_ctx lc, SsspParams p)
{
    if (proact::agent_dispatch(lc)) return;
    const region_dev &Ri = lc.ctx->region[p.region_in];
    const int32_t *din = reinterpret_cast<const int32_t *>(Ri.base);
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t P = proact::producer_grid(lc), pb = proact::producer_block(lc);
    __shared__ unsigned long long cs_cta;
    if (threadIdx.x == 0) {
        proact::wait_all(lc, p.region_in);   // (a7) the previous generation is here
        cs_cta = 0ull;
        if (pb == 0) p.q.dcnt[p.q.par ^ 1u] = 0ull;   // the next round's accumulator
    }
    __syncthreads();
    // 1. frontier: sources whose input changed since the previous round (dprev := input); the
    //    light ones are relaxed at once, warp-cooperatively, the heavy ones queued.  Each lane
    //    takes 4 consecutive sources (16-byte loads of input and dprev; V % 4 sources at the end
    //    by the first warp)
    {
        const uint64_t W = (uint64_t)P * (PB / 32), gw = (uint64_t)pb * (PB / 32) + (threadIdx.x >> 5);
        const uint64_t n4 = p.g.V / 4;
        const int4 *a4 = reinterpret_cast<const int4 *>(din);
        int4 *b4 = reinterpret_cast<int4 *>(p.q.dprev);
        auto frontier = [&](uint64_t u, int32_t du, int32_t dp) {   // -> (du, e0, e1) or e1 == e0
            uint32_t e0 = 0, e1 = 0;
            if ((p.first || du != dp) && du != INT32_MAX) {
                e0 = __ldg(p.q.prp + u);
                e1 = __ldg(p.q.prp + u + 1);
                if (e1 - e0 > PUSH_HEAVY) {   // pieces of PUSH_PIECE edges, claimed by CTAs in step 2
                    const uint32_t np = (e1 - e0 + PUSH_PIECE - 1) / PUSH_PIECE;
                    const uint32_t k0 = atomicAdd(&p.q.pctl[0], np);
                    for (uint32_t k = 0; k < np; ++k) p.q.heavy[k0 + k] = make_uint2((uint32_t)u, e0 + k * PUSH_PIECE);
                    e1 = e0;
                }
            }
            return make_uint2(e0, e1);
        };
        auto relax_ballot = [&](int32_t du, uint2 r) {
            uint32_t m = __ballot_sync(0xFFFFFFFFu, r.y > r.x);
            while (m) {
                const int j = __ffs(m) - 1;
                m &= m - 1;
                const int32_t dj = __shfl_sync(0xFFFFFFFFu, du, j);
                const uint32_t x = __shfl_sync(0xFFFFFFFFu, r.x, j), y = __shfl_sync(0xFFFFFFFFu, r.y, j);
                for (uint32_t e = x + lane; e < y; e += 32) push_relax(p, e, dj);
            }
        };
        // the warp's light frontier sources of one window (<= 128) as a flat edge list: entry k =
        // (first edge, source distance, end offset in the list); lane f relaxes edges f, f+32, ..
        // -- independent loads in every lane instead of one source at a time
        __shared__ uint32_t fl_e0[PB / 32][128], fl_end[PB / 32][128];
        __shared__ int32_t fl_du[PB / 32][128];
        uint32_t *we0 = fl_e0[threadIdx.x >> 5], *wend = fl_end[threadIdx.x >> 5];
        int32_t *wdu = fl_du[threadIdx.x >> 5];
        auto relax_flat = [&](const int32_t *dus, const uint2 *rs) {
            uint32_t ne = 0, ned = 0;
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                ne += rs[q].y > rs[q].x;
                ned += rs[q].y - rs[q].x;
            }
            uint32_t pe = ne, pd = ned;   // inclusive warp scans
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint32_t a = __shfl_up_sync(0xFFFFFFFFu, pe, o), b = __shfl_up_sync(0xFFFFFFFFu, pd, o);
                if (lane >= (uint32_t)o) {
                    pe += a;
                    pd += b;
                }
            }
            const uint32_t n = __shfl_sync(0xFFFFFFFFu, pe, 31), T = __shfl_sync(0xFFFFFFFFu, pd, 31);
            if (T == 0) return;
            uint32_t k = pe - ne, end = pd - ned;
#pragma unroll
            for (int q = 0; q < 4; ++q)
                if (rs[q].y > rs[q].x) {
                    end += rs[q].y - rs[q].x;
                    we0[k] = rs[q].x;
                    wdu[k] = dus[q];
                    wend[k] = end;
                    ++k;
                }
            __syncwarp();
            for (uint32_t f = lane; f < T; f += 32) {
                uint32_t lo = 0, hi = n - 1;   // first entry whose end > f
                while (lo < hi) {
                    const uint32_t mid = (lo + hi) >> 1;
                    if (wend[mid] > f) hi = mid;
                    else lo = mid + 1;
                }
                const uint32_t start = lo ? wend[lo - 1] : 0u;
                push_relax(p, we0[lo] + (f - start), wdu[lo]);
            }
            __syncwarp();
        };
        for (uint64_t base = gw * 32; base < n4; base += W * 32) {
            const uint64_t i = base + lane;
            int4 x = make_int4(INT32_MAX, INT32_MAX, INT32_MAX, INT32_MAX), y = x;
            if (i < n4) {
                x = a4[i];
                y = b4[i];
                if (x.x != y.x || x.y != y.y || x.z != y.z || x.w != y.w) b4[i] = x;
            }
            const int32_t xs[4] = {x.x, x.y, x.z, x.w}, ys[4] = {y.x, y.y, y.z, y.w};
            uint2 rs[4];
#pragma unroll
            for (int q = 0; q < 4; ++q) rs[q] = i < n4 ? frontier(4 * i + q, xs[q], ys[q]) : make_uint2(0u, 0u);
            relax_flat(xs, rs);
        }
        if (pb == 0 && threadIdx.x < 32)   // the last V % 4 sources
            for (uint64_t u0 = n4 * 4; u0 < p.g.V; u0 += 32) {
                const uint64_t u = u0 + lane;
                int32_t du = INT32_MAX;
                uint2 r = make_uint2(0u, 0u);
                if (u < p.g.V) {
                    du = din[u];
                    const int32_t dp = p.q.dprev[u];
                    if (dp != du) p.q.dprev[u] = du;
                    r = frontier(u, du, dp);
                }
                relax_ballot(du, r);
            }
    }
    if (!grid_barrier(lc, p.q.pctl)) return;
    // 2. heavy frontier sources, in pieces of PUSH_PIECE edges claimed dynamically by CTAs (a
    //    piece's edges: one per thread, independent loads)
    {
        __shared__ uint32_t hk;
        const uint32_t nh = __ldcg(p.q.pctl);
        for (;;) {
            if (threadIdx.x == 0) hk = atomicAdd(&p.q.pctl[3], 1u);
            __syncthreads();
            const uint32_t k = hk;
            __syncthreads();
            if (k >= nh) break;
            const uint2 pc = __ldcg(p.q.heavy + k);
            const int32_t du = din[pc.x];
            const uint32_t b = min(pc.y + PUSH_PIECE, __ldg(p.q.prp + pc.x + 1));
            for (uint32_t e = pc.y + threadIdx.x; e < b; e += PB) push_relax(p, e, du);
        }
    }
    if (!grid_barrier(lc, p.q.pctl)) return;
    if (pb == 0 && threadIdx.x == 0) {   // every CTA has read the piece count and left its claims
        p.q.pctl[0] = 0u;
        p.q.pctl[3] = 0u;
    }
    // 3. my vertices in blocks of 1024 (4 KiB, inside one chunk: chunks are multiples of 4 KiB
    //    and slices chunk-aligned), 4 per thread with 16-byte loads: d' = min(d, minima),
    //    instrumented stores, chunk state, vote, commit (a2, a3); the minima are reset to
    //    INT32_MAX for the next push round
    //    A block no frontier edge reached, in a chunk that did not change last round, already
    //    holds d' in the output replica (it holds d^{k-1} = d^k = d^{k+1} there, and so do the
    //    peers' copies): it is committed without loads or stores.
    unsigned long long cs = 0;
    const uint32_t nblk = (p.g.nv + 1023) / 1024;
    __shared__ uint32_t blk_work[PB];
    // the CTA's blocks pb, pb + P, ... in passes of PB: thread j reads block j's flags (one round
    // trip for the pass instead of one per block)
    for (uint32_t b0 = 0; pb + b0 * P < nblk; b0 += PB) {
        {
            const uint32_t tj = pb + (b0 + threadIdx.x) * P;
            uint32_t w = 0u;
            if (tj < nblk) {
                const bool prev = !p.first && proact::local_changed(lc, p.region_in, (uint64_t)(p.g.v0 + tj * 1024) * 4);
                const bool touched = !p.q.skip || __ldcg(p.q.ptouch + tj) != 0u;
                if (touched && p.q.skip) p.q.ptouch[tj] = 0u;
                w = (prev ? 2u : 0u) | (touched ? 1u : 0u);
            }
            blk_work[threadIdx.x] = w;
            __syncthreads();
        }
        for (uint32_t jb = 0; jb < PB; ++jb) {
            const uint32_t t = pb + (b0 + jb) * P;
            if (t >= nblk) break;
            const uint32_t lo = p.g.v0 + t * 1024, nvt = min(lo + 1024, p.g.v0 + p.g.nv) - lo;
            const uint32_t i = 4 * threadIdx.x;
            const uint64_t off = (uint64_t)lo * 4;
            const uint32_t work = blk_work[jb];
            if (work == 0u) {   // untouched, unchanged: commit only (a3)
                if (threadIdx.x == 0) proact::commit_span(lc, p.region_out, off, (uint64_t)nvt * 4);
                continue;
            }
            bool changed = false;
            if (i + 4 <= nvt) {
                const int4 old = *reinterpret_cast<const int4 *>(din + lo + i);
                int4 *mp = reinterpret_cast<int4 *>(p.q.ptmp + (lo - p.g.v0) + i);
                int4 m;
                asm volatile("ld.global.cg.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(m.x), "=r"(m.y), "=r"(m.z), "=r"(m.w) : "l"(mp));
                if (m.x != INT32_MAX || m.y != INT32_MAX || m.z != INT32_MAX || m.w != INT32_MAX)
                    *mp = make_int4(INT32_MAX, INT32_MAX, INT32_MAX, INT32_MAX);
                const int4 best = make_int4(min(old.x, m.x), min(old.y, m.y), min(old.z, m.z), min(old.w, m.w));
                proact::put(lc, p.region_out, (uint64_t)(lo + i) * 4, best);
                const int32_t ob[4] = {old.x, old.y, old.z, old.w}, bb[4] = {best.x, best.y, best.z, best.w};
    #pragma unroll
                for (int q = 0; q < 4; ++q)
                    if (bb[q] != ob[q]) {
                        changed = true;
                        cs += __ldg(p.g.outdeg + lo + i + q);
                    }
            } else {
                for (uint32_t j = i; j < nvt && j < i + 4; ++j) {
                    const uint32_t v = lo + j;
                    const int32_t old = din[v];
                    const int32_t m = ld_cg_i(p.q.ptmp + (v - p.g.v0));
                    if (m != INT32_MAX) p.q.ptmp[v - p.g.v0] = INT32_MAX;
                    const int32_t best = min(old, m);
                    proact::put(lc, p.region_out, (uint64_t)v * 4, best);
                    if (best != old) {
                        changed = true;
                        cs += __ldg(p.g.outdeg + v);
                    }
                }
            }
            const int any = __syncthreads_or(changed);   // orders the block's puts before the commit
            if (threadIdx.x == 0) {
                if (any) {
                    proact::mark_changed(lc, p.region_out, off);
                    proact::vote(lc);
                }
                if (any || (work & 2u)) proact::mark_push(lc, p.region_out, off);
                proact::commit_span(lc, p.region_out, off, (uint64_t)nvt * 4);
            }
        }
        __syncthreads();   // blk_work is rewritten by the next pass
    }
    count_changed(p, cs, &cs_cta);
    count_flush(p, &cs_cta);
}

__global__ void push_count_kernel(const uint32_t *rowidx, uint64_t E, uint32_t *cnt)
{
    for (uint64_t e = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; e < E; e += (uint64_t)gridDim.x * blockDim.x)
        atomicAdd(&cnt[rowidx[e]], 1u);
}
__global__ void push_scatter_kernel(const uint32_t *colptr, const uint32_t *rowidx, const int32_t *w, uint32_t nv,
                                    uint32_t *cursor, uint32_t *pcol, int32_t *pwt)
{
    for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < nv; v += gridDim.x * blockDim.x)
        for (uint32_t e = colptr[v]; e < colptr[v + 1]; ++e) {
            const uint32_t pos = atomicAdd(&cursor[rowidx[e]], 1u);
            pcol[pos] = v;
            pwt[pos] = w[e];
        }
}
__global__ void push_heavy_count_kernel(const uint32_t *prp, uint32_t V, uint32_t *n)
{
    uint32_t c = 0;   // pieces of all sources that can be heavy
    for (uint32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < V; u += gridDim.x * blockDim.x) {
        const uint32_t d = prp[u + 1] - prp[u];
        if (d > PUSH_HEAVY) c += (d + PUSH_PIECE - 1) / PUSH_PIECE;
    }
    if (c) atomicAdd(n, c);
}

__global__ void pr_init_kernel(float *contrib, const uint32_t *outdeg, uint32_t V, float r0)
{
    for (uint32_t u = blockIdx.x * blockDim.x + threadIdx.x; u < V; u += gridDim.x * blockDim.x)
        contrib[u] = outdeg[u] ? __fdiv_rn(r0, (float)outdeg[u]) : 0.f;
}

}  // namespace
extern "C" __attribute__((visibility("hidden"))) void proact_internal_l2_window(const void *base, size_t bytes);
extern "C" __attribute__((visibility("hidden"))) void proact_internal_keep_l1(const void *kernel);
extern "C" __attribute__((visibility("hidden"))) int proact_internal_smem_attr(const void *kernel, size_t bytes);
namespace {

// PROACT_L2_WINDOW=1: mark the gathered replica persisting in L2 for the phase launch
int l2_window_on()
{
    static const int on = [] {
        const char *e = getenv("PROACT_L2_WINDOW");
        return e ? atoi(e) : 0;
    }();
    return on;
}

// Cluster size of the hot-table kernels for a table of nhot entries: 0 = no table (plain kernels),
// 1 = one CTA holds it all (nhot <= HOT_SLICE), else the power of two of CTAs whose slices cover
// it.  A cluster kernel cannot share its grid with fused agent CTAs (PROACT_AGENT_FUSED while the
// launch tallies): then the plain kernels run (same results: the sums are exact).
int hot_cluster(uint32_t nhot)
{
    if (!nhot) return 0;
    if (nhot <= HOT_SLICE) return 1;
    int cl = 2;
    while ((uint32_t)cl * HOT_SLICE < nhot) cl *= 2;
    proact_config c;
    if (proact_get_config(&c) == PROACT_OK && c.agent_kernel == PROACT_AGENT_FUSED && proact_launch_tallies()) return 0;
    return cl;
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
    g->items = G.items;
    g->acc_f = G.acc_f;
    g->acc_i = G.acc_i;
    g->acc_cnt = G.acc_cnt;
    g->runv_pr = G.runv_pr;
    g->runv_ss = G.runv_ss;
    g->runv_ph = G.runv_ph;
    g->runv_p8 = G.runv_p8;
    g->rowidx_h = G.rowidx_h ? G.rowidx_h : G.rowidx;   // no table: plain ids (all < HOT_BIT)
    g->hot_ids = G.hot_ids;
    g->nhot = G.nhot;
    g->V = G.V;
    g->v0 = G.v0;
    g->nv = G.nv;
    g->nitems = G.nitems;
    return PROACT_OK;
}

}  // namespace

// ================================================================ C entry points
extern "C" {

int proact_graph_partition(const uint32_t *d_dst, unsigned long long E, unsigned V, int G, unsigned align,
                           unsigned *bounds, void *stream)
{
    if ((!d_dst && E) || !bounds || G < 1 || align == 0 || V == 0) return PROACT_ERR_INVALID;
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
    return proact_graph_build_ex(d_src, d_dst, d_w, E, V, v0, v1, -1, stream);
}

int proact_graph_build_ex(const uint32_t *d_src, const uint32_t *d_dst, const int32_t *d_w, unsigned long long E,
                          unsigned V, unsigned v0, unsigned v1, int hot, void *stream)
{
    if (((!d_src || !d_dst) && E) || v1 < v0 || v1 > V || V >= HOT_BIT) return PROACT_ERR_INVALID;
    if (hot < 0) {
        const char *e = getenv("PROACT_GRAPH_HOT");
        hot = e ? atoi(e) : (int)HOT_DEFAULT;
    }
    if ((uint32_t)hot > HOT_MAX) hot = (int)HOT_MAX;
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
    GCK(cudaMalloc((void **)&G.rowidx, 4 * ((size_t)e_own + 8)));   // +8: 16-byte index loads, runs of 8
    if (d_w) GCK(cudaMalloc((void **)&G.w, 4 * ((size_t)e_own + 4)));   // +4: 16-byte loads
    GCK(cudaMemcpyAsync(indeg, G.colptr, 4 * ((size_t)G.nv + 1), cudaMemcpyDeviceToDevice, s));   // cursors
    if (E) scatter_kernel<<<1184, 256, 0, s>>>(d_src, d_dst, d_w, E, v0, v1, indeg, G.rowidx, G.w);
    GCK(cudaGetLastError());
    GCK(cudaFreeAsync(indeg, s));
    // work items: one per 4 KiB vertex tile, tiles with more than SPLIT in-edges split
    {
        std::vector<uint32_t> cp((size_t)G.nv + 1);
        GCK(cudaMemcpyAsync(cp.data(), G.colptr, 4 * cp.size(), cudaMemcpyDeviceToHost, s));
        GCK(cudaStreamSynchronize(s));
        const uint32_t ntiles = (G.nv + GT - 1) / GT;
        std::vector<Item> split, whole;
        for (uint32_t t = 0; t < ntiles; ++t) {
            const uint32_t a = cp[(size_t)t * GT], b = cp[std::min<size_t>((size_t)(t + 1) * GT, G.nv)];
            const uint32_t n = std::max<uint32_t>(1, (b - a + SPLIT - 1) / SPLIT);
            for (uint32_t q = 0; q < n; ++q) {
                Item it{};
                it.tile = t;
                it.e0 = a + (uint32_t)((uint64_t)(b - a) * q / n);
                it.e1 = a + (uint32_t)((uint64_t)(b - a) * (q + 1) / n);
                it.nsplit = n;
                it.slot = n > 1 ? G.nslot : 0;
                (n > 1 ? split : whole).push_back(it);
            }
            if (n > 1) ++G.nslot;
        }
        split.insert(split.end(), whole.begin(), whole.end());   // big (hub) work first
        G.nitems = (uint32_t)split.size();
        uint64_t npr = 0, nss = 0, nph = 0, np8 = 0;
        for (Item &it : split) {
            it.run_pr = (uint32_t)npr;
            it.run_ss = (uint32_t)nss;
            it.run_ph = (uint32_t)nph;
            it.run_p8 = (uint32_t)np8;
            npr += (it.e1 - it.e0 + PROACT_PR_RUN - 1) / PROACT_PR_RUN;
            nss += (it.e1 - it.e0 + PROACT_SSSP_RUN - 1) / PROACT_SSSP_RUN;
            nph += (it.e1 - (PROACT_PRH_VEC ? (it.e0 & ~3u) : it.e0) + PROACT_PRH_RUN - 1) / PROACT_PRH_RUN;
            np8 += (it.e1 - (PROACT_PRH_VEC ? (it.e0 & ~3u) : it.e0) + PROACT_PRH_RUN_PR - 1) / PROACT_PRH_RUN_PR;
        }
        if (npr >= (1ull << 32) || nss >= (1ull << 32) || nph >= (1ull << 32) || np8 >= (1ull << 32)) return PROACT_ERR_NOMEM;
        GCK(cudaMalloc((void **)&G.items, sizeof(Item) * std::max<size_t>(1, split.size())));
        GCK(cudaMemcpy(G.items, split.data(), sizeof(Item) * split.size(), cudaMemcpyHostToDevice));
        GCK(cudaMalloc((void **)&G.runv_pr, 2 * std::max<uint64_t>(1, npr)));
        GCK(cudaMalloc((void **)&G.runv_ss, 2 * std::max<uint64_t>(1, nss)));
        GCK(cudaMalloc((void **)&G.runv_ph, 2 * std::max<uint64_t>(1, nph)));
        if (PROACT_PRH_RUN_PR != PROACT_PRH_RUN) GCK(cudaMalloc((void **)&G.runv_p8, 2 * std::max<uint64_t>(1, np8)));
        else G.runv_p8 = G.runv_ph;   // same runs: one array
        if (G.nitems) {
            runv_kernel<<<G.nitems, 256, 0, s>>>(G.items, G.colptr, G.nv, PROACT_PR_RUN, 0, G.runv_pr);
            runv_kernel<<<G.nitems, 256, 0, s>>>(G.items, G.colptr, G.nv, PROACT_SSSP_RUN, 1, G.runv_ss);
            runv_kernel<<<G.nitems, 256, 0, s>>>(G.items, G.colptr, G.nv, PROACT_PRH_RUN, 2, G.runv_ph);
            if (PROACT_PRH_RUN_PR != PROACT_PRH_RUN)
                runv_kernel<<<G.nitems, 256, 0, s>>>(G.items, G.colptr, G.nv, PROACT_PRH_RUN_PR, 3, G.runv_p8);
            GCK(cudaGetLastError());
        }
        const size_t ns = std::max<uint32_t>(1, G.nslot);
        GCK(cudaMalloc((void **)&G.acc_f, 8 * ns * GT));
        GCK(cudaMemset(G.acc_f, 0, 8 * ns * GT));
        GCK(cudaMalloc((void **)&G.acc_i, 4 * ns * GT));
        GCK(cudaMemset(G.acc_i, 0x7F, 4 * ns * GT));   // 0x7F7F7F7F: re-set to INT32_MAX below
        {
            std::vector<int32_t> inf(ns * GT, INT32_MAX);
            GCK(cudaMemcpy(G.acc_i, inf.data(), 4 * ns * GT, cudaMemcpyHostToDevice));
        }
        GCK(cudaMalloc((void **)&G.acc_cnt, 4 * ns));
        GCK(cudaMemset(G.acc_cnt, 0, 4 * ns));
    }
    // hot sources: the `hot` highest out-degree vertices (ties: smaller id), ascending ids
    if (hot > 0 && G.E_own > 0) {
        std::vector<uint32_t> od(V);
        GCK(cudaMemcpyAsync(od.data(), G.outdeg, 4 * (size_t)V, cudaMemcpyDeviceToHost, s));
        GCK(cudaStreamSynchronize(s));
        std::vector<uint32_t> ids;
        ids.reserve(V);
        for (uint32_t v = 0; v < V; ++v)
            if (od[v]) ids.push_back(v);
        const size_t H = std::min<size_t>((size_t)hot, ids.size());
        auto hotter = [&](uint32_t a, uint32_t b) { return od[a] != od[b] ? od[a] > od[b] : a < b; };
        if (H < ids.size()) std::nth_element(ids.begin(), ids.begin() + H, ids.end(), hotter);
        ids.resize(H);
        std::sort(ids.begin(), ids.end());
        G.nhot = (uint32_t)H;
        if (H) {
            uint32_t *slot = nullptr;
            GCK(cudaMalloc((void **)&G.hot_ids, 4 * H));
            GCK(cudaMemcpy(G.hot_ids, ids.data(), 4 * H, cudaMemcpyHostToDevice));
            GCK(cudaMalloc((void **)&slot, 4 * (size_t)V));
            GCK(cudaMemsetAsync(slot, 0xFF, 4 * (size_t)V, s));
            hot_slot_kernel<<<(unsigned)((H + 255) / 256), 256, 0, s>>>(G.hot_ids, (uint32_t)H, slot);
            GCK(cudaMalloc((void **)&G.rowidx_h, 4 * (G.E_own + 8)));
            unsigned long long *neh = nullptr;
            GCK(cudaMalloc((void **)&neh, 8));
            GCK(cudaMemsetAsync(neh, 0, 8, s));
            hot_encode_kernel<<<1184, 256, 0, s>>>(G.rowidx, G.E_own, slot, G.rowidx_h, neh);
            GCK(cudaGetLastError());
            unsigned long long eh = 0;
            GCK(cudaMemcpyAsync(&eh, neh, 8, cudaMemcpyDeviceToHost, s));
            GCK(cudaStreamSynchronize(s));
            G.e_hot = eh;
            GCK(cudaFree(neh));
            GCK(cudaFree(slot));
        }
    }
    // SSSP push rounds (reading R24): my in-edges grouped by source, dprev, minima, heavy list
    G.E_all = E;
    if (d_w) {
        GCK(cudaMalloc((void **)&G.prp, 4 * ((size_t)V + 1)));
        GCK(cudaMalloc((void **)&G.pcol, 4 * std::max<uint64_t>(1, G.E_own)));
        GCK(cudaMalloc((void **)&G.pwt, 4 * std::max<uint64_t>(1, G.E_own)));
        GCK(cudaMalloc((void **)&G.dprev, 4 * (size_t)V));
        GCK(cudaMalloc((void **)&G.ptmp, 4 * std::max<size_t>(1, G.nv)));
        GCK(cudaMalloc((void **)&G.ptouch, 4 * std::max<size_t>(1, (G.nv + 1023) / 1024)));
        GCK(cudaMemsetAsync(G.ptouch, 0, 4 * std::max<size_t>(1, (G.nv + 1023) / 1024), s));
        GCK(cudaMalloc((void **)&G.pctl, 16));
        GCK(cudaMalloc((void **)&G.dcnt, 16));
        GCK(cudaMallocHost((void **)&G.hcnt, 8));
        *G.hcnt = 0ull;
        GCK(cudaMemsetAsync(G.pctl, 0, 16, s));
        GCK(cudaMemsetAsync(G.dcnt, 0, 16, s));
        GCK(cudaMemsetAsync(G.dprev, 0x7F, 4 * (size_t)V, s));   // any value: round 0 rewrites it
        uint32_t *cnt = nullptr, *nh = nullptr;
        GCK(cudaMalloc((void **)&cnt, 4 * ((size_t)V + 1)));
        GCK(cudaMalloc((void **)&nh, 4));
        GCK(cudaMemsetAsync(cnt, 0, 4 * ((size_t)V + 1), s));
        GCK(cudaMemsetAsync(nh, 0, 4, s));
        if (G.E_own) push_count_kernel<<<1184, 256, 0, s>>>(G.rowidx, G.E_own, cnt);
        GCK(cudaGetLastError());
        rc = exclusive_scan(cnt, G.prp, (uint64_t)V + 1, s);
        if (rc) return rc;
        GCK(cudaMemcpyAsync(cnt, G.prp, 4 * ((size_t)V + 1), cudaMemcpyDeviceToDevice, s));   // cursors
        if (G.nv) push_scatter_kernel<<<1184, 256, 0, s>>>(G.colptr, G.rowidx, G.w, G.nv, cnt, G.pcol, G.pwt);
        push_heavy_count_kernel<<<1184, 256, 0, s>>>(G.prp, V, nh);
        GCK(cudaGetLastError());
        GCK(cudaMemcpyAsync(&G.nheavy_max, nh, 4, cudaMemcpyDeviceToHost, s));
        GCK(cudaStreamSynchronize(s));
        GCK(cudaMalloc((void **)&G.heavy, sizeof(uint2) * std::max<uint32_t>(1, G.nheavy_max)));
        GCK(cudaFree(cnt));
        GCK(cudaFree(nh));
        // ptmp must read INT32_MAX (0xFF.. is -1): set it properly
        {
            std::vector<int32_t> inf(std::max<size_t>(1, G.nv), INT32_MAX);
            GCK(cudaMemcpy(G.ptmp, inf.data(), 4 * inf.size(), cudaMemcpyHostToDevice));
        }
    }
    GCK(cudaStreamSynchronize(s));
    {
        // the opt-in stays at the round-1 value (a 45056-entry table): besides allowing the launch,
        // it steers the driver's default shared-memory carve-out for these kernels (they keep the
        // default, proact_internal_keep_l1) -- with a smaller opt-in the SMs they run on are
        // configured with less shared memory, so a separate agent (200 KiB) cannot be placed next
        // to them and 4 loopback ranks' agents no longer find SMs (observed: start-up timeout)
        const size_t b = 4 * ((size_t)PG * CPS + 45056);
        const void *pr[] = {(const void *)pagerank_hot_kernel<1>, (const void *)pagerank_hot_kernel<2>,
                            (const void *)pagerank_hot_kernel<4>, (const void *)pagerank_hot_kernel<8>};
        const void *ss[] = {(const void *)sssp_hot_kernel<1>, (const void *)sssp_hot_kernel<2>,
                            (const void *)sssp_hot_kernel<4>, (const void *)sssp_hot_kernel<8>};
        for (int k = 0; k < 4; ++k) {
            if (proact_internal_smem_attr(pr[k], b) || proact_internal_smem_attr(ss[k], b - 4 * CHG_WORDS))
                return PROACT_ERR_CUDA;
            proact_internal_keep_l1(pr[k]);
            proact_internal_keep_l1(ss[k]);
        }
        proact_internal_keep_l1((const void *)pagerank_kernel);
        proact_internal_keep_l1((const void *)sssp_kernel);
    }
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
    cudaFree(G.items);
    cudaFree(G.acc_f);
    cudaFree(G.acc_i);
    cudaFree(G.acc_cnt);
    cudaFree(G.runv_pr);
    cudaFree(G.runv_ss);
    if (G.runv_p8 != G.runv_ph) cudaFree(G.runv_p8);
    cudaFree(G.runv_ph);
    if (G.rowidx_h) cudaFree(G.rowidx_h);
    if (G.hot_ids) cudaFree(G.hot_ids);
    if (G.prp) {
        cudaFree(G.prp);
        cudaFree(G.pcol);
        cudaFree(G.pwt);
        cudaFree(G.dprev);
        cudaFree(G.ptmp);
        cudaFree(G.ptouch);
        cudaFree(G.heavy);
        cudaFree(G.pctl);
        cudaFree(G.dcnt);
        cudaFreeHost(G.hcnt);
    }
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

int proact_graph_hot(int id, unsigned *nhot, unsigned long long *e_hot)
{
    if (id < 0 || id >= MAXGRAPH || !graphs[id].used) return PROACT_ERR_INVALID;
    if (nhot) *nhot = graphs[id].nhot;
    if (e_hot) *e_hot = graphs[id].e_hot;
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
    static const int plain = [] {
        const char *e = getenv("PROACT_PR_KERNEL");
        return e && !strcmp(e, "plain") ? 1 : 0;
    }();
    if (l2_window_on()) {
        proact_region_info ri;
        if (proact_region_info_get(region_in, &ri) == PROACT_OK)
            proact_internal_l2_window(ri.replica_base, ri.total_bytes);
    }
    const int cl = hot_cluster(p.g.nhot);
    if (!plain && cl > 0) {
        const void *k = cl == 1 ? (const void *)pagerank_hot_kernel<1>
                      : cl == 2 ? (const void *)pagerank_hot_kernel<2>
                      : cl == 4 ? (const void *)pagerank_hot_kernel<4> : (const void *)pagerank_hot_kernel<8>;
        return proact_launch_ex(regs, 1, k, 0, GB * PG, args, 4 * ((size_t)PG * CPS + (cl == 1 ? p.g.nhot : HOT_SLICE)),
                                stream, cl > 1 ? (unsigned)cl << PROACT_LAUNCH_CLUSTER_SHIFT : 0u);
    }
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
    if (!p.g.w && graphs[graph].E_own) return PROACT_ERR_INVALID;   // built without weights
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
    // pull or push this round (reading R24).  PROACT_SSSP_PUSH: 0 = always pull, 1 = always push,
    // unset = by the frontier: the out-degree sum of my vertices that changed last round, scaled
    // to the whole graph (V / nv), below PROACT_SSSP_PUSH_PCT % (default 8) of the edges -> push.
    // The counter is the previous round's (copied after its kernel; stale only if the caller did
    // not synchronise -- either choice computes the same distances)
    Graph &Gr = graphs[graph];
    cudaStream_t s = (cudaStream_t)stream;
    const char *pe = getenv("PROACT_SSSP_PUSH");
    const int pmode = pe ? atoi(pe) : -1;
    if (first) Gr.round = 0;
    memset(&p.q, 0, sizeof(p.q));
    // A push round needs dprev = the previous round's input: push rounds keep it, pull rounds
    // only when asked (track) -- the copy costs a pass over V per round, so pull rounds track only
    // once the frontier is below 4x the push threshold, and a round may push only if the round
    // before it tracked.
    bool push = false, track = false, skip = true;   // skip: tiny frontiers (first round: the source)
    if (Gr.prp && pmode != 0) {
        if (first) {
            GCK(cudaMemsetAsync(Gr.dcnt, 0, 16, s));
            push = true;   // the frontier is the source alone
        } else if (pmode == 1) {
            push = true;
        } else {
            const char *pp = getenv("PROACT_SSSP_PUSH_PCT");
            const double pct = pp ? atof(pp) : 8.0;
            const double est = 100.0 * (double)*Gr.hcnt * (double)Gr.V / (double)std::max(1u, Gr.nv);
            push = Gr.tracked && est < pct * (double)Gr.E_all;
            track = est < 4.0 * pct * (double)Gr.E_all;
            const char *sp = getenv("PROACT_SSSP_SKIP_PCT");
            skip = est < (sp ? atof(sp) : 1.0) * (double)Gr.E_all;
        }
        p.q = PushDev{Gr.prp, Gr.pcol, Gr.pwt, Gr.dprev, Gr.ptmp, Gr.ptouch, Gr.heavy, Gr.pctl, Gr.dcnt,
                      track ? 1u : 0u, Gr.round & 1u, skip ? 1u : 0u, 0u};
    }
    Gr.tracked = push || track;
    Gr.last_mode = push ? 1 : 0;
    launch_ctx lc;
    void *args[2] = {&lc, &p};
    int regs[1] = {region_out};
    if (push) {
        rc = proact_launch(regs, 1, (const void *)sssp_push_kernel, 0, PB, args, 0, stream);
        if (rc) return rc;
        GCK(cudaMemcpyAsync(Gr.hcnt, Gr.dcnt + p.q.par, 8, cudaMemcpyDeviceToHost, s));
        Gr.round++;
        return PROACT_OK;
    }
    if (l2_window_on()) {
        proact_region_info ri;
        if (proact_region_info_get(region_in, &ri) == PROACT_OK)
            proact_internal_l2_window(ri.replica_base, ri.total_bytes);
    }
    auto after = [&](int rc2) {
        if (rc2 == PROACT_OK && p.q.dcnt) {
            if (cudaMemcpyAsync(Gr.hcnt, Gr.dcnt + p.q.par, 8, cudaMemcpyDeviceToHost, s) != cudaSuccess)
                return (int)PROACT_ERR_CUDA;
            Gr.round++;
        }
        return rc2;
    };
    const int cl = hot_cluster(p.g.nhot);
    if (cl > 0) {
        const void *k = cl == 1 ? (const void *)sssp_hot_kernel<1>
                      : cl == 2 ? (const void *)sssp_hot_kernel<2>
                      : cl == 4 ? (const void *)sssp_hot_kernel<4> : (const void *)sssp_hot_kernel<8>;
        return after(proact_launch_ex(regs, 1, k, 0, GB * PG, args, 4 * ((size_t)PG * CPS + (cl == 1 ? p.g.nhot : HOT_SLICE)),
                                      stream, cl > 1 ? (unsigned)cl << PROACT_LAUNCH_CLUSTER_SHIFT : 0u));
    }
    return after(proact_launch(regs, 1, (const void *)sssp_kernel, 0, GB, args, 0, stream));
}

int proact_sssp_last_mode(int graph)
{
    if (graph < 0 || graph >= MAXGRAPH || !graphs[graph].used) return PROACT_ERR_INVALID;
    return graphs[graph].last_mode;
}

// Force-load this translation unit's kernels (see proact_internal_preload_workloads).
__attribute__((visibility("hidden"))) int proact_internal_preload_graph(void)
{
    cudaFuncAttributes a;
    const void *k[] = {(const void *)count_kernel, (const void *)scan_blocks, (const void *)scan_totals,
                       (const void *)scan_add, (const void *)scatter_kernel, (const void *)pagerank_kernel,
                       (const void *)sssp_kernel, (const void *)pr_init_kernel, (const void *)runv_kernel,
                       (const void *)pagerank_hot_kernel<1>, (const void *)pagerank_hot_kernel<2>,
                       (const void *)pagerank_hot_kernel<4>, (const void *)pagerank_hot_kernel<8>,
                       (const void *)hot_slot_kernel, (const void *)hot_encode_kernel,
                       (const void *)sssp_hot_kernel<1>, (const void *)sssp_hot_kernel<2>,
                       (const void *)sssp_hot_kernel<4>, (const void *)sssp_hot_kernel<8>,
                       (const void *)sssp_push_kernel, (const void *)push_count_kernel,
                       (const void *)push_scatter_kernel, (const void *)push_heavy_count_kernel};
    for (const void *f : k)
        if (cudaFuncGetAttributes(&a, f) != cudaSuccess) return PROACT_ERR_CUDA;
    return PROACT_OK;
}

}  // extern "C"
