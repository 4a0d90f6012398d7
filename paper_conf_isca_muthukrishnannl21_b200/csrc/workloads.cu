// workloads.cu -- producer kernels of the PROACT hot path and their C entry points.
//
//   * Jacobi 2D 5-point stencil, fp32, row-partitioned (Sec. IV-C; BASELINE.json
//     configs 1-2; readings R9/R10: Laplace, Dirichlet boundary copied through, fixed
//     association 0.25*((up+down)+(left+right)), no FMA contraction).
//   * Transfer microbenchmark producer (Sec. IV-C, Sec. V-A: each source block
//     generates 4 KB; reading R14: word k of phase p = fmix32 chain of length K).
// Both are persistent producers: agent CTAs first (proact::agent_dispatch), then tiles dealt
// round-robin over the producer CTAs.  All stores go through proact::put (instrumented store,
// a2) and every tile ends with a release commit of its bytes (a3).
#include <cuda_runtime.h>
#include <stdint.h>

#include "agent.cuh"
#include "proact.h"
#include "proact_device.cuh"
#include "proact_workloads.h"

using proact::launch_ctx;
using proact::region_dev;

namespace {

// ---------------------------------------------------------------- commit helpers
// Commit `nb` bytes at region offset `off` for each lane of warp 0 that has a span (has=true);
// lanes whose spans fall in the same chunk are merged into one release atomic (a3).
__device__ __forceinline__ void warp_commit(const launch_ctx &lc, int r, bool has, uint64_t off, uint32_t nb)
{
    if (!proact::uses_agent(lc)) return;
    const region_dev &R = lc.ctx->region[r];
    uint64_t rel = off - R.own_off;
    uint32_t c = has ? (uint32_t)(rel / R.chunk_bytes) : 0xFFFFFFFFu;
    bool single = has && (uint32_t)((rel + nb - 1) / R.chunk_bytes) == c;
    uint32_t key = single ? c : 0xFFFFFFFFu;
    uint32_t grp = __match_any_sync(0xFFFFFFFFu, key);
    if (single) {
        if ((__ffs(grp) - 1) == (int)(threadIdx.x & 31)) {
            uint32_t b = nb * __popc(grp);
            uint32_t old = proact::atom_add_release_gpu(&R.counter[c], b);
            if (old + b > R.expected[c]) proact::raise_error(lc.ctx, proact::SITE_COMMIT, PROACT_ERR_PROTOCOL);
        }
    } else if (has) {
        proact::commit_span(lc, r, off, nb);
    }
}

__device__ __forceinline__ float4 ld_nc_f4(const float *p)
{
    float4 v;
    asm volatile("ld.global.nc.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
    return v;
}
__device__ __forceinline__ float4 ld_f4(const float *p)
{
    float4 v;
    asm volatile("ld.global.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p));
    return v;
}
__device__ __forceinline__ float ld_nc_f(const float *p)
{
    float v;
    asm volatile("ld.global.nc.f32 %0, [%1];" : "=f"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ float ld_f(const float *p)
{
    float v;
    asm volatile("ld.global.f32 %0, [%1];" : "=f"(v) : "l"(p));
    return v;
}

// ---------------------------------------------------------------- Jacobi
constexpr int JB = 256;           // threads per CTA
constexpr int JW = 4 * JB;        // strip width in columns (float4 per thread) = 4 KiB of a row

struct Row { float4 v; float l, r; };

// Row k of the input as seen by this thread: 4 cells at column j and (warp-edge lanes) the
// left/right scalars.  `local` rows (mine, written by my previous phase) use the read-only
// path; halo rows pushed by a peer during this kernel use plain (coherent) loads.
__device__ __forceinline__ Row load_row(const float *in, int64_t N, int64_t k, int64_t j, bool act,
                                        bool local, uint32_t lane)
{
    Row o;
    o.v = make_float4(0.f, 0.f, 0.f, 0.f);
    o.l = 0.f;
    o.r = 0.f;
    if (k < 0 || k >= N || !act) return o;
    const float *p = in + k * N + j;
    if (local) {
        o.v = ld_nc_f4(p);
        if (lane == 0 && j > 0) o.l = ld_nc_f(p - 1);
        if (lane == 31 && j + 4 < N) o.r = ld_nc_f(p + 4);
    } else {
        o.v = ld_f4(p);
        if (lane == 0 && j > 0) o.l = ld_f(p - 1);
        if (lane == 31 && j + 4 < N) o.r = ld_f(p + 4);
    }
    return o;
}

__global__ void __launch_bounds__(JB) jacobi_kernel(launch_ctx lc, proact_jacobi_params p)
{
    if (proact::agent_dispatch(lc)) return;
    const region_dev &Ri = lc.ctx->region[p.region_in];
    const float *in = reinterpret_cast<const float *>(Ri.base);
    const int64_t N = p.N, row0 = p.row0, rend = p.row0 + p.nrows;
    const int rb = p.rows_per_tile;
    const uint32_t lane = threadIdx.x & 31u;
    const int64_t nstrips = (N + JW - 1) / JW;
    const int64_t nbands = (p.nrows + rb - 1) / rb;
    const int64_t ntiles = nbands * nstrips;
    for (int64_t t = proact::producer_block(lc); t < ntiles; t += proact::producer_grid(lc)) {
        // interior bands first, the two halo-dependent edge bands last (they wait on flags)
        int64_t bi = t / nstrips, strip = t % nstrips, band;
        if (nbands <= 2) band = bi;
        else if (bi < nbands - 2) band = bi + 1;
        else band = bi == nbands - 2 ? 0 : nbands - 1;
        const int64_t i0 = row0 + band * rb, i1 = min(i0 + (int64_t)rb, rend);
        const int64_t c0 = strip * JW, c1 = min(c0 + (int64_t)JW, N);
        const bool top_halo = i0 == row0 && i0 > 0, bot_halo = i1 == rend && i1 < N;
        if (top_halo || bot_halo) {   // (a7) wait for the neighbours' boundary rows of gen-1
            if (threadIdx.x == 0) {
                const int64_t a = c0 > 0 ? c0 - 1 : 0, b = c1 < N ? c1 + 1 : N;
                if (top_halo) proact::wait_range(lc, p.region_in, (uint64_t)((i0 - 1) * N + a) * 4, (uint64_t)(b - a) * 4);
                if (bot_halo) proact::wait_range(lc, p.region_in, (uint64_t)(i1 * N + a) * 4, (uint64_t)(b - a) * 4);
            }
            __syncthreads();
        }
        const int64_t j = c0 + 4 * (int64_t)threadIdx.x;
        const bool act = j < c1;
        Row up = load_row(in, N, i0 - 1, j, act, i0 - 1 >= row0, lane);
        Row cur = load_row(in, N, i0, j, act, true, lane);
        Row dn = load_row(in, N, i0 + 1, j, act, i0 + 1 < rend, lane);
        for (int64_t i = i0; i < i1; ++i) {
            Row nx;
            if (i + 2 <= i1) nx = load_row(in, N, i + 2, j, act, i + 2 < rend, lane);
            // horizontal neighbours: lanes exchange, warp-edge lanes use their scalars
            float lft = __shfl_up_sync(0xFFFFFFFFu, cur.v.w, 1);
            float rgt = __shfl_down_sync(0xFFFFFFFFu, cur.v.x, 1);
            if (lane == 0) lft = cur.l;
            if (lane == 31) rgt = cur.r;
            if (act) {
                float4 o;
                if (i == 0 || i == N - 1) {
                    o = cur.v;
                } else {
                    o.x = __fmul_rn(0.25f, __fadd_rn(__fadd_rn(up.v.x, dn.v.x), __fadd_rn(lft, cur.v.y)));
                    o.y = __fmul_rn(0.25f, __fadd_rn(__fadd_rn(up.v.y, dn.v.y), __fadd_rn(cur.v.x, cur.v.z)));
                    o.z = __fmul_rn(0.25f, __fadd_rn(__fadd_rn(up.v.z, dn.v.z), __fadd_rn(cur.v.y, cur.v.w)));
                    o.w = __fmul_rn(0.25f, __fadd_rn(__fadd_rn(up.v.w, dn.v.w), __fadd_rn(cur.v.z, rgt)));
                    if (j == 0) o.x = cur.v.x;
                    if (j + 3 == N - 1) o.w = cur.v.w;
                }
                proact::put(lc, p.region_out, (uint64_t)(i * N + j) * 4, o);
            }
            up = cur;
            cur = dn;
            dn = nx;
        }
        __syncthreads();
        if (threadIdx.x < 32) {   // (a3) one span per row of the tile, merged per chunk
            for (int64_t k0 = i0; k0 < i1; k0 += 32) {
                const int64_t i = k0 + lane;
                warp_commit(lc, p.region_out, i < i1, (uint64_t)(i * N + c0) * 4, (uint32_t)((c1 - c0) * 4));
            }
        }
    }
}

// ---------------------------------------------------------------- microbenchmark
__device__ __forceinline__ uint32_t fmix32(uint32_t h)
{
    h ^= h >> 16;
    h *= 0x85EBCA6Bu;
    h ^= h >> 13;
    h *= 0xC2B2AE35u;
    h ^= h >> 16;
    return h;
}
__device__ __forceinline__ uint32_t micro_value(uint32_t k, uint32_t phase, uint32_t seed, int K)
{
    uint32_t v = fmix32(k ^ (phase * 0x9E3779B9u) ^ seed);
    for (int i = 1; i < K; ++i) v = fmix32(v);
    return v;
}

constexpr int MB = 256;            // threads; one 4 KiB tile (1024 words) per CTA pass (L279)

__global__ void __launch_bounds__(MB) micro_kernel(launch_ctx lc, proact_micro_params p)
{
    if (proact::agent_dispatch(lc)) return;
    const region_dev &R = lc.ctx->region[p.region];
    const uint64_t w_lo = R.own_off / 4, w_hi = (R.own_off + R.own_bytes) / 4;
    const uint64_t ntiles = (w_hi - w_lo + 1023) / 1024;
    for (uint64_t t = proact::producer_block(lc); t < ntiles; t += proact::producer_grid(lc)) {
        const uint64_t t0 = w_lo + t * 1024, t1 = min(t0 + 1024, w_hi);
        if (!p.scattered) {
            const uint64_t k = t0 + 4 * threadIdx.x;
            if (k + 4 <= t1) {
                uint4 v;
                v.x = micro_value((uint32_t)k, p.phase, p.seed, p.K);
                v.y = micro_value((uint32_t)k + 1, p.phase, p.seed, p.K);
                v.z = micro_value((uint32_t)k + 2, p.phase, p.seed, p.K);
                v.w = micro_value((uint32_t)k + 3, p.phase, p.seed, p.K);
                proact::put(lc, p.region, k * 4, v);
            } else {
                for (uint64_t q = k; q < t1 && q < k + 4; ++q)
                    proact::put(lc, p.region, q * 4, micro_value((uint32_t)q, p.phase, p.seed, p.K));
            }
        } else {
            // scattered store order inside the 4 KiB tile: position (j*389) mod 1024 (bijection)
            for (int s = 0; s < 4; ++s) {
                const uint32_t jj = threadIdx.x + MB * s;
                const uint64_t q = t0 + ((jj * 389u) & 1023u);
                if (q < t1) proact::put(lc, p.region, q * 4, micro_value((uint32_t)q, p.phase, p.seed, p.K));
            }
        }
        __syncthreads();
        if (threadIdx.x == 0) proact::commit_span(lc, p.region, t0 * 4, (t1 - t0) * 4);
    }
}

}  // namespace

// ================================================================ C entry points
extern "C" {

int proact_jacobi_phase(int region_in, int region_out, long long N, int rows_per_tile, void *stream)
{
    proact_region_info ri, ro;
    int rc = proact_region_info_get(region_in, &ri);
    if (rc) return rc;
    rc = proact_region_info_get(region_out, &ro);
    if (rc) return rc;
    if (N < 1 || N % 4 || region_in == region_out) return PROACT_ERR_INVALID;
    const uint64_t rowb = (uint64_t)N * 4;
    if (ri.own_offset != ro.own_offset || ri.own_bytes != ro.own_bytes || ri.total_bytes != rowb * N ||
        ro.total_bytes != rowb * N || ro.own_offset % rowb || ro.own_bytes % rowb)
        return PROACT_ERR_INVALID;
    if (rows_per_tile <= 0) rows_per_tile = 16;
    proact_jacobi_params p;
    p.region_in = region_in;
    p.region_out = region_out;
    p.N = N;
    p.row0 = (long long)(ro.own_offset / rowb);
    p.nrows = (long long)(ro.own_bytes / rowb);
    p.rows_per_tile = rows_per_tile;
    p.pad = 0;
    launch_ctx lc;
    void *args[2] = {&lc, &p};
    int regs[1] = {region_out};
    return proact_launch(regs, 1, (const void *)jacobi_kernel, 0, JB, args, 0, stream);
}

int proact_micro_phase(int region, unsigned phase, unsigned seed, int K, int scattered, void *stream)
{
    if (K < 1) return PROACT_ERR_INVALID;
    proact_micro_params p;
    p.region = region;
    p.phase = phase;
    p.seed = seed;
    p.K = K;
    p.scattered = scattered;
    p.pad = 0;
    launch_ctx lc;
    void *args[2] = {&lc, &p};
    int regs[1] = {region};
    return proact_launch(regs, 1, (const void *)micro_kernel, 0, MB, args, 0, stream);
}

}  // extern "C"

// ================================================================ host-buffer Jacobi (e2e)
namespace {
struct JacobiHost {
    long long N = 0;
    size_t chunk = 0;
    float *a = nullptr, *b = nullptr;
    int ra = -1, rb = -1;
};
thread_local JacobiHost jh;
}  // namespace

extern "C" int proact_jacobi_solve_host(const float *h_x0, float *h_out, long long N, int iters,
                                        size_t chunk_bytes, int rows_per_tile, void *stream,
                                        unsigned long long *bytes_h2d, unsigned long long *bytes_d2h)
{
    const int G = proact_world(), g = proact_rank();
    if (G <= 0) return PROACT_ERR_STATE;
    if (!h_x0 || !h_out || N < 4 || N % 4 || iters < 0) return PROACT_ERR_INVALID;
    const long long r0 = N * g / G, r1 = N * (g + 1) / G;
    const size_t rowb = (size_t)N * 4;
    cudaStream_t s = (cudaStream_t)stream;
    if (jh.N && jh.N != N) return PROACT_ERR_STATE;   // regions cannot be unregistered
    if (!jh.N) {
        if (cudaMalloc((void **)&jh.a, rowb * N) != cudaSuccess) return PROACT_ERR_NOMEM;
        if (cudaMalloc((void **)&jh.b, rowb * N) != cudaSuccess) return PROACT_ERR_NOMEM;
        const uint64_t all = G >= 64 ? ~0ull : ((1ull << G) - 1);
        jh.ra = proact_register_region((char *)jh.a + r0 * rowb, (r1 - r0) * rowb, chunk_bytes, all);
        if (jh.ra < 0) return jh.ra;
        jh.rb = proact_register_region((char *)jh.b + r0 * rowb, (r1 - r0) * rowb, chunk_bytes, all);
        if (jh.rb < 0) return jh.rb;
        jh.N = N;
        jh.chunk = chunk_bytes;
    } else if (jh.chunk != chunk_bytes) {
        int rc = proact_region_rechunk(jh.ra, chunk_bytes);
        if (rc) return rc;
        rc = proact_region_rechunk(jh.rb, chunk_bytes);
        if (rc) return rc;
        jh.chunk = chunk_bytes;
    }
    if (cudaMemcpyAsync(jh.a, h_x0, rowb * N, cudaMemcpyHostToDevice, s) != cudaSuccess) return PROACT_ERR_CUDA;
    for (int k = 0; k < iters; ++k) {
        const int in = (k & 1) ? jh.rb : jh.ra, out = (k & 1) ? jh.ra : jh.rb;
        int rc = proact_jacobi_phase(in, out, N, rows_per_tile, stream);
        if (rc) return rc;
        rc = proact_phase_sync(stream, k == iters - 1 ? PROACT_SYNC_BARRIER : PROACT_SYNC_SIGNAL);
        if (rc) return rc;
    }
    const float *res = (iters & 1) ? jh.b : jh.a;
    if (cudaMemcpyAsync(h_out + r0 * N, res + r0 * N, (r1 - r0) * rowb, cudaMemcpyDeviceToHost, s) != cudaSuccess)
        return PROACT_ERR_CUDA;
    if (bytes_h2d) *bytes_h2d = (unsigned long long)(rowb * N);
    if (bytes_d2h) *bytes_d2h = (unsigned long long)((r1 - r0) * rowb);
    return PROACT_OK;
}
