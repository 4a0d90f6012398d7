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

#include <cstdlib>
#include <type_traits>

#include "proact.h"
#include "proact_device.cuh"
#include "proact_workloads.h"

using proact::launch_ctx;
using proact::region_dev;

// runtime.cu: cudaFuncAttributeMaxDynamicSharedMemorySize for the current device, once per
// (device, kernel) and never lowered; 0 or a cudaError_t
extern "C" __attribute__((visibility("hidden"))) int proact_internal_smem_attr(const void *kernel, size_t bytes);

namespace {

using proact::warp_commit;

// ---------------------------------------------------------------- Jacobi
// Tile = rows_per_tile rows x one 1024-column strip (4 KiB of a row).  Warp-specialised CTA:
// one producer warp streams the tile's input rows (plus the two halo rows) into a JS-deep
// shared-memory ring with 1D bulk async copies (cp.async.bulk = TMA engine, completion on a
// per-slot "full" mbarrier); eight compute warps consume them (each thread: 4 columns, float4
// up/cur/dn rolled in registers, horizontal neighbours by warp shuffle, warp-edge lanes from
// shared memory) and release slots on per-slot "empty" mbarriers.  The row stream runs across
// the CTA's tiles without draining.  Every input row is read from HBM once per tile (+2 halo
// rows per tile, L2 hits); outputs are 16-byte stores.
#ifndef PROACT_JACOBI_JC
#define PROACT_JACOBI_JC 8
#endif
#ifndef PROACT_JACOBI_JV
#define PROACT_JACOBI_JV 1
#endif
constexpr int JC = PROACT_JACOBI_JC;    // compute warps
constexpr int JV = PROACT_JACOBI_JV;    // float4 column groups per compute thread (JC * JV = 8)
// Three instantiations (proact_launch_mode): MODE 0 (no remote destinations this launch: LOCAL /
// INLINE / BULK / G = 1) has 8 compute + 1 TMA warp and the register budget of 4 CTAs/SM; MODE 1
// (tallies for a polling agent) adds a committer warp that publishes the tile tallies so the
// compute warps never wait on a release; MODE 2 (PROACT_AGENT_PRODUCER) replaces it with a
// transfer warp: the compute warps store each output row strip to the local replica and into a
// shared-memory ring, and the transfer warp bulk-stores the ring's spans (JSR rows) to every
// destination mirror, then counts the delivered bytes (proact::tile_pusher).
#ifndef PROACT_JACOBI_RING_TP
#define PROACT_JACOBI_RING_TP 10
#endif
#ifndef PROACT_JACOBI_OUT_RING
#define PROACT_JACOBI_OUT_RING 2
#endif
#ifndef PROACT_JACOBI_SPAN_ROWS
#define PROACT_JACOBI_SPAN_ROWS 4
#endif
constexpr uint32_t JOS = PROACT_JACOBI_OUT_RING;   // MODE 2: output slots of JSR row strips (4 KiB each)
constexpr int JSR = PROACT_JACOBI_SPAN_ROWS;       // rows per pushed span
constexpr int JW = JC * 32 * 4 * JV;    // strip width in columns = 4 KiB of a row
#ifndef PROACT_JACOBI_OUT_STORE   // output stores: 0 plain, 1 st.cs in MODE 0 (an evict-first hint
#define PROACT_JACOBI_OUT_STORE 1   // measured between the two, profiles/r02k_jacobi_store_policy.log)
#endif
#ifndef PROACT_JACOBI_OUT_EVICT_LAST   // G > 1: output rows evict-last until the agent has read them
#define PROACT_JACOBI_OUT_EVICT_LAST 0
#endif
#ifndef PROACT_JACOBI_RING
#define PROACT_JACOBI_RING 16
#endif
constexpr int SLOT = JW + 8;            // floats per slot: columns [c0-4, c0+JW+4)
constexpr int JTD = 32;                 // tile-id ring (stream warp -> compute -> committer)
template <int MODE> struct JCfg {
    static constexpr int threads = (JC + 1 + (MODE ? 1 : 0)) * 32;
    static constexpr int minb = MODE ? 3 : 4;
    static constexpr int js = MODE == 2 ? PROACT_JACOBI_RING_TP : PROACT_JACOBI_RING;   // input ring depth
    static constexpr size_t ctl = (size_t)js * SLOT * 4 + (size_t)2 * js * 8 + 4 * 8 + JTD * 4;
    static constexpr size_t out = (ctl + 127) / 128 * 128;   // MODE 2: output ring, then its control
    static constexpr size_t smem = MODE == 2 ? out + (size_t)JOS * JSR * JW * 4 + sizeof(proact::tile_ring_ctl<JOS>) : ctl;
};

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *b, uint32_t cnt)
{
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(cnt) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *b, uint32_t bytes)
{
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *b)
{
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *b, uint32_t parity)
{
    // (a suspend-time hint on this try_wait measured no different: profiles/r02k_jacobi_wait_hint.log)
    uint32_t done;
    do {
        asm volatile("{\n\t.reg .pred p;\n\t"
                     "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
                     "selp.u32 %0, 1, 0, p;\n\t}"
                     : "=r"(done) : "r"(smem_u32(b)), "r"(parity) : "memory");
    } while (!done);
}
__device__ __forceinline__ void bulk_g2s(void *sdst, const void *gsrc, uint32_t bytes, uint64_t *bar)
{
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(smem_u32(sdst)), "l"(gsrc), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ float4 lds128(const float *p) { return *reinterpret_cast<const float4 *>(p); }

struct JTile {
    int i0, i1, c0, c1, kfirst, klast;
};

#ifndef PROACT_JACOBI_EDGES_FIRST
#define PROACT_JACOBI_EDGES_FIRST 1
#endif
__device__ __forceinline__ bool edges_first(const launch_ctx &lc)
{
    return PROACT_JACOBI_EDGES_FIRST && (lc.mech == PROACT_MECH_FUSED || lc.mech == PROACT_MECH_ELIDE);
}

// Tile t of this rank.  Credit-synchronised mechanisms (INLINE / BULK / DMA): interior bands
// first, the two halo-dependent edge bands last, so the wait for the neighbours' phase credit
// (a7) comes as late as possible.  Flag-synchronised ones (FUSED / ELIDE, edges_first): the edge
// bands FIRST -- they are what the neighbours need next phase, so their pushes overlap this
// phase's interior instead of trailing it, and the neighbours produced the rows they wait on at
// the start of the previous phase.
__device__ __forceinline__ JTile jtile(int t, int nstrips, int nbands, int rb, int row0, int rend, int N,
                                       bool edges_first)
{
    const int bi = t / nstrips, strip = t - bi * nstrips;
    int band;
    if (nbands <= 2) band = bi;
    else if (edges_first) band = bi == 0 ? 0 : (bi == 1 ? nbands - 1 : bi - 1);
    else if (bi < nbands - 2) band = bi + 1;
    else band = bi == nbands - 2 ? 0 : nbands - 1;
    JTile T;
    T.i0 = row0 + band * rb;
    T.i1 = min(T.i0 + rb, rend);
    T.c0 = strip * JW;
    T.c1 = min(T.c0 + JW, N);
    T.kfirst = T.i0 > 0 ? T.i0 - 1 : 0;
    T.klast = T.i1 < N - 1 ? T.i1 : N - 1;
    return T;
}

// Producer warp (one lane): the CTA's row stream, slot by slot.  Tiles are claimed dynamically
// (proact::claim_tile); the claimed id goes to tids[k % JTD] before the tile's first row is
// armed, so the mbarrier arrival (release) publishes it to the compute warps.  After the last
// tile an end marker (-1, a tx-less arrival on the next slot) lets them exit.
template <int JS>
__device__ __noinline__ void jacobi_stream(const launch_ctx &lc, const proact_jacobi_params &p, float *ring,
                                           uint64_t *full, uint64_t *empty, int *tids, int ntiles,
                                           int nstrips, int nbands)
{
    const int N = (int)p.N, row0 = (int)p.row0, rend = (int)(p.row0 + p.nrows), rb = p.rows_per_tile;
    const char *in = lc.ctx->region[p.region_in].base;
    uint32_t q = 0;
    for (uint32_t kt = 0;; ++kt) {
        const uint32_t t = proact::claim_tile(lc, (uint32_t)ntiles);
        const uint32_t slot0 = q % JS;
        if (q >= JS) mbar_wait(&empty[slot0], ((q / JS) - 1) & 1u);
        if (t >= (uint32_t)ntiles) {
            tids[kt % JTD] = -1;
            mbar_arrive(&full[slot0]);
            return;
        }
        tids[kt % JTD] = (int)t;
        const JTile T = jtile((int)t, nstrips, nbands, rb, row0, rend, N, edges_first(lc));
        const int lo = T.c0 >= 4 ? T.c0 - 4 : 0, hi = min(T.c0 + JW + 4, N);
        const uint32_t bytes = (uint32_t)(hi - lo) * 4;
        for (int k = T.kfirst; k <= T.klast; ++k, ++q) {
            const uint32_t slot = q % JS;
            if (q >= JS && k != T.kfirst) mbar_wait(&empty[slot], ((q / JS) - 1) & 1u);
            const uint64_t goff = ((uint64_t)k * N + lo) * 4;
            if (k < row0 || k >= rend) {   // (a7) halo row produced by a peer: wait, then
                proact::wait_range(lc, p.region_in, goff, bytes);
                asm volatile("fence.proxy.async;" ::: "memory");   // generic -> async proxy
            }
            mbar_expect_tx(&full[slot], bytes);
            bulk_g2s(ring + slot * SLOT + (lo - (T.c0 - 4)), in + goff, bytes, &full[slot]);
        }
    }
}

template <int MODE>
__global__ void __launch_bounds__(JCfg<MODE>::threads, JCfg<MODE>::minb)
jacobi_kernel(launch_ctx lc, proact_jacobi_params p)
{
    constexpr bool TALLY = MODE == 1;
    constexpr int JS = JCfg<MODE>::js;
    if (proact::agent_dispatch(lc)) return;
#ifdef PROACT_TIMING_EXP
    unsigned long long *xprof = lc.ctx->prof;
    const unsigned long long xt0 = proact::globaltimer();
    if (xprof && threadIdx.x == 0) atomicMax(&xprof[2], ~xt0);
    struct XEnd {
        unsigned long long *p, t0;
        __device__ ~XEnd() {
            if (p) {
                const unsigned long long t = proact::globaltimer();
                atomicMax(&p[3], t);
                atomicAdd(&p[4], t - t0);
                atomicAdd(&p[5], 1ull);
            }
        }
    } xend{(xprof && threadIdx.x == 0) ? xprof : nullptr, xt0};
#endif
    extern __shared__ __align__(128) unsigned char jsm[];
    float *ring = reinterpret_cast<float *>(jsm);
    uint64_t *full = reinterpret_cast<uint64_t *>(jsm + (size_t)JS * SLOT * 4);
    uint64_t *empty = full + JS;
    uint64_t *tdone = empty + JS;    // [2] compute warps finished tile k (k & 1)
    uint64_t *cdone = tdone + 2;     // [2] committer finished tile k (k & 1)
    int *tids = reinterpret_cast<int *>(cdone + 2);   // [JTD] claimed tile ids, by sequence
    float *oring = reinterpret_cast<float *>(jsm + JCfg<MODE>::out);   // MODE 2: JOS x JSR row strips
    auto *tp = reinterpret_cast<proact::tile_ring_ctl<JOS> *>(jsm + JCfg<MODE>::out + (size_t)JOS * JSR * JW * 4);
#ifndef PROACT_JACOBI_RT_TALLY
#define PROACT_JACOBI_RT_TALLY 1
#endif
    // (the runtime test in the TALLY=false instantiation keeps its compute loop's code identical
    //  to the measured-fastest build; with tallies off at compile time it was ~15% slower)
    const bool tally = MODE != 2 && (TALLY || PROACT_JACOBI_RT_TALLY) && proact::uses_agent(lc);
    const int N = (int)p.N, row0 = (int)p.row0, rend = (int)(p.row0 + p.nrows);
    const int rb = p.rows_per_tile;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int nstrips = (N + JW - 1) / JW;
    const int nbands = ((int)p.nrows + rb - 1) / rb;
    const int ntiles = nbands * nstrips;
    if (tid == 0) {
        for (int s = 0; s < JS; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], JC);
        }
        for (int s = 0; s < 2; ++s) {
            mbar_init(&tdone[s], JC);
            mbar_init(&cdone[s], 1);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        if (MODE == 2) proact::tp_init(tp, JC);
    }
    __syncthreads();
    if (warp == JC) {
        if (lane == 0) jacobi_stream<JS>(lc, p, ring, full, empty, tids, ntiles, nstrips, nbands);
        return;
    }
    if (MODE == 2 && warp == JC + 1) {   // the transfer warp (PROACT_AGENT_PRODUCER)
        proact::tile_pusher<JOS>(lc, p.region_out, reinterpret_cast<const unsigned char *>(oring), JSR * JW * 4, tp,
                                 JW * 4, (uint64_t)N * 4, true);
        return;
    }
    if constexpr (TALLY) if (warp == JC + 1) {
        // (a3) committer warp: after the compute warps' mbarrier arrival for tile k (release ->
        // acquire at CTA scope), commit the tile's rows with release RMWs, merged per chunk.
        // The compute warps never stall on the commit's fence latency.
        if (!tally) return;
        for (uint32_t k = 0;; ++k) {
            mbar_wait(&tdone[k & 1u], (k >> 1) & 1u);
            const int t = tids[k % JTD];   // written by the stream warp, ordered by the tile's
            if (t < 0) return;             // row barriers and the compute warps' tdone arrival
            const JTile T = jtile(t, nstrips, nbands, rb, row0, rend, N, edges_first(lc));
            for (int k0 = T.i0; k0 < T.i1; k0 += 32) {
                const int i = k0 + lane;
                warp_commit(lc, p.region_out, i < T.i1, ((uint64_t)i * N + T.c0) * 4, (uint32_t)(T.c1 - T.c0) * 4);
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&cdone[k & 1u]);
        }
        return;
    }
    char *outb = lc.ctx->region[p.region_out].base;
    uint64_t pol_out = 0;
    if (PROACT_JACOBI_OUT_EVICT_LAST) asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol_out));
    uint32_t q = 0;    // next stream item (same sequence as the producer warp's)
    uint32_t kt = 0;   // tiles handed to the committer
    uint32_t oq = 0;   // MODE 2: next output span of this CTA
    for (;;) {
        // the next tile's first stream item carries its id (or the end marker)
        mbar_wait(&full[q % JS], (q / JS) & 1u);
        const int t = tids[kt % JTD];
        if (t < 0) {
            if (tally && TALLY && lane == 0) mbar_arrive(&tdone[kt & 1u]);   // release the committer
            if (MODE == 2) {   // end marker for the transfer warp
                proact::tp_acquire(tp, oq);
                if (tid == 0) tp->desc[oq % JOS] = proact::tile_desc{0, 0, proact::TD_END};
                proact::tp_publish(tp, oq);
            }
            break;
        }
        const JTile T = jtile(t, nstrips, nbands, rb, row0, rend, N, edges_first(lc));
        // group g of this thread: columns [c0 + 4*tid + g*GW, +4), GW = the compute warps' width
        constexpr int GW = JC * 32 * 4;
        const float *ringf = ring + 4 + 4 * tid;
        float4 up[JV], cur[JV], dn[JV];
        bool act[JV];
#pragma unroll
        for (int g = 0; g < JV; ++g) {
            act[g] = T.c0 + 4 * tid + g * GW < T.c1;
            up[g] = make_float4(0.f, 0.f, 0.f, 0.f);
            dn[g] = up[g];
        }
        if (T.i0 > 0) {   // top halo / previous row: registers only, release at once
            mbar_wait(&full[q % JS], (q / JS) & 1u);
#pragma unroll
            for (int g = 0; g < JV; ++g)
                if (act[g]) up[g] = lds128(ringf + (q % JS) * SLOT + g * GW);
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[q % JS]);
            ++q;
        }
        uint32_t qcur = q;
        mbar_wait(&full[q % JS], (q / JS) & 1u);
#pragma unroll
        for (int g = 0; g < JV; ++g) cur[g] = act[g] ? lds128(ringf + (q % JS) * SLOT + g * GW) : up[g];
        ++q;
        // interior tiles (no Dirichlet row or column, full strip, plain stores) run a copy of the
        // row loop with those checks compiled out
        const bool fast = T.i0 > 0 && T.i1 < N && T.c0 > 0 && T.c0 + JW < N &&
                          (MODE == 2 || (lc.mech != PROACT_MECH_INLINE && !(PROACT_JACOBI_OUT_EVICT_LAST && tally)));
        // MODE 2: does any chunk this tile writes have a destination?  Tiles that only write
        // chunks bound nowhere (halo-only interiors, a single rank) store straight to global
        // memory and skip the transfer warp: nothing to push, nothing to count
        bool tpush = true;
        if (MODE == 2) {
            const region_dev &Ro = lc.ctx->region[p.region_out];
            const uint64_t a0 = ((uint64_t)T.i0 * N + T.c0) * 4 - Ro.own_off;
            const uint64_t a1 = ((uint64_t)(T.i1 - 1) * N + T.c1) * 4 - Ro.own_off;
            tpush = false;
            for (uint64_t c = a0 / Ro.chunk_bytes; c * Ro.chunk_bytes < a1 && !tpush; ++c)
                tpush = proact::transfers(lc, Ro, (uint32_t)c);
        }
        auto rows = [&](auto fast_tag) {
            constexpr bool FAST = decltype(fast_tag)::value;
            for (int i = T.i0; i < T.i1; ++i) {
                const uint32_t qdn = q;
                const bool has_dn = i + 1 <= T.klast;
                const int orow = (i - T.i0) % JSR;              // MODE 2: row within the span
                float *ostrip = oring + ((oq % JOS) * JSR + orow) * JW;
                if (MODE == 2 && tpush && orow == 0) proact::tp_acquire(tp, oq);
                if (has_dn) {
                    mbar_wait(&full[q % JS], (q / JS) & 1u);
    #pragma unroll
                    for (int g = 0; g < JV; ++g)
                        if (act[g]) dn[g] = lds128(ringf + (q % JS) * SLOT + g * GW);
                    ++q;
                }
    #pragma unroll
                for (int g = 0; g < JV; ++g) {
                const int j = T.c0 + 4 * tid + g * GW;
                const float *cs = ringf + (qcur % JS) * SLOT + g * GW;
                float lft = __shfl_up_sync(0xFFFFFFFFu, cur[g].w, 1);
                float rgt = __shfl_down_sync(0xFFFFFFFFu, cur[g].x, 1);
                if (lane == 0) lft = cs[-1];
                if (lane == 31) rgt = cs[4];
                if (FAST || act[g]) {
                    const float4 c = cur[g], u = up[g], d = dn[g];
                    float4 o;
                    if (!FAST && (i == 0 || i == N - 1)) {
                        o = c;
                    } else {
                        o.x = __fmul_rn(0.25f, __fadd_rn(__fadd_rn(u.x, d.x), __fadd_rn(lft, c.y)));
                        o.y = __fmul_rn(0.25f, __fadd_rn(__fadd_rn(u.y, d.y), __fadd_rn(c.x, c.z)));
                        o.z = __fmul_rn(0.25f, __fadd_rn(__fadd_rn(u.z, d.z), __fadd_rn(c.y, c.w)));
                        o.w = __fmul_rn(0.25f, __fadd_rn(__fadd_rn(u.w, d.w), __fadd_rn(c.z, rgt)));
                        if (!FAST && j == 0) o.x = c.x;
                        if (!FAST && j + 3 == N - 1) o.w = c.w;
                    }
                    const uint64_t off = ((uint64_t)i * N + j) * 4;
                    if (MODE == 2) {   // the local copy now, the span for the transfer warp
                        if (tpush) *reinterpret_cast<float4 *>(ostrip + 4 * tid + g * GW) = o;
                        *reinterpret_cast<float4 *>(outb + off) = o;
                    } else if (!FAST && lc.mech == PROACT_MECH_INLINE) {
                        proact::put(lc, p.region_out, off, o);
                    } else if (!FAST && PROACT_JACOBI_OUT_EVICT_LAST && tally) {
                        // the agent pushes this chunk within microseconds: keep it in L2 for that read
                        asm volatile("st.global.L2::cache_hint.v4.f32 [%0], {%1, %2, %3, %4}, %5;"
                                     ::"l"(outb + off), "f"(o.x), "f"(o.y), "f"(o.z), "f"(o.w), "l"(pol_out) : "memory");
                    } else {
#if PROACT_JACOBI_OUT_STORE == 1
                        // no agent reads this output back (MODE 0): streaming stores (st.cs), ~1 %
                        // faster under the power cap (profiles/r02k_jacobi_store_policy.log); an
                        // agent's read-back (MODE 1) wants the lines kept in L2
                        if (MODE == 0) __stcs(reinterpret_cast<float4 *>(outb + off), o);
                        else *reinterpret_cast<float4 *>(outb + off) = o;
#else
                        *reinterpret_cast<float4 *>(outb + off) = o;
#endif
                    }
                }
                }
                if (MODE == 2 && tpush && (orow == JSR - 1 || i + 1 == T.i1)) {   // hand the span to the transfer warp
                    if (tid == 0)
                        tp->desc[oq % JOS] = proact::tile_desc{((uint64_t)(i - orow) * N + T.c0) * 4,
                                                               (uint32_t)(T.c1 - T.c0) * 4, proact::td_rows(orow + 1)};
                    proact::tp_publish(tp, oq);
                    ++oq;
                }
                __syncwarp();
                if (lane == 0) {
                    mbar_arrive(&empty[qcur % JS]);                    // row i: done
                    if (has_dn && i + 1 == T.i1) mbar_arrive(&empty[qdn % JS]);   // bottom halo row
                }
    #pragma unroll
                for (int g = 0; g < JV; ++g) {
                    up[g] = cur[g];
                    cur[g] = dn[g];
                }
                qcur = qdn;
            }
        };
        if (fast)
            rows(std::true_type{});
        else
            rows(std::false_type{});
        if (MODE == 2) {
            ++kt;
            continue;
        }
        if (tally && TALLY) {   // hand the tile to the committer warp; never run > 2 tiles ahead
            __syncwarp();
            if (lane == 0) mbar_arrive(&tdone[kt & 1u]);
            ++kt;
            if (kt >= 2) mbar_wait(&cdone[kt & 1u], ((kt - 2) >> 1) & 1u);
            continue;
        }
        ++kt;
        if (tally) {   // no committer warp: compute warps meet, warp 0 commits
            asm volatile("bar.sync 1, %0;" ::"r"(JC * 32) : "memory");
            if (warp == 0)
                for (int k0 = T.i0; k0 < T.i1; k0 += 32) {
                    const int i = k0 + lane;
                    warp_commit(lc, p.region_out, i < T.i1, ((uint64_t)i * N + T.c0) * 4,
                                (uint32_t)(T.c1 - T.c0) * 4);
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
constexpr int MBLK = 8;            // tiles per CTA block: one commit per 32 KiB block

// Litmus consumer prologue (proact_litmus_phase): wait for the whole current generation of the
// verify region (flags or credits, as its producing mechanism requires), then check every word
// against phase-1's value; this CTA checks a grid-stride share of the words.
__device__ __forceinline__ void litmus_check(const launch_ctx &lc, const proact_micro_params &p, int nthreads)
{
    if (p.verify_region < 0 || p.phase == 0) return;
    const region_dev &V = lc.ctx->region[p.verify_region];
    if (threadIdx.x == 0) proact::wait_range(lc, p.verify_region, 0, V.total_bytes);
    __syncthreads();
    const uint32_t *w = reinterpret_cast<const uint32_t *>(V.base);
    const uint64_t W = V.total_bytes / 4;
    uint32_t bad = 0;
    for (uint64_t k = (uint64_t)proact::producer_block(lc) * nthreads + threadIdx.x; k < W;
         k += (uint64_t)proact::producer_grid(lc) * nthreads)
        bad += w[k] != micro_value((uint32_t)k, p.phase - 1, p.seed, 1);
    bad = __reduce_add_sync(0xFFFFFFFFu, bad);
    if (bad && (threadIdx.x & 31) == 0 && p.bad) atomicAdd(p.bad, bad);
}

__global__ void __launch_bounds__(MB, 4) micro_kernel(launch_ctx lc, proact_micro_params p)
{
    if (proact::agent_dispatch(lc)) return;
    litmus_check(lc, p, MB);
    const region_dev &R = lc.ctx->region[p.region];
    const uint64_t w_lo = R.own_off / 4, w_hi = (R.own_off + R.own_bytes) / 4;
    const uint64_t ntiles = (w_hi - w_lo + 1023) / 1024;
    const uint64_t nblk = (ntiles + MBLK - 1) / MBLK;
    for (uint64_t bk = proact::producer_block(lc); bk < nblk; bk += proact::producer_grid(lc)) {
        const uint64_t tb0 = bk * MBLK, tb1 = min(tb0 + MBLK, ntiles);
        for (uint64_t t = tb0; t < tb1; ++t) {   // the paper's 4 KiB per source block pass
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
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            const uint64_t a = w_lo + tb0 * 1024, b = min(w_lo + tb1 * 1024, w_hi);
            proact::commit_span(lc, p.region, a * 4, (b - a) * 4);
        }
    }
}

// PROACT_AGENT_PRODUCER variant: 8 compute warps write each 4 KiB tile (L279) into a shared-memory
// ring slot (same values and store-order options); MTS consecutive tiles of the CTA's block form
// one span (contiguous in the region), which the transfer warp bulk-stores to the local replica
// and every destination mirror with one TMA store each, and counts once delivered
// (proact::tile_pusher).  Spans of 4 tiles: the transfer warp's per-span work is amortised over
// 16 KiB instead of 4 KiB.
#ifndef PROACT_MICRO_SPAN_TILES
#define PROACT_MICRO_SPAN_TILES 4
#endif
#ifndef PROACT_MICRO_OUT_RING
#define PROACT_MICRO_OUT_RING 3
#endif
constexpr uint32_t MTS = PROACT_MICRO_SPAN_TILES;   // 4 KiB tiles per pushed span
constexpr uint32_t MOS = PROACT_MICRO_OUT_RING;     // output ring slots (MTS x 4 KiB each)
constexpr size_t MTP_SMEM = (size_t)MOS * MTS * 4096 + sizeof(proact::tile_ring_ctl<MOS>);

__global__ void __launch_bounds__(MB + 32, 4) micro_tp_kernel(launch_ctx lc, proact_micro_params p)
{
    if (proact::agent_dispatch(lc)) return;
    extern __shared__ __align__(128) unsigned char msm[];
    uint32_t *oring = reinterpret_cast<uint32_t *>(msm);
    auto *tp = reinterpret_cast<proact::tile_ring_ctl<MOS> *>(msm + (size_t)MOS * MTS * 4096);
    if (threadIdx.x == 0) proact::tp_init(tp, MB / 32);
    __syncthreads();
    if (threadIdx.x >= MB) {
        proact::tile_pusher<MOS>(lc, p.region, msm, MTS * 4096, tp);
        return;
    }
    if (p.verify_region >= 0 && p.phase > 0) {   // litmus: the producer warps check (named barrier)
        const region_dev &V = lc.ctx->region[p.verify_region];
        if (threadIdx.x == 0) proact::wait_range(lc, p.verify_region, 0, V.total_bytes);
        asm volatile("bar.sync 1, %0;" ::"r"(MB) : "memory");
        const uint32_t *w = reinterpret_cast<const uint32_t *>(V.base);
        const uint64_t W = V.total_bytes / 4;
        uint32_t bad = 0;
        for (uint64_t k = (uint64_t)proact::producer_block(lc) * MB + threadIdx.x; k < W;
             k += (uint64_t)proact::producer_grid(lc) * MB)
            bad += w[k] != micro_value((uint32_t)k, p.phase - 1, p.seed, 1);
        bad = __reduce_add_sync(0xFFFFFFFFu, bad);
        if (bad && (threadIdx.x & 31) == 0 && p.bad) atomicAdd(p.bad, bad);
    }
    const region_dev &R = lc.ctx->region[p.region];
    const uint64_t w_lo = R.own_off / 4, w_hi = (R.own_off + R.own_bytes) / 4;
    const uint64_t ntiles = (w_hi - w_lo + 1023) / 1024;
    const uint64_t nblk = (ntiles + MBLK - 1) / MBLK;
    uint32_t q = 0;
    for (uint64_t bk = proact::producer_block(lc); bk < nblk; bk += proact::producer_grid(lc)) {
        const uint64_t tb0 = bk * MBLK, tb1 = min(tb0 + MBLK, ntiles);
        for (uint64_t t = tb0; t < tb1; ++t) {
            const uint64_t t0 = w_lo + t * 1024, t1 = min(t0 + 1024, w_hi);
            const uint32_t sub = (uint32_t)((t - tb0) % MTS);   // tile within the span
            if (sub == 0) proact::tp_acquire(tp, q);
            uint32_t *slot = oring + ((q % MOS) * MTS + sub) * 1024;
            if (!p.scattered) {
                const uint64_t k = t0 + 4 * threadIdx.x;
                if (k + 4 <= t1) {
                    uint4 v;
                    v.x = micro_value((uint32_t)k, p.phase, p.seed, p.K);
                    v.y = micro_value((uint32_t)k + 1, p.phase, p.seed, p.K);
                    v.z = micro_value((uint32_t)k + 2, p.phase, p.seed, p.K);
                    v.w = micro_value((uint32_t)k + 3, p.phase, p.seed, p.K);
                    *reinterpret_cast<uint4 *>(slot + 4 * threadIdx.x) = v;
                } else {
                    for (uint64_t w = k; w < t1 && w < k + 4; ++w) slot[w - t0] = micro_value((uint32_t)w, p.phase, p.seed, p.K);
                }
            } else {
                for (int s = 0; s < 4; ++s) {
                    const uint32_t jj = threadIdx.x + MB * s;
                    const uint64_t w = t0 + ((jj * 389u) & 1023u);
                    if (w < t1) slot[w - t0] = micro_value((uint32_t)w, p.phase, p.seed, p.K);
                }
            }
            if (sub == MTS - 1 || t + 1 == tb1) {   // hand the span (tiles t - sub .. t) over
                if (threadIdx.x == 0) {
                    const uint64_t s0 = t0 - (uint64_t)sub * 1024;
                    tp->desc[q % MOS] = proact::tile_desc{s0 * 4, (uint32_t)(t1 - s0) * 4, proact::td_rows(1)};
                }
                proact::tp_publish(tp, q);
                ++q;
            }
        }
    }
    proact::tp_acquire(tp, q);
    if (threadIdx.x == 0) tp->desc[q % MOS] = proact::tile_desc{0, 0, proact::TD_END};
    proact::tp_publish(tp, q);
}

// ---------------------------------------------------------------- fault injection (tests)
__global__ void double_commit_kernel(launch_ctx lc, int region)
{
    if (proact::agent_dispatch(lc)) return;
    if (proact::producer_block(lc) == 0 && threadIdx.x == 0) {
        const region_dev &R = lc.ctx->region[region];
        if (R.n_own) {
            const uint32_t b = proact::chunk_len(R, 0);
            proact::commit_chunk(lc, region, 0, b);
            proact::commit_chunk(lc, region, 0, b);   // the second commit over-counts chunk 0
        }
    }
}

// ---------------------------------------------------------------- banded Jacobi (NEXT-2)
constexpr int BB = 256;    // threads
constexpr int BT = 1024;   // rows per tile (4 KiB of output)

__device__ __forceinline__ float ld_stream_f(const float *p)
{
    float v;
    asm volatile("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(v) : "l"(p));
    return v;
}

__global__ void __launch_bounds__(BB) banded_kernel(launch_ctx lc, proact_banded_params p)
{
    if (proact::agent_dispatch(lc)) return;
    extern __shared__ float xs[];   // x window [i0 - w, i1 + w) of the tile
    const float *x = reinterpret_cast<const float *>(lc.ctx->region[p.region_in].base);
    const int64_t N = p.N, w = p.w, rend = p.row0 + p.nrows;
    const int64_t ntiles = (p.nrows + BT - 1) / BT;
    for (int64_t t = proact::producer_block(lc); t < ntiles; t += proact::producer_grid(lc)) {
        const int64_t i0 = p.row0 + t * BT, i1 = min(i0 + (int64_t)BT, rend);
        const int64_t lo = i0 - w > 0 ? i0 - w : 0, hi = i1 + w < N ? i1 + w : N;
        if (threadIdx.x == 0)   // (a7) peers' rows of the previous generation within the band
            proact::wait_range(lc, p.region_in, (uint64_t)lo * 4, (uint64_t)(hi - lo) * 4);
        __syncthreads();
        for (int64_t k = threadIdx.x; k < hi - lo; k += BB) xs[k] = __ldcg(x + lo + k);
        __syncthreads();
        // BR rows per thread (coalesced across the CTA); the diagonals are walked in groups of
        // BU whose loads are all issued before the group's adds, so BR x BU streaming loads are
        // in flight per thread while each row still sums o = -w..w in order (reading R19)
        constexpr int BR = BT / BB, BU = 8;
        float sum[BR];
#pragma unroll
        for (int r = 0; r < BR; ++r) sum[r] = 0.0f;
        for (int64_t ob = -w; ob <= w; ob += BU) {
            float av[BU][BR];
#pragma unroll
            for (int u = 0; u < BU; ++u)
#pragma unroll
                for (int r = 0; r < BR; ++r) {
                    const int64_t o = ob + u, i = i0 + threadIdx.x + r * BB, j = i + o;
                    av[u][r] = (o <= w && o != 0 && i < i1 && j >= 0 && j < N) ? ld_stream_f(p.a + (o + w) * N + i)
                                                                                 : 0.0f;
                }
#pragma unroll
            for (int u = 0; u < BU; ++u)
#pragma unroll
                for (int r = 0; r < BR; ++r) {
                    const int64_t o = ob + u, i = i0 + threadIdx.x + r * BB, j = i + o;
                    if (o <= w && o != 0 && i < i1 && j >= 0 && j < N)
                        sum[r] = __fadd_rn(sum[r], __fmul_rn(av[u][r], xs[j - lo]));
                }
        }
#pragma unroll
        for (int r = 0; r < BR; ++r) {
            const int64_t i = i0 + threadIdx.x + r * BB;
            if (i < i1) {
                const float v = __fdiv_rn(__fsub_rn(p.b[i], sum[r]), p.a[w * N + i]);
                proact::put(lc, p.region_out, (uint64_t)i * 4, v);
            }
        }
        __syncthreads();
        if (threadIdx.x == 0) proact::commit_span(lc, p.region_out, (uint64_t)i0 * 4, (uint64_t)(i1 - i0) * 4);
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
    // > 48 KiB of dynamic shared memory needs the opt-in, per device (set once per device)
    if (proact_internal_smem_attr((const void *)jacobi_kernel<0>, JCfg<0>::smem) ||
        proact_internal_smem_attr((const void *)jacobi_kernel<1>, JCfg<1>::smem) ||
        proact_internal_smem_attr((const void *)jacobi_kernel<2>, JCfg<2>::smem))
        return PROACT_ERR_CUDA;
    switch (proact_launch_mode()) {
    case 2:
        return proact_launch_ex(regs, 1, (const void *)jacobi_kernel<2>, 0, JCfg<2>::threads, args, JCfg<2>::smem,
                                stream, PROACT_LAUNCH_TILE_PUSH);
    case 1:
        return proact_launch(regs, 1, (const void *)jacobi_kernel<1>, 0, JCfg<1>::threads, args, JCfg<1>::smem, stream);
    default:
        return proact_launch(regs, 1, (const void *)jacobi_kernel<0>, 0, JCfg<0>::threads, args, JCfg<0>::smem, stream);
    }
}

static int micro_launch(proact_micro_params &p, void *stream)
{
    launch_ctx lc;
    void *args[2] = {&lc, &p};
    int regs[1] = {p.region};
    if (proact_launch_mode() == 2) {
        if (proact_internal_smem_attr((const void *)micro_tp_kernel, MTP_SMEM)) return PROACT_ERR_CUDA;
        return proact_launch_ex(regs, 1, (const void *)micro_tp_kernel, 0, MB + 32, args, MTP_SMEM, stream,
                                PROACT_LAUNCH_TILE_PUSH);
    }
    return proact_launch(regs, 1, (const void *)micro_kernel, 0, MB, args, 0, stream);
}

int proact_litmus_phase(int region_in, int region_out, unsigned phase, unsigned seed, unsigned *d_bad, void *stream)
{
    proact_region_info ri, ro;
    int rc = proact_region_info_get(region_in, &ri);
    if (rc) return rc;
    if ((rc = proact_region_info_get(region_out, &ro))) return rc;
    if (region_in == region_out || ri.total_bytes != ro.total_bytes || ri.own_offset != ro.own_offset)
        return PROACT_ERR_INVALID;
    proact_micro_params p;
    p.region = region_out;
    p.phase = phase;
    p.seed = seed;
    p.K = 1;
    p.scattered = 0;
    p.verify_region = region_in;
    p.bad = d_bad;
    return micro_launch(p, stream);
}

int proact_inject_double_commit(int region, void *stream)
{
    launch_ctx lc;
    int r = region;
    void *args[2] = {&lc, &r};
    int regs[1] = {region};
    return proact_launch(regs, 1, (const void *)double_commit_kernel, 1, 64, args, 0, stream);
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
    p.verify_region = -1;
    p.bad = nullptr;
    return micro_launch(p, stream);
}

}  // extern "C"

// ---- banded Jacobi, TMA-fed (default when N % 4 == 0 and w <= BW_MAX): the first kernel was
// latency bound (one CTA iteration = 7 serialised global round trips; 2.0 TB/s).  Here one
// producer warp streams, per BT2-row tile, the x window + b + diagonal slices (tile slots, double
// buffered) and then the tile's off-diagonals in groups of BDG through a BNS-deep shared-memory
// ring (cp.async.bulk, 8 KiB per diagonal slice, contiguous in the DIA layout); eight compute
// warps sum each row over o = -w..w (o != 0) in order from shared memory (reading R19).
namespace {
// measured at N = 2^24, w = 16 (tools/bench_workloads.py --workload banded, one variant per
// build): 2048 rows x 2 diagonals x 4 stages, 2 CTAs/SM: 0.414 ms (0.89 of HBM); 512 x 8 x 6:
// 0.634 ms; 1024 x 4 x 5: 0.482 ms; 4096 x 1 x 3 (1 CTA/SM): 0.617 ms -- 8 KiB bulk copies beat
// 2 KiB ones (TMA issue cost), two CTAs per SM beat one (latency hiding)
#ifndef PROACT_BANDED_BT
#define PROACT_BANDED_BT 2048
#endif
#ifndef PROACT_BANDED_DG
#define PROACT_BANDED_DG 2
#endif
#ifndef PROACT_BANDED_RING
#define PROACT_BANDED_RING 4
#endif
#ifndef PROACT_BANDED_MINB
#define PROACT_BANDED_MINB 2
#endif
constexpr int BT2 = PROACT_BANDED_BT;    // rows per tile
constexpr int BCW = 8;                   // compute warps
constexpr int BRT = BT2 / (BCW * 32);    // rows per compute thread
constexpr int BDG = PROACT_BANDED_DG;    // diagonals per ring stage
constexpr int BNS = PROACT_BANDED_RING;  // ring stages
constexpr int BW_MAX = 4096;             // larger bands use banded_kernel

__host__ __device__ __forceinline__ int banded_xw(long long w) { return (int)((BT2 + 2 * w + 8 + 3) & ~3LL); }
__host__ __device__ __forceinline__ size_t banded_smem(long long w)
{
    return (size_t)BNS * BDG * BT2 * 4 + 2 * ((size_t)banded_xw(w) + 2 * BT2) * 4 + (2 * BNS + 4) * 8 + 16;
}
// i-th off-diagonal of the band in the summation order o = -w..-1, 1..w
__device__ __forceinline__ int64_t band_o(int64_t idx, int64_t w) { return idx < w ? idx - w : idx - w + 1; }

__device__ __noinline__ void banded_stream(const launch_ctx &lc, const proact_banded_params &p, float *ring,
                                           float *slots, int xw, uint64_t *full, uint64_t *empty, uint64_t *tfull,
                                           uint64_t *tempty, int *tids, int64_t ntiles)
{
    const int64_t N = p.N, w = p.w, rend = p.row0 + p.nrows, ngroups = (2 * w + BDG - 1) / BDG;
    const float *x = reinterpret_cast<const float *>(lc.ctx->region[p.region_in].base);
    uint32_t q = 0;
    for (uint32_t kt = 0;; ++kt) {
        const uint32_t t = proact::claim_tile(lc, (uint32_t)ntiles);
        const uint32_t slot = kt & 1u;
        if (kt >= 2) mbar_wait(&tempty[slot], ((kt >> 1) - 1) & 1u);
        if (t >= (uint32_t)ntiles) {
            tids[slot] = -1;
            mbar_arrive(&tfull[slot]);
            return;
        }
        tids[slot] = (int)t;
        const int64_t i0 = p.row0 + (int64_t)t * BT2, i1 = min(i0 + (int64_t)BT2, rend), nr = i1 - i0;
        const int64_t lo = i0 - w > 0 ? i0 - w : 0, hi = i1 + w < N ? i1 + w : N;
        const int64_t lo4 = lo & ~(int64_t)3, hi4 = min(N, (int64_t)((hi + 3) & ~(int64_t)3));
        // (a7) peers' rows of the previous generation within the band, then generic -> async proxy
        proact::wait_range(lc, p.region_in, (uint64_t)lo * 4, (uint64_t)(hi - lo) * 4);
        asm volatile("fence.proxy.async;" ::: "memory");
        float *xs = slots + slot * (xw + 2 * BT2);
        mbar_expect_tx(&tfull[slot], (uint32_t)((hi4 - lo4) + 2 * nr) * 4);
        bulk_g2s(xs, x + lo4, (uint32_t)(hi4 - lo4) * 4, &tfull[slot]);
        bulk_g2s(xs + xw, p.b + i0, (uint32_t)nr * 4, &tfull[slot]);
        bulk_g2s(xs + xw + BT2, p.a + w * N + i0, (uint32_t)nr * 4, &tfull[slot]);
        for (int64_t g = 0; g < ngroups; ++g, ++q) {
            const uint32_t st = q % BNS;
            if (q >= BNS) mbar_wait(&empty[st], ((q / BNS) - 1) & 1u);
            const int64_t nd = min((int64_t)BDG, 2 * w - g * BDG);
            mbar_expect_tx(&full[st], (uint32_t)(nd * nr) * 4);
            for (int64_t k = 0; k < nd; ++k) {
                const int64_t o = band_o(g * BDG + k, w);
                bulk_g2s(ring + ((size_t)st * BDG + k) * BT2, p.a + (o + w) * N + i0, (uint32_t)nr * 4, &full[st]);
            }
        }
    }
}
}  // namespace

__global__ void __launch_bounds__((BCW + 1) * 32, PROACT_BANDED_MINB) banded_tma_kernel(launch_ctx lc, proact_banded_params p)
{
    if (proact::agent_dispatch(lc)) return;
    extern __shared__ __align__(128) unsigned char bsm[];
    const int64_t N = p.N, w = p.w, rend = p.row0 + p.nrows, ngroups = (2 * w + BDG - 1) / BDG;
    const int xw = banded_xw(w);
    float *ring = reinterpret_cast<float *>(bsm);
    float *slots = ring + (size_t)BNS * BDG * BT2;
    uint64_t *full = reinterpret_cast<uint64_t *>(slots + 2 * (xw + 2 * BT2));
    uint64_t *empty = full + BNS, *tfull = empty + BNS, *tempty = tfull + 2;
    int *tids = reinterpret_cast<int *>(tempty + 2);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int64_t ntiles = (p.nrows + BT2 - 1) / BT2;
    if (tid == 0) {
        for (int s = 0; s < BNS; ++s) {
            mbar_init(&full[s], 1);
            mbar_init(&empty[s], BCW);
        }
        for (int s = 0; s < 2; ++s) {
            mbar_init(&tfull[s], 1);
            mbar_init(&tempty[s], BCW);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    if (warp == BCW) {
        if (lane == 0) banded_stream(lc, p, ring, slots, xw, full, empty, tfull, tempty, tids, ntiles);
        return;
    }
    uint32_t q = 0;
    for (uint32_t kt = 0;; ++kt) {
        const uint32_t slot = kt & 1u;
        mbar_wait(&tfull[slot], (kt >> 1) & 1u);
        const int t = tids[slot];
        if (t < 0) break;
        const int64_t i0 = p.row0 + (int64_t)t * BT2, i1 = min(i0 + (int64_t)BT2, rend), nr = i1 - i0;
        const int64_t lo = i0 - w > 0 ? i0 - w : 0, lo4 = lo & ~(int64_t)3;
        const float *xs = slots + slot * (xw + 2 * BT2);
        const bool clean = nr == BT2 && i0 - w >= 0 && i1 + w <= N;
        float sum[BRT];
#pragma unroll
        for (int r = 0; r < BRT; ++r) sum[r] = 0.0f;
        for (int64_t g = 0; g < ngroups; ++g, ++q) {
            const uint32_t st = q % BNS;
            mbar_wait(&full[st], (q / BNS) & 1u);
            const float *sa = ring + (size_t)st * BDG * BT2;
            const int64_t nd = min((int64_t)BDG, 2 * w - g * BDG);
            if (clean) {   // full tile, band inside [0, N): no per-element bounds tests
                for (int k = 0; k < (int)nd; ++k) {
                    const int o = (int)band_o(g * BDG + k, w);
                    const float *ao = sa + k * BT2 + tid;
                    const float *xo = xs + (int)(i0 - lo4) + o + tid;
#pragma unroll
                    for (int r = 0; r < BRT; ++r)
                        sum[r] = __fadd_rn(sum[r], __fmul_rn(ao[r * (BCW * 32)], xo[r * (BCW * 32)]));
                }
            } else {
                for (int64_t k = 0; k < nd; ++k) {
                    const int64_t o = band_o(g * BDG + k, w);
#pragma unroll
                    for (int r = 0; r < BRT; ++r) {
                        const int64_t ii = tid + r * (BCW * 32), i = i0 + ii, j = i + o;
                        if (ii < nr && j >= 0 && j < N)
                            sum[r] = __fadd_rn(sum[r], __fmul_rn(sa[k * BT2 + ii], xs[j - lo4]));
                    }
                }
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&empty[st]);
        }
#pragma unroll
        for (int r = 0; r < BRT; ++r) {
            const int64_t ii = tid + r * (BCW * 32);
            if (ii < nr) {
                const float v = __fdiv_rn(__fsub_rn(xs[xw + ii], sum[r]), xs[xw + BT2 + ii]);
                proact::put(lc, p.region_out, (uint64_t)(i0 + ii) * 4, v);
            }
        }
        asm volatile("bar.sync 1, %0;" ::"r"(BCW * 32) : "memory");   // the compute warps' stores
        if (tid == 0) proact::commit_span(lc, p.region_out, (uint64_t)i0 * 4, (uint64_t)nr * 4);
        __syncwarp();
        if (lane == 0) mbar_arrive(&tempty[slot]);
    }
}

extern "C" int proact_banded_phase(int region_in, int region_out, const float *a, const float *b, long long N,
                                   long long w, void *stream)
{
    proact_region_info ri, ro;
    int rc = proact_region_info_get(region_in, &ri);
    if (rc) return rc;
    rc = proact_region_info_get(region_out, &ro);
    if (rc) return rc;
    if (!a || !b || N < 1 || w < 0 || w > 8192 || region_in == region_out) return PROACT_ERR_INVALID;
    if (ri.own_offset != ro.own_offset || ri.own_bytes != ro.own_bytes || ri.total_bytes != 4ull * N ||
        ro.total_bytes != 4ull * N)
        return PROACT_ERR_INVALID;
    proact_banded_params p;
    p.region_in = region_in;
    p.region_out = region_out;
    p.N = N;
    p.w = w;
    p.row0 = (long long)(ro.own_offset / 4);
    p.nrows = (long long)(ro.own_bytes / 4);
    p.a = a;
    p.b = b;
    launch_ctx lc;
    void *args[2] = {&lc, &p};
    int regs[1] = {region_out};
    static const int tma_off = [] {
        const char *e = getenv("PROACT_BANDED_PLAIN");
        return e && atoi(e) ? 1 : 0;
    }();
    if (!tma_off && N % 4 == 0 && w <= BW_MAX && (uintptr_t)a % 16 == 0 && (uintptr_t)b % 16 == 0) {
        const size_t tsmem = banded_smem(w);
        if (proact_internal_smem_attr((const void *)banded_tma_kernel, tsmem)) return PROACT_ERR_CUDA;
        return proact_launch(regs, 1, (const void *)banded_tma_kernel, 0, (BCW + 1) * 32, args, tsmem, stream);
    }
    const size_t smem = (size_t)(BT + 2 * w) * 4;
    if (proact_internal_smem_attr((const void *)banded_kernel, smem)) return PROACT_ERR_CUDA;
    return proact_launch(regs, 1, (const void *)banded_kernel, 0, BB, args, smem, stream);
}

// ================================================================ host-buffer Jacobi (e2e)
// The host-solve entry points keep library-owned device buffers (registered regions) between
// calls.  They belong to the calling thread's rank context: proact_finalize runs the hook below,
// which frees them, so a later proact_init on the same thread starts clean (regions cannot be
// unregistered individually, so the state must never outlive the context that registered it).
extern "C" __attribute__((visibility("hidden"))) void proact_internal_on_finalize(void (*fn)(void));
namespace {
struct JacobiHost {
    long long N = 0;
    size_t chunk = 0;
    float *a = nullptr, *b = nullptr;
    int ra = -1, rb = -1;
};
thread_local JacobiHost jh;

void jh_release()
{
    cudaFree(jh.a);
    cudaFree(jh.b);
    jh = JacobiHost();
}

// rows of the input a rank reads before any peer pushes into its replica: its own rows and the
// two halo rows (iteration 0 reads generation 0, identical on every rank, reading R16); every
// other row of the replica is overwritten by the peers' pushes before it is read
inline void input_rows(long long N, long long r0, long long r1, long long *lo, long long *hi)
{
    *lo = r0 > 0 ? r0 - 1 : 0;
    *hi = r1 < N ? r1 + 1 : N;
}
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
        // replicas are initialised before registration (as workloads.Jacobi does): once the
        // collective returns, peers may push into them.  Registering never-written allocations
        // produced wrong halo rows in ~10 % of G = 2 loopback solves
        // (tools/probes/jacobi_race.py: 16/40 -> 0/30 with the buffers written first)
        if (cudaMemset(jh.a, 0, rowb * N) != cudaSuccess || cudaMemset(jh.b, 0, rowb * N) != cudaSuccess ||
            cudaDeviceSynchronize() != cudaSuccess)
            return PROACT_ERR_CUDA;
        const uint64_t all = G >= 64 ? ~0ull : ((1ull << G) - 1);
        jh.ra = proact_register_region((char *)jh.a + r0 * rowb, (r1 - r0) * rowb, chunk_bytes, all);
        if (jh.ra < 0) return jh.ra;
        jh.rb = proact_register_region((char *)jh.b + r0 * rowb, (r1 - r0) * rowb, chunk_bytes, all);
        if (jh.rb < 0) return jh.rb;
        jh.N = N;
        jh.chunk = chunk_bytes;
        proact_internal_on_finalize(jh_release);
    } else if (jh.chunk != chunk_bytes) {
        int rc = proact_region_rechunk(jh.ra, chunk_bytes);
        if (rc) return rc;
        rc = proact_region_rechunk(jh.rb, chunk_bytes);
        if (rc) return rc;
        jh.chunk = chunk_bytes;
    }
    long long lo, hi;
    input_rows(N, r0, r1, &lo, &hi);
    // Both replicas are rewritten on the solve's stream before its input lands.  KNOWN ISSUE
    // (DESIGN.md Sec. 12): without this, ~10-35 % of G = 2 loopback solves of this entry point got
    // wrong halo rows (tools/probes/jacobi_race.py); with it, 0 of 90; the root cause is not yet
    // identified (initialising the buffers before registration alone does not help).
    if (cudaMemsetAsync(jh.a, 0, rowb * N, s) != cudaSuccess || cudaMemsetAsync(jh.b, 0, rowb * N, s) != cudaSuccess)
        return PROACT_ERR_CUDA;
    if (cudaMemcpyAsync(jh.a + lo * N, h_x0 + lo * N, (hi - lo) * rowb, cudaMemcpyHostToDevice, s) != cudaSuccess)
        return PROACT_ERR_CUDA;
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
    if (bytes_h2d) *bytes_h2d = (unsigned long long)((hi - lo) * rowb);
    if (bytes_d2h) *bytes_d2h = (unsigned long long)((r1 - r0) * rowb);
    return PROACT_OK;
}

// Pipelined host-buffer solves: nsolve independent solves, each with its own H2D of the input
// and D2H of its result, over two device buffer sets so that solve k's phases overlap the H2D of
// solve k+1 and the D2H of solve k-1 (PCIe is full duplex; both copies run on the copy engines
// while the SMs compute).  Streams: `stream` computes, two library streams copy.
namespace {
struct JacobiPipe {
    long long N = 0;
    size_t chunk = 0;
    float *buf[2][2] = {{nullptr, nullptr}, {nullptr, nullptr}};
    int rid[2][2] = {{-1, -1}, {-1, -1}};
    cudaStream_t h2d = nullptr, d2h = nullptr;
    cudaEvent_t ev_in[2] = {nullptr, nullptr}, ev_done[2] = {nullptr, nullptr}, ev_out[2] = {nullptr, nullptr};
    float *stage = nullptr;                 // H2D landing buffer (not a region)
    cudaEvent_t ev_staged = nullptr, ev_stage_free = nullptr;
};
thread_local JacobiPipe jp;

void jp_release()
{
    for (auto &b : jp.buf)
        for (float *f : b) cudaFree(f);
    cudaFree(jp.stage);
    if (jp.h2d) cudaStreamDestroy(jp.h2d);
    if (jp.d2h) cudaStreamDestroy(jp.d2h);
    for (int b = 0; b < 2; ++b)
        for (cudaEvent_t e : {jp.ev_in[b], jp.ev_done[b], jp.ev_out[b]})
            if (e) cudaEventDestroy(e);
    if (jp.ev_staged) cudaEventDestroy(jp.ev_staged);
    if (jp.ev_stage_free) cudaEventDestroy(jp.ev_stage_free);
    jp = JacobiPipe();
}
}  // namespace

extern "C" int proact_jacobi_solve_host_pipelined(const float *h_x0, float *const *h_outs, int nsolve,
                                                  long long N, int iters, size_t chunk_bytes, int rows_per_tile,
                                                  void *stream, unsigned long long *bytes_h2d,
                                                  unsigned long long *bytes_d2h)
{
    const int G = proact_world(), g = proact_rank();
    if (G <= 0) return PROACT_ERR_STATE;
    if (!h_x0 || !h_outs || nsolve < 1 || N < 4 || N % 4 || iters < 0) return PROACT_ERR_INVALID;
    for (int k = 0; k < nsolve; ++k)
        if (!h_outs[k]) return PROACT_ERR_INVALID;
    const long long r0 = N * g / G, r1 = N * (g + 1) / G;
    const size_t rowb = (size_t)N * 4;
    long long lo, hi;
    input_rows(N, r0, r1, &lo, &hi);
    const size_t in_bytes = (size_t)(hi - lo) * rowb;
    cudaStream_t s = (cudaStream_t)stream;
    if (jp.N && jp.N != N) return PROACT_ERR_STATE;   // regions cannot be unregistered
    if (!jp.N) {
        jp.N = N;   // from here on the finalize hook owns whatever was allocated
        proact_internal_on_finalize(jp_release);
        const uint64_t all = G >= 64 ? ~0ull : ((1ull << G) - 1);
        for (int b = 0; b < 2; ++b)
            for (int h = 0; h < 2; ++h) {
                if (cudaMalloc((void **)&jp.buf[b][h], rowb * N) != cudaSuccess) return PROACT_ERR_NOMEM;
                if (cudaMemset(jp.buf[b][h], 0, rowb * N) != cudaSuccess || cudaDeviceSynchronize() != cudaSuccess)
                    return PROACT_ERR_CUDA;   // initialised before registration (see proact_jacobi_solve_host)
                jp.rid[b][h] = proact_register_region((char *)jp.buf[b][h] + r0 * rowb, (r1 - r0) * rowb,
                                                      chunk_bytes, all);
                if (jp.rid[b][h] < 0) return jp.rid[b][h];
            }
        if (cudaStreamCreateWithFlags(&jp.h2d, cudaStreamNonBlocking) != cudaSuccess ||
            cudaStreamCreateWithFlags(&jp.d2h, cudaStreamNonBlocking) != cudaSuccess)
            return PROACT_ERR_CUDA;
        for (int b = 0; b < 2; ++b)
            if (cudaEventCreateWithFlags(&jp.ev_in[b], cudaEventDisableTiming) != cudaSuccess ||
                cudaEventCreateWithFlags(&jp.ev_done[b], cudaEventDisableTiming) != cudaSuccess ||
                cudaEventCreateWithFlags(&jp.ev_out[b], cudaEventDisableTiming) != cudaSuccess)
                return PROACT_ERR_CUDA;
        if (cudaMalloc((void **)&jp.stage, rowb * N) != cudaSuccess) return PROACT_ERR_NOMEM;
        if (cudaEventCreateWithFlags(&jp.ev_staged, cudaEventDisableTiming) != cudaSuccess ||
            cudaEventCreateWithFlags(&jp.ev_stage_free, cudaEventDisableTiming) != cudaSuccess)
            return PROACT_ERR_CUDA;
        jp.chunk = chunk_bytes;
    } else if (jp.chunk != chunk_bytes) {
        for (int b = 0; b < 2; ++b)
            for (int h = 0; h < 2; ++h) {
                int rc = proact_region_rechunk(jp.rid[b][h], chunk_bytes);
                if (rc) return rc;
            }
        jp.chunk = chunk_bytes;
    }
    // the copy streams start after everything already on `stream`
    if (cudaEventRecord(jp.ev_out[0], s) != cudaSuccess || cudaEventRecord(jp.ev_out[1], s) != cudaSuccess ||
        cudaEventRecord(jp.ev_stage_free, s) != cudaSuccess)
        return PROACT_ERR_CUDA;
    // H2D of solve k lands in the staging buffer (it waits only for the previous solve's device
    // copy out of it), so it never queues behind the D2H of solve k - 2 that reads set k & 1:
    // H2D and D2H run at the same time on the full-duplex link, both under the phases.  Only the
    // rows this rank reads before the peers' first pushes travel (input_rows).
    auto h2d = [&]() -> int {
        if (cudaStreamWaitEvent(jp.h2d, jp.ev_stage_free, 0) != cudaSuccess) return PROACT_ERR_CUDA;
        if (cudaMemcpyAsync(jp.stage + lo * N, h_x0 + lo * N, in_bytes, cudaMemcpyHostToDevice, jp.h2d) != cudaSuccess)
            return PROACT_ERR_CUDA;
        return cudaEventRecord(jp.ev_staged, jp.h2d) == cudaSuccess ? PROACT_OK : PROACT_ERR_CUDA;
    };
    int rc = h2d();
    if (rc) return rc;
    for (int k = 0; k < nsolve; ++k) {
        const int b = k & 1;
        // set b is free once solve k - 2's D2H read it; the input moves in by a device copy
        if (cudaStreamWaitEvent(s, jp.ev_staged, 0) != cudaSuccess ||
            cudaStreamWaitEvent(s, jp.ev_out[b], 0) != cudaSuccess ||
            cudaMemcpyAsync(jp.buf[b][0] + lo * N, jp.stage + lo * N, in_bytes, cudaMemcpyDeviceToDevice, s) !=
                cudaSuccess ||
            cudaEventRecord(jp.ev_stage_free, s) != cudaSuccess)
            return PROACT_ERR_CUDA;
        if (k + 1 < nsolve && (rc = h2d())) return rc;   // overlaps this solve's phases
        for (int it = 0; it < iters; ++it) {
            const int in = jp.rid[b][it & 1], out = jp.rid[b][(it & 1) ^ 1];
            if ((rc = proact_jacobi_phase(in, out, N, rows_per_tile, stream))) return rc;
            if ((rc = proact_phase_sync(stream, it == iters - 1 ? PROACT_SYNC_BARRIER : PROACT_SYNC_SIGNAL)))
                return rc;
        }
        if (cudaEventRecord(jp.ev_done[b], s) != cudaSuccess) return PROACT_ERR_CUDA;
        if (cudaStreamWaitEvent(jp.d2h, jp.ev_done[b], 0) != cudaSuccess) return PROACT_ERR_CUDA;
        const float *res = jp.buf[b][iters & 1];
        if (cudaMemcpyAsync(h_outs[k] + r0 * N, res + r0 * N, (r1 - r0) * rowb, cudaMemcpyDeviceToHost, jp.d2h) !=
            cudaSuccess)
            return PROACT_ERR_CUDA;
        // the next solve of set b (k + 2) overwrites these buffers only after its H2D, which waits
        // for this event: no wait on `stream` here, so solve k + 1 computes during this D2H
        if (cudaEventRecord(jp.ev_out[b], jp.d2h) != cudaSuccess) return PROACT_ERR_CUDA;
    }
    // completion on `stream`: the last D2H
    for (int b = 0; b < 2; ++b)
        if (cudaStreamWaitEvent(s, jp.ev_out[b], 0) != cudaSuccess) return PROACT_ERR_CUDA;
    if (bytes_h2d) *bytes_h2d = (unsigned long long)in_bytes;
    if (bytes_d2h) *bytes_d2h = (unsigned long long)((r1 - r0) * rowb);
    return PROACT_OK;
}

extern "C" {
// Force-load this translation unit's kernels (called by proact_init).  Under CUDA's lazy module
// loading the first launch of a kernel loads it, and a load waits for the device's running
// kernels -- with loopback ranks one of those can be a spin waiting for this very thread's next
// launch (observed: smoke deadlocks until the watchdog).  Loading up front removes the hazard.
__attribute__((visibility("hidden"))) int proact_internal_preload_workloads(void)
{
    cudaFuncAttributes a;
    const void *k[] = {(const void *)jacobi_kernel<0>, (const void *)jacobi_kernel<1>, (const void *)jacobi_kernel<2>,
                       (const void *)micro_kernel, (const void *)micro_tp_kernel, (const void *)double_commit_kernel,
                       (const void *)banded_kernel,
                       (const void *)banded_tma_kernel};
    for (const void *f : k)
        if (cudaFuncGetAttributes(&a, f) != cudaSuccess) return PROACT_ERR_CUDA;
    return PROACT_OK;
}

}  // extern "C"
