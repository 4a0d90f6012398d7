/*
 * proact_device.cuh -- device side of libproact (sm_100a).
 *
 * What a producer kernel uses instead of the paper's compiler pass (Sec. IV-A,
 * L172-L176, Listing 1 user_kernel_decoupled L198-L219):
 *
 *   __global__ void k(proact::launch_ctx lc, Params p) {
 *       if (proact::agent_dispatch(lc)) return;            // agent CTAs run the transfer loop
 *       for (tile = proact::producer_block(lc); tile < ntiles; tile += proact::producer_grid(lc)) {
 *           ... proact::wait_range(lc, in_region, off, bytes) ...  // consumer wait (a7), 1 thread
 *           ... proact::put(lc, out_region, byte_off, value) ...   // instrumented store (a2)
 *           __syncthreads();
 *           if (threadIdx.x == 0) proact::commit_span(lc, out_region, tile_off, tile_bytes); // a3
 *       }
 *   }
 *
 * Host side: proact_launch() fills `lc` (include/proact.h).
 *
 * Memory-model protocol (PTX ISA memory consistency model; DESIGN.md Sec. "Ordering"):
 *   producer  weak stores -> bar.sync -> atom.add.release.gpu(counter[c], bytes)         (a2, a3)
 *   agent     ld.acquire.gpu(counter[c]) == expected[c] -> __syncwarp -> ld.global.cg data
 *             -> st.global.v4 to every peer mirror -> __syncwarp -> fence.acq_rel.sys
 *             -> st.relaxed.sys arrive_peer[gchunk] = gen<<1|changed                    (a4-a6)
 *   consumer  ld.acquire.sys(arrive[gchunk]) >= gen -> bar.sync -> plain loads          (a7)
 *   credits   kernel end -> sync kernel: fence.acq_rel.sys -> st peer_done[me] = e+1;
 *             agents wait ld.acquire.sys(done[p]) >= e before overwriting p's replica   (a8)
 * The paper's counters count writer CTAs down to zero (L127-L129); here they count BYTES up to
 * expected[c] (reading R1), which needs no block-to-chunk mapping table (Listing 1)
 * and detects over-counting.  The last arriver is decided from the atomic's return value, never
 * by re-reading (Listing 1 L207-L208 re-reads counter[chunk], a race; reading R2).
 */
#ifndef PROACT_DEVICE_CUH
#define PROACT_DEVICE_CUH

#include <stdint.h>
#include "proact.h"

namespace proact {

/* ---------------------------------------------------------------- shared layouts ----------- */
/* These structs are written by the host runtime (csrc/runtime.cpp) into device memory. */

struct region_dev {
    char *base;                 /* local full-extent replica */
    uint64_t own_off;           /* my slice [own_off, own_off + own_bytes) */
    uint64_t own_bytes;
    uint64_t total_bytes;
    uint32_t chunk_bytes;
    uint32_t n_own;             /* my chunks */
    uint32_t chunk0;            /* global id of my first chunk */
    uint32_t n_total;           /* global chunks */
    uint32_t n_in;              /* chunks pushed INTO me per generation (wait_all); ~0u = n/a */
    uint32_t flags;             /* PROACT_REGION_* */
    uint64_t dest_mask;         /* default destinations of my chunks */
    uint32_t *counter;          /* [n_own] bytes committed this generation (a3) */
    uint32_t *expected;         /* [n_own] bytes of each chunk */
    uint32_t *piecedone;        /* [n_own] agent pieces finished this generation */
    uint32_t *changed_gen;      /* [n_own] generation in which the chunk's data changed */
    uint32_t *push_gen;         /* [n_own] generation in which the chunk must be pushed (SPARSE) */
    uint32_t *chunk_dest;       /* [n_own] per-chunk destination override, or nullptr */
    uint32_t *arrive;           /* [n_total] consumer-side flags: gen << 1 | changed */
    uint32_t *arrive_count;     /* monotonic count of chunks that arrived from peers */
    uint32_t *deliv;            /* debug: [n_own * world] deliveries, or nullptr */
    unsigned long long *queue;  /* [qcap] ready units (gen << 32 | unit), QUEUE discovery */
    uint32_t *qctl;             /* [8]: tail[2], head[2] by generation parity, agents_done */
    uint32_t qcap;              /* queue capacity in units */
    uint32_t dma_group;         /* MECH_DMA: chunks per copy-engine transfer group (>= 1) */
    uint32_t *group_cnt;        /* MECH_DMA: [n_own / dma_group] chunks completed in the group */
    uint64_t rank_off[PROACT_MAX_RANKS + 1];
    uint32_t rank_chunk0[PROACT_MAX_RANKS + 1];
    char *peer_base[PROACT_MAX_RANKS];            /* peers' replica bases (mapped) */
    uint32_t *peer_arrive[PROACT_MAX_RANKS];      /* peers' arrive[] */
    char *mc_base;                                /* multicast address of the replica base, or null */
    uint32_t *peer_arrive_count[PROACT_MAX_RANKS];
};

struct dev_ctx {
    int32_t rank;
    int32_t world;
    uint64_t watchdog_ns;
    uint32_t *done;                            /* [world] credits from peers: (epoch+1)<<1|vote */
    uint32_t *peer_done[PROACT_MAX_RANKS];     /* peers' done[] */
    uint32_t *err;                             /* device error word (atomics) */
    uint32_t *err_host;                        /* host-mapped mirror (plain stores) */
    uint32_t *vote;                            /* [2] local vote words, by epoch parity */
    uint32_t *vote_host;                       /* host-mapped: (epoch+1)<<1 | global vote */
    unsigned long long *prof;                  /* PROACT_DEBUG=2: agent cycle accounting [8] */
    uint32_t *resident;                        /* SEPARATE agent: CTAs that became resident
                                                  (monotonic; the producer launch waits on it) */
    uint32_t *sched;                           /* [2] producer work counter + finished claimers:
                                                  dynamic tile scheduling (see claim_tile) */
    uint32_t *started;                         /* epoch + 1 once the producer grid of that epoch
                                                  started (SEPARATE agent start-up deadline) */
    region_dev region[PROACT_MAX_REGIONS];
};

/* Passed BY VALUE as the first kernel parameter; filled by proact_launch. */
struct launch_ctx {
    const dev_ctx *ctx;
    uint32_t epoch;                            /* phase index on this rank */
    uint32_t armed;                            /* bit r: region r written by this launch */
    uint32_t gen[PROACT_MAX_REGIONS];          /* armed: generation produced now; else current */
    uint32_t gen_epoch[PROACT_MAX_REGIONS];    /* epoch that produced gen[r] */
    uint8_t gen_mech[PROACT_MAX_REGIONS];      /* mechanism that produced gen[r]: decides how a
                                                  consumer waits for it (flags / credits / none) */
    uint16_t mech;                             /* PROACT_MECH_* */
    uint16_t push;                             /* PROACT_PUSH_* */
    uint16_t agent_ctas;                       /* leading CTAs that run the agent (FUSED/ELIDE) */
    uint16_t agent_warps;                      /* warps of those CTAs that poll/push */
    uint32_t piece_bytes;                      /* agent work unit */
    uint16_t discovery;                        /* PROACT_DISCOVER_* */
    uint16_t flags;                            /* LCF_* */
};

/* launch_ctx::flags */
enum { LCF_SEPARATE = 1,   /* this is the SEPARATE agent kernel's copy (start-up deadline armed) */
       LCF_TILE_PUSH = 2,  /* PROACT_AGENT_PRODUCER: every producer CTA's transfer warp pushes its
                              own tiles (proact::tile_pusher); counters count DELIVERED bytes and
                              the last contributor of a chunk publishes its arrival flags */
       LCF_BULK_WARPS_SHIFT = 8   /* bits 8..11: issuing warps per BULK (TMA) agent CTA (0 = 1) */
};

/* error word encoding: (site << 8) | (-PROACT_ERR_*) */
enum { SITE_AGENT_POLL = 1, SITE_AGENT_CREDIT = 2, SITE_WAIT_RANGE = 3, SITE_WAIT_ALL = 4,
       SITE_SYNC = 5, SITE_COMMIT = 6, SITE_AGENT_COUNT = 7, SITE_AGENT_PUSH = 8,
       SITE_AGENT_START = 9,   /* SEPARATE agent: its producer grid never started (serialised?) */
       SITE_TILE_PUSH = 10,    /* tile pusher: credit wait / store completion */
       SITE_GRID_BARRIER = 11 };  /* a producer's grid-wide barrier (SSSP push rounds) */

#ifdef __CUDACC__

/* ---------------------------------------------------------------- PTX wrappers ------------- */
__device__ __forceinline__ uint32_t ld_acquire_gpu(const uint32_t *p)
{
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint32_t ld_acquire_sys(const uint32_t *p)
{
    uint32_t v;
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint32_t ld_relaxed_gpu(const uint32_t *p)
{
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint32_t ld_relaxed_sys(const uint32_t *p)
{
    uint32_t v;
    asm volatile("ld.relaxed.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_relaxed_sys(uint32_t *p, uint32_t v)
{
    asm volatile("st.relaxed.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_release_sys(uint32_t *p, uint32_t v)
{
    asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t atom_add_release_gpu(uint32_t *p, uint32_t v)
{
    uint32_t old;
    asm volatile("atom.release.gpu.global.add.u32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
    return old;
}
__device__ __forceinline__ uint32_t atom_add_acqrel_gpu(uint32_t *p, uint32_t v)
{
    uint32_t old;
    asm volatile("atom.acq_rel.gpu.global.add.u32 %0, [%1], %2;" : "=r"(old) : "l"(p), "r"(v) : "memory");
    return old;
}
__device__ __forceinline__ void red_add_relaxed_sys(uint32_t *p, uint32_t v)
{
    asm volatile("red.relaxed.sys.global.add.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void fence_acq_rel_sys() { asm volatile("fence.acq_rel.sys;" ::: "memory"); }
__device__ __forceinline__ void fence_acq_rel_gpu() { asm volatile("fence.acq_rel.gpu;" ::: "memory"); }
__device__ __forceinline__ uint4 ld_cg_v4(const uint4 *p)
{
    uint4 v;
    asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    return v;
}
__device__ __forceinline__ void st_v4(uint4 *p, uint4 v)
{
    asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
                 : "memory");
}
__device__ __forceinline__ uint64_t globaltimer()
{
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

/* ---------------------------------------------------------------- errors / spinning -------- */
__device__ __forceinline__ void raise_error(const dev_ctx *C, int site, int status)
{
    uint32_t code = ((uint32_t)site << 8) | (uint32_t)(-status);
    if (atomicCAS(C->err, 0u, code) == 0u) *(volatile uint32_t *)C->err_host = code;
}
__device__ __forceinline__ bool error_latched(const dev_ctx *C)
{
    return *(volatile uint32_t *)C->err != 0u;
}
/* One back-off step of a spin; true = give up (error latched by anyone, or watchdog expired). */
__device__ __forceinline__ bool spin_step(const dev_ctx *C, uint64_t t0, uint32_t &it, int site)
{
    ++it;
    if ((it & 31u) == 0u) {
        if (error_latched(C)) return true;
        if (globaltimer() - t0 > C->watchdog_ns) {
            raise_error(C, site, PROACT_ERR_TIMEOUT);
            return true;
        }
    }
    __nanosleep(it < 64 ? 32 : 256);
    return false;
}

/* ---------------------------------------------------------------- roles ------------------- */
__device__ __forceinline__ bool uses_agent(const launch_ctx &lc)
{
    return lc.mech == PROACT_MECH_FUSED || lc.mech == PROACT_MECH_ELIDE || lc.mech == PROACT_MECH_DMA;
}
__device__ __forceinline__ uint32_t producer_block(const launch_ctx &lc) { return blockIdx.x - lc.agent_ctas; }
__device__ __forceinline__ uint32_t producer_grid(const launch_ctx &lc) { return gridDim.x - lc.agent_ctas; }

__device__ __forceinline__ uint32_t chunk_len(const region_dev &R, uint32_t c)
{
    uint64_t lo = (uint64_t)c * R.chunk_bytes;
    uint64_t hi = lo + R.chunk_bytes;
    if (hi > R.own_bytes) hi = R.own_bytes;
    return (uint32_t)(hi - lo);
}
__device__ __forceinline__ uint32_t dests_of(const launch_ctx &lc, const region_dev &R, uint32_t c)
{
    const dev_ctx *C = lc.ctx;
    uint32_t m = R.chunk_dest ? R.chunk_dest[c] : (uint32_t)R.dest_mask;
    m &= ~(1u << C->rank);
    if (C->world < 32) m &= (1u << C->world) - 1u;
    return m;
}

/* Does my chunk c take part in the transfer this launch?  Chunks with destinations do.  Under
 * ELIDE (tracking and agent run as if pushing: the overhead methodology) every chunk does when
 * the region has one default destination mask -- at G = 1 it is empty -- and the chunks with
 * destinations do when per-chunk destinations are set (halo-only: as if pushing the halo). */
__device__ __forceinline__ bool transfers(const launch_ctx &lc, const region_dev &R, uint32_t c)
{
    return (lc.mech == PROACT_MECH_ELIDE && !R.chunk_dest) || dests_of(lc, R, c) != 0u;
}

/* ---------------------------------------------------------------- producer side (a2, a3) -- */

/* Instrumented store (a2): a weak store into the LOCAL replica at byte offset `off` (relative to
 * the replica base).  Under PROACT-inline (L143, Listing 1) the same value is also
 * stored to every destination peer's mirror (naive fine-grained P2P). */
template <class T>
__device__ __forceinline__ void put(const launch_ctx &lc, int r, uint64_t off, const T &v)
{
    const region_dev &R = lc.ctx->region[r];
    *reinterpret_cast<T *>(R.base + off) = v;
    if (lc.mech == PROACT_MECH_INLINE) {
        uint32_t c = (uint32_t)((off - R.own_off) / R.chunk_bytes);
        uint32_t m = dests_of(lc, R, c);
        while (m) {
            int p = __ffs(m) - 1;
            m &= m - 1;
            *reinterpret_cast<T *>(R.peer_base[p] + off) = v;
        }
    }
}

/* Dynamic work distribution for persistent producers: the next tile index of this launch, or
 * a value >= ntiles when none is left.  Call from ONE thread per CTA until it returns >= ntiles;
 * that final call also counts the CTA out, and the last CTA out re-arms the counters for the next
 * launch on this rank (stream order makes the reset visible to it).  Balances CTAs that share SMs
 * with agents or run slower, instead of the static round-robin's straggler tail. */
__device__ __forceinline__ uint32_t claim_tile(const launch_ctx &lc, uint32_t ntiles)
{
    uint32_t *S = lc.ctx->sched;
    const uint32_t t = atomicAdd(&S[0], 1u);
    if (t >= ntiles) {
        const uint32_t P = gridDim.x - lc.agent_ctas;
        if (atomicAdd(&S[1], 1u) + 1u == P) {
            S[0] = 0u;
            S[1] = 0u;
        }
    }
    return t;
}

/* Pieces of my chunk c under piece size `piece` (agent work units). */
__device__ __forceinline__ uint32_t pieces_of(const region_dev &R, uint32_t c, uint32_t piece)
{
    return (chunk_len(R, c) + piece - 1) / piece;
}
__device__ __forceinline__ uint32_t piece_size(const launch_ctx &lc, const region_dev &R)
{
    return lc.piece_bytes < R.chunk_bytes ? lc.piece_bytes : R.chunk_bytes;
}

/* Add `b` committed bytes to my chunk c of region r (a3).  The RMW is acq_rel: release publishes
 * this CTA's stores; acquire lets the LAST committer (old + b == expected, decided from the
 * returned value, reading R2) hand the chunk to the agent with everything ordered before it:
 * under QUEUE discovery it enqueues the chunk's pieces with release stores. */
/* PROACT_AGENT_PRODUCER (LCF_TILE_PUSH): my chunk c of region r has been DELIVERED to every
 * destination (its last contributor calls this, after acquiring every contributor's release):
 * raise its arrival flag (gen << 1 | changed) on every destination and bump their arrival
 * counters (a6), set my own flag, reset the counter for the next generation (reading R4).  The
 * contributors each executed fence.acq_rel.sys after their bulk stores completed, so the
 * release-store of the flag is ordered after every byte of the chunk at system scope. */
__device__ __forceinline__ void publish_chunk(const launch_ctx &lc, int r, uint32_t c)
{
    const dev_ctx *C = lc.ctx;
    const region_dev &R = C->region[r];
    const uint32_t gen = lc.gen[r];
    const uint32_t changed = (R.flags & PROACT_REGION_SPARSE) ? (R.changed_gen[c] == gen ? 1u : 0u) : 1u;
    const uint32_t flag = (gen << 1) | changed;
    const uint32_t g = R.chunk0 + c;
    uint32_t m = dests_of(lc, R, c);
    while (m) {
        const int p = __ffs(m) - 1;
        m &= m - 1;
        st_release_sys(R.peer_arrive[p] + g, flag);
        red_add_relaxed_sys(R.peer_arrive_count[p], 1u);
        if (R.deliv) atomicAdd(&R.deliv[(uint64_t)c * C->world + p], 1u);
    }
    R.arrive[g] = flag;
    R.counter[c] = 0u;
}

__device__ __forceinline__ void commit_chunk(const launch_ctx &lc, int r, uint32_t c, uint32_t b)
{
    const region_dev &R = lc.ctx->region[r];
    const uint32_t old = atom_add_acqrel_gpu(&R.counter[c], b);
    const uint32_t ex = R.expected[c];
    if (old + b > ex) {
        raise_error(lc.ctx, SITE_COMMIT, PROACT_ERR_PROTOCOL);
    } else if (old + b == ex && (lc.flags & LCF_TILE_PUSH)) {
        publish_chunk(lc, r, c);
    } else if (old + b == ex && lc.mech == PROACT_MECH_DMA) {
        // NEXT-3: the copy engines wait on the chunk's GROUP counter (prepared descriptors copy a
        // whole group); the last committer resets its chunk counter (no more commits can come
        // this generation) and counts the chunk into its group with system-scope release
        R.counter[c] = 0u;
        asm volatile("red.release.sys.global.add.u32 [%0], 1;" ::"l"(R.group_cnt + c / R.dma_group) : "memory");
    } else if (old + b == ex && !transfers(lc, R, c)) {
        // bound nowhere (halo-only interiors): nothing to push, no agent round trip -- the last
        // committer sets my own flag and resets the counter; the agent never sees the chunk
        publish_chunk(lc, r, c);
    } else if (old + b == ex && lc.discovery == PROACT_DISCOVER_QUEUE && lc.mech != PROACT_MECH_DMA) {
        const uint32_t piece = piece_size(lc, R);
        const uint32_t P = (R.chunk_bytes + piece - 1) / piece;
        const uint32_t np = pieces_of(R, c, piece);
        const uint32_t gen = lc.gen[r];
        const uint32_t idx = atomicAdd(&R.qctl[gen & 1u], np);
        fence_acq_rel_gpu();   // one release fence for all np entries (fence + relaxed stores)
        for (uint32_t k = 0; k < np; ++k) {
            const unsigned long long e = ((unsigned long long)gen << 32) | (unsigned long long)(c * P + k);
            asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(R.queue + idx + k), "l"(e) : "memory");
        }
    }
}

/* PROACT_AGENT_PRODUCER count of DELIVERED bytes (reading R21), for a caller that has already
 * fenced after its bulk stores completed (fence.proxy.async + fence.acq_rel.sys/gpu, tile_pusher's
 * flush): that fence is the release, so the count is a relaxed RMW -- no per-chunk membar -- and only
 * the contributor that completes the chunk acquires (fence.acq_rel.gpu: every other contributor's
 * fence-then-count is ordered before it) and publishes the chunk's flags. */
__device__ __forceinline__ void commit_delivered(const launch_ctx &lc, int r, uint32_t c, uint32_t b)
{
    const region_dev &R = lc.ctx->region[r];
    uint32_t old;
    asm volatile("atom.relaxed.gpu.global.add.u32 %0, [%1], %2;" : "=r"(old) : "l"(&R.counter[c]), "r"(b) : "memory");
    const uint32_t ex = R.expected[c];
    if (old + b > ex) {
        raise_error(lc.ctx, SITE_COMMIT, PROACT_ERR_PROTOCOL);
    } else if (old + b == ex) {
        fence_acq_rel_gpu();
        publish_chunk(lc, r, c);
    }
}

/* Tally commit (a3) for a contiguous span [off, off + nbytes) of region r (offsets relative to
 * the replica base, inside my slice) whose stores by this CTA are complete.  Call from ONE thread
 * after a __syncthreads() that follows the stores.  Adds the bytes to every covered chunk's
 * counter with release semantics; a chunk whose counter would exceed expected latches
 * PROACT_ERR_PROTOCOL (non-deterministic store count, L129). */
__device__ __forceinline__ void commit_span(const launch_ctx &lc, int r, uint64_t off, uint64_t nbytes)
{
    if (!uses_agent(lc)) return;
    const region_dev &R = lc.ctx->region[r];
    uint64_t rel = off - R.own_off;
    while (nbytes) {
        uint32_t c = (uint32_t)(rel / R.chunk_bytes);
        uint64_t end = (uint64_t)(c + 1) * R.chunk_bytes;
        if (end > R.own_bytes) end = R.own_bytes;
        uint32_t b = (uint32_t)((end - rel) < nbytes ? (end - rel) : nbytes);
        commit_chunk(lc, r, c, b);
        rel += b;
        nbytes -= b;
    }
}

/* Commit `nb` bytes at region offset `off` for each lane of the calling warp that has a span
 * (has = true; whole warp, converged); lanes whose spans fall in the same chunk are merged into
 * one release atomic (a3). */
__device__ __forceinline__ void warp_commit(const launch_ctx &lc, int r, bool has, uint64_t off, uint32_t nb)
{
    if (!uses_agent(lc)) return;
    const region_dev &R = lc.ctx->region[r];
    uint64_t rel = off - R.own_off;
    uint32_t c = has ? (uint32_t)(rel / R.chunk_bytes) : 0xFFFFFFFFu;
    bool single = has && (uint32_t)((rel + nb - 1) / R.chunk_bytes) == c;
    uint32_t key = single ? c : 0xFFFFFFFFu;
    uint32_t grp = __match_any_sync(0xFFFFFFFFu, key);
    const uint32_t tot = __reduce_add_sync(grp, single ? nb : 0u);   // spans may differ in size
    if (single) {
        if ((__ffs(grp) - 1) == (int)(threadIdx.x & 31)) commit_chunk(lc, r, c, tot);
    } else if (has) {
        commit_span(lc, r, off, nb);
    }
}

/* Chunk-state marks for SPARSE regions (SSSP dirty frontier, reading R13).  Plain stores; call
 * before the commit that covers the chunk (the commit's release publishes them). */
__device__ __forceinline__ void mark_changed(const launch_ctx &lc, int r, uint64_t off)
{
    const region_dev &R = lc.ctx->region[r];
    R.changed_gen[(off - R.own_off) / R.chunk_bytes] = lc.gen[r];
}
__device__ __forceinline__ void mark_push(const launch_ctx &lc, int r, uint64_t off)
{
    const region_dev &R = lc.ctx->region[r];
    R.push_gen[(off - R.own_off) / R.chunk_bytes] = lc.gen[r];
}
/* Did my chunk containing `off` change in region r's current generation? */
__device__ __forceinline__ bool local_changed(const launch_ctx &lc, int r, uint64_t off)
{
    const region_dev &R = lc.ctx->region[r];
    return R.changed_gen[(off - R.own_off) / R.chunk_bytes] == lc.gen[r];
}
/* Phase vote (e.g. "something changed"): OR-ed over all ranks by a BARRIER phase_sync.  The
 * word is tagged with the epoch (epoch + 1 marks a vote cast in `epoch`), so a slot never needs
 * clearing: a stale tag from an earlier epoch simply does not match. */
__device__ __forceinline__ void vote(const launch_ctx &lc)
{
    atomicMax(&lc.ctx->vote[lc.epoch & 1u], lc.epoch + 1u);
}

/* ---------------------------------------------------------------- consumer side (a7) ------- */

/* Wait (ONE thread; the caller then __syncthreads()) until every REMOTE chunk overlapping
 * [off, off + nbytes) of region r holds the region's current generation lc.gen[r].  How depends on
 * the mechanism that PRODUCED that generation (lc.gen_mech[r]): FUSED/ELIDE -> the per-chunk
 * arrival flags (ld.acquire.sys); INLINE/BULK -> the owner's phase credit (the data is complete
 * when its producer's phase is); LOCAL -> nothing (single rank, or moved by the caller).  Returns the OR of
 * the covered chunks' "changed" bits (FUSED/ELIDE only; 1 otherwise).  Generation 0 (identical
 * initial replicas, reading R16) never waits.  Must not be used on a region armed by the same
 * launch (a launch reads the previous generation of what it does not write). */
__device__ __forceinline__ uint32_t wait_range(const launch_ctx &lc, int r, uint64_t off, uint64_t nbytes)
{
    const dev_ctx *C = lc.ctx;
    const region_dev &R = C->region[r];
    uint32_t gen = lc.gen[r];
    const uint32_t pm = lc.gen_mech[r];
    if (gen == 0 || nbytes == 0 || pm == PROACT_MECH_LOCAL) return 1u;
    const bool flags = pm == PROACT_MECH_FUSED || pm == PROACT_MECH_ELIDE;
    uint64_t hi = off + nbytes;
    uint32_t changed = 0;
    uint64_t t0 = globaltimer();
    uint32_t it = 0;
    for (int p = 0; p < C->world; ++p) {
        uint64_t plo = R.rank_off[p], phi = R.rank_off[p + 1];
        if (p == C->rank || phi <= off || plo >= hi || plo == phi) continue;
        if (flags) {
            uint64_t a = (off > plo ? off : plo) - plo, b = (hi < phi ? hi : phi) - plo;
            uint32_t c0 = (uint32_t)(a / R.chunk_bytes), c1 = (uint32_t)((b - 1) / R.chunk_bytes);
            for (uint32_t c = c0; c <= c1; ++c) {
                const uint32_t *f = &R.arrive[R.rank_chunk0[p] + c];
                uint32_t v;
                while (((v = ld_acquire_sys(f)) >> 1) < gen)
                    if (spin_step(C, t0, it, SITE_WAIT_RANGE)) return 1u;
                changed |= v & 1u;
            }
        } else {
            uint32_t need = lc.gen_epoch[r] + 1u;
            while ((ld_acquire_sys(&C->done[p]) >> 1) < need)
                if (spin_step(C, t0, it, SITE_WAIT_RANGE)) return 1u;
            changed = 1u;
        }
    }
    return changed;
}

/* Wait (ONE thread) until every chunk pushed into this rank for region r's current generation has
 * arrived: FUSED/ELIDE poll the region's arrival counter (gen * n_in), INLINE/BULK every peer's
 * credit.  For all-to-all consumers (PageRank, SSSP gathers). */
__device__ __forceinline__ void wait_all(const launch_ctx &lc, int r)
{
    const dev_ctx *C = lc.ctx;
    const region_dev &R = C->region[r];
    uint32_t gen = lc.gen[r];
    const uint32_t pm = lc.gen_mech[r];
    if (gen == 0 || pm == PROACT_MECH_LOCAL) return;
    const bool flags = pm == PROACT_MECH_FUSED || pm == PROACT_MECH_ELIDE;
    uint64_t t0 = globaltimer();
    uint32_t it = 0;
    if (flags && R.n_in != 0xFFFFFFFFu) {
        uint32_t need = gen * R.n_in;
        while (ld_acquire_sys(R.arrive_count) < need)
            if (spin_step(C, t0, it, SITE_WAIT_ALL)) return;
    } else {
        uint32_t need = lc.gen_epoch[r] + 1u;   /* owner finished the producing phase */
        for (int p = 0; p < C->world; ++p) {
            if (p == C->rank) continue;
            while ((ld_acquire_sys(&C->done[p]) >> 1) < need)
                if (spin_step(C, t0, it, SITE_WAIT_ALL)) return;
        }
    }
}

/* Changed bit of global chunk g of region r as last published (valid after wait_all/wait_range;
 * covers my own chunks too: the agent raises my local flag as well). */
__device__ __forceinline__ uint32_t chunk_flag(const launch_ctx &lc, int r, uint32_t g)
{
    return lc.ctx->region[r].arrive[g];
}

#endif /* __CUDACC__ */
} /* namespace proact */

#ifdef __CUDACC__
#include "proact_agent.cuh"
#include "proact_tile.cuh"
namespace proact {
/* Agent CTAs (the first lc.agent_ctas blocks of a FUSED/ELIDE launch) run the polling agent and
 * return true; producer CTAs get false.  Call first thing in a producer kernel. */
__device__ __forceinline__ bool agent_dispatch(const launch_ctx &lc)
{
    if (blockIdx.x >= lc.agent_ctas) {
        // the producer grid of this epoch has started (a separate agent's start-up deadline)
        if (blockIdx.x == lc.agent_ctas && threadIdx.x == 0) *(volatile uint32_t *)lc.ctx->started = lc.epoch + 1u;
        return false;
    }
    agent_loop(lc);
    return true;
}
} /* namespace proact */
#endif

#endif /* PROACT_DEVICE_CUH */
