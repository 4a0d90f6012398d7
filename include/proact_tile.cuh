// proact_tile.cuh -- PROACT_AGENT_PRODUCER: the transfer warp INSIDE each producer CTA (sm_100a).
// Included by proact_device.cuh; internal to each translation unit (no -rdc).
//
// PAPER.md Sec. III-C: "a small configurable number of GPU warps are specialized to perform
// data transfers ... the transfer threads read a chunk from the local staging array and perform
// remote writes to the target GPU(s)".  On B200 the cheapest place for those warps is next to the
// compute warps that produce the data: the compute warps stage each finished output row / tile in
// a shared-memory ring, and ONE transfer warp per CTA hands every staged span to the TMA engine as
// bulk stores (cp.async.bulk.global.shared::cta) -- to the local replica and to every destination
// mirror (same offset, reading R7) -- so the produced bytes are never read back from HBM and no SM
// is set aside for an agent.  Readiness (a3) then counts DELIVERED bytes: after its stores
// completed (cp.async.bulk.wait_group), the transfer warp fences at system scope and adds the
// span's bytes to the chunk counter with acq_rel; the contributor that completes the chunk
// (return value == expected, reading R2) publishes its arrival flags (proact::publish_chunk, a6).
//
// Ring protocol (q = output span sequence number of the CTA, OS slots):
//   compute warps: tp_acquire(q)  -> write slot q % OS -> (one thread) desc[q % OS] = {off, bytes,
//                  flags} -> tp_publish(q)   (fence.proxy.async.shared::cta + mbarrier arrive)
//   transfer warp: tile_pusher(): wait full, issue the span's bulk stores as one bulk group,
//                  release the slot once the group's shared-memory reads are done, count the span
//                  once the group completed; flush (fence + commits) every PROACT_TP_FLUSH rows.
#pragma once

namespace proact {

struct tile_desc {
    uint64_t off;      // byte offset in the region's replica (inside my slice) of the first row
    uint32_t bytes;    // bytes per row, multiple of 16 (rows are 16-byte aligned)
    uint32_t flags;    // TD_* | rows << 8: a span is `rows` rows of `bytes` bytes, row k at global
                       // offset off + k * pitch and at shared offset k * srow of its slot
};
enum { TD_END = 1 };   // no more spans: the transfer warp drains and returns
__host__ __device__ constexpr uint32_t td_rows(uint32_t rows) { return rows << 8; }

#ifndef PROACT_TP_RD
#define PROACT_TP_RD 0   // release a slot as soon as its bulk stores have read it (r02z sweep: 0.650 vs 0.715 ms loopback G = 2)
#endif
#ifndef PROACT_TP_CD
#define PROACT_TP_CD 8
#endif
#ifndef PROACT_TP_SYSFENCE
#define PROACT_TP_SYSFENCE 1
#endif
// completed rows per flush (one fence + the merged counter commits).  Under full HBM load a fence
// waits ~4 us for the SM's write queue to drain, and the transfer warp issues no span meanwhile, so
// flushes are rare (r02z sweep, loopback G = 2 at 1 MiB chunks: 64 -> 256 rows 0.647 -> 0.553 ms)
#ifndef PROACT_TP_FLUSH
#define PROACT_TP_FLUSH 256
#endif
#ifndef PROACT_TP_RELAXED_COMMIT   // flush commits: relaxed counts after the flush fence
#define PROACT_TP_RELAXED_COMMIT 1
#endif
#ifndef PROACT_TP_PROXYFENCE
#define PROACT_TP_PROXYFENCE 1
#endif
constexpr uint32_t TP_FLY = 16;   // descriptors of in-flight spans (> TP_CD)
constexpr int TP_RD = PROACT_TP_RD;   // bulk groups whose shared-memory reads may still be pending
constexpr int TP_CD = PROACT_TP_CD;   // bulk groups that may still be in flight (not complete)
#ifndef PROACT_TP_PEND
#define PROACT_TP_PEND 128   // 128 KiB chunks: a 32-row tile strip touches 16 chunks
#endif
constexpr uint32_t TP_PEND = PROACT_TP_PEND;  // (chunk, bytes) entries of completed, uncommitted rows
static_assert(TP_CD < (int)TP_FLY, "in-flight descriptors");

// Shared-memory block of a tile pusher (placed in the kernel's dynamic shared memory).
template <uint32_t OS>
struct tile_ring_ctl {
    uint64_t full[OS];       // producer warps -> transfer warp (count = producer warps)
    uint64_t empty[OS];      // transfer warp -> producer warps (count 1)
    tile_desc desc[OS];
    tile_desc fly[TP_FLY];
    uint32_t pend_c[TP_PEND];   // completed bytes not yet committed, merged per chunk
    uint32_t pend_b[TP_PEND];
    char *peer[PROACT_MAX_RANKS];
};

__device__ __forceinline__ uint32_t tp_smem(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
#ifndef PROACT_TP_IDLE_NS
#define PROACT_TP_IDLE_NS 8000   // producers idle this long: publish what is in flight
#endif
#ifndef PROACT_TP_SUSPEND_NS
#define PROACT_TP_SUSPEND_NS 20000   // try_wait suspend-time hint: a waiting warp sleeps until the
#endif                               // phase completes instead of spinning on issue slots
__device__ __forceinline__ void tp_mbar_wait(uint64_t *b, uint32_t parity)
{
    uint32_t done;
    do {
        asm volatile("{\n\t.reg .pred p;\n\t"
                     "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
                     "selp.u32 %0, 1, 0, p;\n\t}"
                     : "=r"(done) : "r"(tp_smem(b)), "r"(parity), "n"(PROACT_TP_SUSPEND_NS) : "memory");
    } while (!done);
}
__device__ __forceinline__ bool tp_mbar_test(uint64_t *b, uint32_t parity)
{
    uint32_t done;
    asm volatile("{\n\t.reg .pred p;\n\t"
                 "mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
                 "selp.u32 %0, 1, 0, p;\n\t}"
                 : "=r"(done) : "r"(tp_smem(b)), "r"(parity) : "memory");
    return done != 0;
}
// Wait up to (about) PROACT_TP_IDLE_NS for the phase: suspending try_waits (the hardware wakes
// the thread when the phase completes, so a waiting transfer warp takes no issue slots from the
// compute warps and reacts at once), the elapsed time checked between them.  True if completed.
__device__ __forceinline__ bool tp_mbar_try(uint64_t *b, uint32_t parity)
{
    if (tp_mbar_test(b, parity)) return true;
    const uint64_t t0 = globaltimer();
    do {
        uint32_t done;
        asm volatile("{\n\t.reg .pred p;\n\t"
                     "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\t"
                     "selp.u32 %0, 1, 0, p;\n\t}"
                     : "=r"(done) : "r"(tp_smem(b)), "r"(parity), "n"(1000) : "memory");
        if (done) return true;
    } while (globaltimer() - t0 < PROACT_TP_IDLE_NS);
    return false;
}
__device__ __forceinline__ void tp_mbar_arrive(uint64_t *b)
{
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(tp_smem(b)) : "memory");
}

// One thread: initialise the ring's barriers (producers = producer warps arriving per span).
template <uint32_t OS>
__device__ __forceinline__ void tp_init(tile_ring_ctl<OS> *T, uint32_t producers)
{
    for (uint32_t s = 0; s < OS; ++s) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(tp_smem(&T->full[s])), "r"(producers) : "memory");
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(tp_smem(&T->empty[s])) : "memory");
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}

// Producer warp: wait until slot q % OS may be overwritten (its previous span's reads are done).
template <uint32_t OS>
__device__ __forceinline__ void tp_acquire(tile_ring_ctl<OS> *T, uint32_t q)
{
    if (q >= OS) tp_mbar_wait(&T->empty[q % OS], ((q / OS) - 1) & 1u);
}
// Producer warp, after its shared-memory writes of span q (and the descriptor, by one of the
// producer threads): make the generic-proxy writes visible to the TMA engine, then arrive.
template <uint32_t OS>
__device__ __forceinline__ void tp_publish(tile_ring_ctl<OS> *T, uint32_t q)
{
    if (PROACT_TP_PROXYFENCE) asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncwarp();
    if ((threadIdx.x & 31) == 0) tp_mbar_arrive(&T->full[q % OS]);
}

__device__ __forceinline__ void tp_store(void *gdst, uint32_t ssrc, uint32_t bytes)
{
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(gdst), "r"(ssrc), "r"(bytes)
                 : "memory");
}

// Chunk of byte offset `rel` (relative to my slice) for chunk size cb (a multiple of 16):
// 32-bit division on 16-byte units while rel < 64 GiB.
__device__ __forceinline__ uint32_t tp_chunk(uint64_t rel, uint32_t cb)
{
    return rel < (1ull << 36) ? (uint32_t)(rel >> 4) / (cb >> 4) : (uint32_t)(rel / cb);
}

// The transfer warp (all 32 lanes, converged).  `ring` = OS slots of `slot_bytes` bytes; a span's
// row k sits at shared offset k * srow of its slot and goes to global offset off + k * pitch.
// Lane 0 runs the per-span loop alone (wait, issue, release, completion accounting: a short
// dependent chain per row); completed bytes are merged per chunk into a pending list, and the
// whole warp joins only for credit waits and for the flushes that commit the list -- one fence
// (proxy fence + fence.acq_rel.sys when a pending byte went to a peer) per PROACT_TP_FLUSH rows,
// then one relaxed RMW per pending chunk (lane j: entries j, j + 32, ...; commit_delivered: the
// flush fence is the release, the completing contributor acquires before publishing).
//
// local_done = true: the producer warps already stored the span to the local replica themselves
// (plain st.global, before their tp_publish, whose release the transfer warp acquires): only the
// peer copies go through the TMA engine, which then moves (G-1)/G of what it would otherwise.
template <uint32_t OS>
__device__ __noinline__ void tile_pusher(const launch_ctx &lc, int r, const unsigned char *ring, uint32_t slot_bytes,
                                         tile_ring_ctl<OS> *T, uint32_t srow = 0, uint64_t pitch = 0,
                                         bool local_done = false)
{
    constexpr int RD = TP_RD < (int)OS ? TP_RD : (int)OS - 1;   // a slot must come back before the ring wraps
    const dev_ctx *C = lc.ctx;
    const region_dev &R = C->region[r];
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t FULLM = 0xFFFFFFFFu;
    const bool elide = lc.mech == PROACT_MECH_ELIDE;
    const uint32_t peers = (C->world < 32 ? (1u << C->world) - 1u : FULLM) & ~(1u << C->rank);
    const uint32_t dmask = (uint32_t)R.dest_mask & peers;
    const uint32_t *chunk_dest = R.chunk_dest;
    const uint64_t own_off = R.own_off;
    const uint32_t cb = R.chunk_bytes;
    char *const mine = R.base + own_off;
    if (lane < PROACT_MAX_RANKS) T->peer[lane] = R.peer_base[lane] ? R.peer_base[lane] + own_off : nullptr;
    __syncwarp();
    const uint32_t ring_s = tp_smem(ring);
    enum { EV_FLUSH = 1, EV_CREDIT = 2, EV_END = 3 };
    uint32_t q = 0;          // next span to issue
    uint32_t rel = 0;        // spans [0, rel) released to the producers (their slots are free)
    uint32_t done = 0;       // spans [0, done) completed (lane 0)
    uint32_t npend = 0;      // pending (chunk, bytes) entries (lane 0)
    uint32_t nrows = 0;      // completed rows since the last flush (lane 0)
    bool remote = false;     // a pending row went to a peer: the flush needs the system fence
    // peers known to have finished phase epoch-1 (reading R6); without per-chunk destinations
    // every destination is needed at once
    uint32_t credit_ok = 0;
    bool dead = false;       // an error latched: keep cycling the ring, store nothing
    // lane 0's caches of the chunk of the previous issued / completed row
    uint64_t cur_lo = 1, cur_hi = 0, cmp_lo = 1, cmp_hi = 0;
    uint32_t cur_dm = 0, cmp_c = 0;
    auto add_pend = [&](uint32_t c, uint32_t b) {   // lane 0
        if (npend && T->pend_c[npend - 1] == c) {
            T->pend_b[npend - 1] += b;
        } else {
            T->pend_c[npend] = c;
            T->pend_b[npend] = b;
            ++npend;
        }
    };
    auto dests = [&](uint32_t c) { return chunk_dest ? chunk_dest[c] & peers : dmask; };
    // lane 0: merge the rows of completed spans [done, upto) into the pending list while it has
    // room; returns true when the list is (nearly) full
    auto merge = [&](uint32_t upto) {
        bool full_list = npend + 2 * 8 > TP_PEND;   // room for a span of <= 8 straddling rows
        while ((int32_t)(upto - done) > 0 && !full_list) {
            const tile_desc f = T->fly[done % TP_FLY];
            const uint32_t fr = f.flags >> 8;
            if (f.flags & 1u) remote = true;
            for (uint32_t k = 0; k < fr; ++k) {
                const uint64_t a0 = f.off - own_off + k * pitch, a1 = a0 + f.bytes;
                if (a0 >= cmp_lo && a1 <= cmp_hi) {
                    add_pend(cmp_c, f.bytes);
                } else {
                    for (uint64_t a = a0; a < a1;) {
                        const uint32_t c = tp_chunk(a, cb);
                        const uint64_t b = min(a1, (uint64_t)(c + 1) * cb);
                        add_pend(c, (uint32_t)(b - a));
                        cmp_c = c;
                        cmp_lo = (uint64_t)c * cb;
                        cmp_hi = cmp_lo + cb;
                        a = b;
                    }
                }
            }
            ++done;
            nrows += fr;
            full_list = npend + 2 * 8 > TP_PEND;
        }
        return full_list;
    };
    for (;;) {
        uint32_t ev = 0, arg = 0;
        if (lane == 0) {
            for (;;) {
                const uint32_t slot = q % OS;
                if ((done < q || npend) && !tp_mbar_try(&T->full[slot], (q / OS) & 1u)) {
                    // the producers have had nothing for us for a while (a stretch of tiles bound
                    // nowhere, e.g. halo-only interiors): complete and publish what is in flight
                    // instead of holding its arrival flags back until the next flush
                    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
                    merge(q);
                    ev = EV_FLUSH;
                    break;
                }
                tp_mbar_wait(&T->full[slot], (q / OS) & 1u);
                const tile_desc d = T->desc[slot];
                if (d.flags & TD_END) {
                    asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
                    ev = EV_END;
                    break;
                }
                const uint32_t nr = d.flags >> 8;
                const uint64_t rel0 = d.off - own_off;
                // credits for every destination of the span's rows
                uint32_t need = 0;
                if (!chunk_dest) {
                    need = dmask & ~credit_ok;
                } else {
                    for (uint32_t k = 0; k < nr; ++k) {
                        const uint64_t a0 = rel0 + k * pitch, a1 = a0 + d.bytes;
                        for (uint32_t c = tp_chunk(a0, cb), c1 = tp_chunk(a1 - 1, cb); c <= c1; ++c) need |= dests(c);
                    }
                    need &= ~credit_ok;
                }
                if (need && !dead) {
                    ev = EV_CREDIT;
                    arg = need;
                    break;
                }
                const uint32_t src0 = ring_s + slot * slot_bytes;
                uint32_t to_peer = 0;
                if (!dead) {
                    for (uint32_t k = 0; k < nr; ++k) {
                        const uint64_t a0 = rel0 + k * pitch, a1 = a0 + d.bytes;
                        const uint32_t src = src0 + k * srow;
                        if (!(a0 >= cur_lo && a1 <= cur_hi)) {
                            const uint32_t c0 = tp_chunk(a0, cb);
                            cur_lo = (uint64_t)c0 * cb;
                            cur_hi = cur_lo + cb;
                            cur_dm = dests(c0);
                        }
                        if (a1 <= cur_hi) {   // one chunk (the common case)
                            if (!local_done) tp_store(mine + a0, src, d.bytes);
                            uint32_t m = elide ? 0u : cur_dm;
                            to_peer |= m;
                            while (m) {
                                const int p = __ffs(m) - 1;
                                m &= m - 1;
                                tp_store(T->peer[p] + a0, src, d.bytes);
                            }
                        } else {   // split at chunk boundaries (per-chunk destinations)
                            for (uint64_t a = a0; a < a1;) {
                                const uint32_t c = tp_chunk(a, cb);
                                const uint64_t b = min(a1, (uint64_t)(c + 1) * cb);
                                const uint32_t s_off = (uint32_t)(a - a0), n = (uint32_t)(b - a);
                                if (!local_done) tp_store(mine + a, src + s_off, n);
                                uint32_t m = elide ? 0u : dests(c);
                                to_peer |= m;
                                while (m) {
                                    const int p = __ffs(m) - 1;
                                    m &= m - 1;
                                    tp_store(T->peer[p] + a, src + s_off, n);
                                }
                                a = b;
                            }
                        }
                    }
                }
                T->fly[q % TP_FLY] = tile_desc{d.off, d.bytes, (d.flags & ~0xFFu) | (to_peer ? 1u : 0u)};
                asm volatile("cp.async.bulk.commit_group;" ::: "memory");
                asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(RD) : "memory");
                for (; rel + RD <= q; ++rel) tp_mbar_arrive(&T->empty[rel % OS]);
                asm volatile("cp.async.bulk.wait_group %0;" ::"n"(TP_CD) : "memory");
                ++q;
                // spans [done, q - CD) have completed: merge their rows' bytes into the pending list
                const bool full_list = merge(q - TP_CD);
                if (full_list || nrows >= PROACT_TP_FLUSH) {
                    ev = EV_FLUSH;
                    break;
                }
            }
        }
        ev = __shfl_sync(FULLM, ev, 0);
        __syncwarp();   // lane 0's shared-memory writes (pending list) -> the other lanes
        if (ev == EV_CREDIT) {
            arg = __shfl_sync(FULLM, arg, 0);
            bool bad = false;
            if (arg >> lane & 1u) {
                const uint64_t t0 = globaltimer();
                uint32_t it = 0;
                while ((ld_acquire_sys(&C->done[lane]) >> 1) < lc.epoch)
                    if (spin_step(C, t0, it, SITE_TILE_PUSH)) { bad = true; break; }
            }
            dead = dead || __any_sync(FULLM, bad);
            credit_ok |= arg;
            continue;
        }
        for (;;) {
            if (ev == EV_END && lane == 0) merge(q);   // everything issued has completed: merge the rest
            __syncwarp();
            const uint32_t n = __shfl_sync(FULLM, npend, 0);
            const bool sys = __shfl_sync(FULLM, remote, 0);
            if (n) {
                asm volatile("fence.proxy.async;" ::: "memory");   // async-proxy writes -> generic
                if (PROACT_TP_SYSFENCE && sys) fence_acq_rel_sys(); // ... ordered before the counts (a3)
                else fence_acq_rel_gpu();
                // chunks bound nowhere are never counted (tiles that write only such chunks skip
                // the transfer warp altogether, so their counts would be partial)
                for (uint32_t j = lane; j < n; j += 32) {
                    if (dead || !transfers(lc, R, T->pend_c[j])) continue;
#if PROACT_TP_RELAXED_COMMIT
                    commit_delivered(lc, r, T->pend_c[j], T->pend_b[j]);
#else
                    commit_chunk(lc, r, T->pend_c[j], T->pend_b[j]);
#endif
                }
                __syncwarp();
            }
            if (lane == 0) {
                npend = 0;
                nrows = 0;
                remote = false;
            }
            if (ev != EV_END || __shfl_sync(FULLM, done, 0) == __shfl_sync(FULLM, q, 0)) break;
        }
        if (ev == EV_END) break;
    }
}

}  // namespace proact
