/*
 * proact.h -- C ABI of libproact, the B200-native PROACT runtime.
 *
 * PROACT (PAPER.md, ISCA'21): producer kernels store peer-bound data into the LOCAL copy of a
 * "PROACT-enabled region" that has a 1:1 address correspondence with every peer replica
 * (Sec. III-B); per-chunk atomic counters track when each chunk is fully written
 * (L127-L131); a polling transfer agent made of a few specialised warps pushes each completed
 * chunk to the peers at interconnect-friendly granularity while the producer still runs
 * (Sec. III-C); a profiler picks mechanism, chunk size and transfer-thread count per
 * application and platform (Sec. III-A; Table II).  Listing 1 (L178-L239)
 * sketches the paper's interface (proact_init, counters, region1[gpu], mapping); this header is
 * the B200 re-design of that interface.
 *
 * Model.  SPMD: `world` ranks, one per GPU (one process per GPU under torchrun, or one host
 * thread per rank inside a process; several ranks may share a device -- "loopback", used to
 * exercise the whole protocol on one GPU).  Every call below operates on the calling thread's
 * rank context (thread-local), created by proact_init / proact_init_ex.  Calls marked
 * COLLECTIVE must be made by every rank in the same order.
 *
 * Errors.  Every int-returning call returns PROACT_OK (0) or a negative PROACT_ERR_* code;
 * proact_error_string() names it.  Device-side failures (watchdog timeout in a spin, counter
 * over-count) are latched in a device error word and surface on the next host call that checks
 * it (proact_phase_sync, proact_check).  No call aborts the process.
 *
 * Memory ownership.  Region memory belongs to the CALLER (e.g. torch tensors allocated with the
 * caching allocator's expandable_segments disabled, so cudaIpcGetMemHandle works) and must
 * outlive the region.  Counters, flags, credits, the device context and IPC mappings belong to
 * the library and are released by proact_finalize().
 */
#ifndef PROACT_H
#define PROACT_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define PROACT_MAX_RANKS 16
#define PROACT_BULK_SMEM (33 * 1024)   /* min dynamic smem of a launch with TMA pushes */
#define PROACT_MAX_REGIONS 8

/* ---- status codes ------------------------------------------------------------------------ */
enum {
    PROACT_OK = 0,
    PROACT_ERR_INVALID = -1,   /* bad argument (alignment, sizes, ids, unsupported launch) */
    PROACT_ERR_CUDA = -2,      /* a CUDA runtime/driver call failed: see proact_last_cuda_error */
    PROACT_ERR_NOPEER = -3,    /* peer access / IPC mapping between two ranks impossible */
    PROACT_ERR_STATE = -4,     /* call out of order (not initialised, already initialised ...) */
    PROACT_ERR_TIMEOUT = -5,   /* rendezvous or device watchdog expired (a spin never completed) */
    PROACT_ERR_PROTOCOL = -6,  /* device detected a protocol violation (counter over-count) */
    PROACT_ERR_NOMEM = -7      /* host or device allocation failed */
};

/* ---- transfer mechanisms (Sec. III-C, Sec. IV-B) ----------- */
enum {
    PROACT_MECH_FUSED = 0,   /* PROACT-decoupled, polling agent: persistent agent CTAs fused
                                into the producer's grid (L137; replaces the separate
                                long-lived kernel of Listing 1) */
    PROACT_MECH_INLINE = 1,  /* PROACT-inline: producer stores every value to every peer (L143,
                                Listing 1 user_kernel_inline L190-L197); "naive P2P" baseline */
    PROACT_MECH_BULK = 2,    /* cudaMemcpy duplication after the kernel (L245): bulk-DMA baseline */
    PROACT_MECH_LOCAL = 3,   /* no transfer by the library: uninstrumented kernel; data moved by
                                the caller (NCCL all-gather baseline) or G = 1 reference */
    PROACT_MECH_ELIDE = 4,   /* FUSED with the remote stores elided: tracking + agent only, the
                                paper's overlap methodology (Sec. V-C); output NOT valid */
    PROACT_MECH_DMA = 5      /* "hardware PROACT" emulation (Sec. III-D; SURVEY
                                NEXT-3): producers tally as under FUSED, but the transfer agent is
                                the copy engines: per chunk, a stream wait on counter == expected,
                                one DMA copy per destination, a counter reset -- prepared by the
                                host, triggered by the counters, no SM does any transfer.
                                Consumers wait on phase credits.  Best with large chunks. */
};

/* ---- agent push instruction (a5) -------------------------------------------------------- */
enum {
    PROACT_PUSH_VEC16 = 0,   /* 16-byte ld.global.cg / st.global.v4, 512 B per warp instruction */
    PROACT_PUSH_BULK = 1,    /* cp.async.bulk (TMA): global->smem stage, then one smem->global bulk
                                store per destination; one agent warp per CTA (lane 0 issues),
                                the CTA's dynamic shared memory is its staging ring */
    PROACT_PUSH_MULTICAST = 2 /* NVLS: one 16-byte multimem.st.global.v4 per lane to
                                the region's multicast address reaches every peer's replica through
                                the NVSwitch; for regions in replicas from proact_alloc_replica on a
                                multicast-capable system, units bound for every peer; anything
                                else is pushed as PROACT_PUSH_VEC16 */
};

/* ---- agent discovery of completed chunks (a4) ------------------------------------------- */
enum {
    PROACT_DISCOVER_QUEUE = 0, /* the last committer of a chunk enqueues its pieces; agent warps
                                  pop them in completion order (O(1) per chunk, no scanning) */
    PROACT_DISCOVER_SCAN = 1   /* agent warps poll the readiness counters of statically owned
                                  32-unit windows and claim ready ones with a warp ballot */
};

/* ---- where the transfer agent runs ----------------------------------------------------- */
enum {
    PROACT_AGENT_FUSED = 0,    /* leading CTAs of the producer's own grid (cooperative launch on a
                                  dedicated GPU: co-residency guaranteed); shares its registers */
    PROACT_AGENT_SEPARATE = 1, /* its own small kernel, launched first on a high-priority stream
                                  (the paper's "independently launched long-lived kernel", L137),
                                  with its own registers and a 200 KiB TMA staging ring; the
                                  producer grid leaves room for it */
    PROACT_AGENT_PRODUCER = 2  /* a transfer warp inside every producer CTA: the compute warps
                                  stage each finished output row/tile in shared memory, the
                                  transfer warp bulk-stores it (TMA, cp.async.bulk smem->global)
                                  to the local replica and to every destination mirror, and once
                                  the stores completed counts the chunk's DELIVERED bytes; the
                                  last contributor publishes the chunk's arrival flags.  No
                                  read-back of the produced bytes, no agent SMs (B200 re-design
                                  of L137's specialised transfer warps).  Only for kernels
                                  launched with PROACT_LAUNCH_TILE_PUSH; other launches fall back
                                  to PROACT_AGENT_SEPARATE. */
};

/* ---- proact_launch_ex flags ------------------------------------------------------------- */
enum {
    PROACT_LAUNCH_TILE_PUSH = 1, /* the kernel implements proact::tile_pusher (a transfer warp that
                                    pushes its own tiles) and may run under PROACT_AGENT_PRODUCER */
    PROACT_LAUNCH_CLUSTER_SHIFT = 8 /* bits 8..11: thread-block cluster size (2, 4 or 8; 0/1 = none)
                                    of the producer grid; the grid is a whole number of clusters
                                    sized by cudaOccupancyMaxActiveClusters.  Not with agent CTAs in
                                    the producer grid (PROACT_AGENT_FUSED): INVALID */
};

/* ---- phase synchronisation modes (a8) ----------------------------------------------------- */
enum {
    PROACT_SYNC_SIGNAL = 0,  /* credit peers "phase e done"; consumers rely on arrival flags */
    PROACT_SYNC_BARRIER = 1  /* additionally wait until every peer finished phase e: the paper's
                                "succeeding global synchronization barrier" (L125, L145) */
};

/* ---- region flags -------------------------------------------------------------------------- */
enum {
    PROACT_REGION_SPARSE = 1 /* push a chunk only when the producer marked it (proact::mark_push);
                                flags are still raised for every chunk (SSSP dirty frontier) */
};

/* Per-rank tunables; what the profiler (proact_autotune) chooses.  Zero fields mean "default". */
typedef struct proact_config {
    int32_t mech;          /* PROACT_MECH_* */
    int32_t push;          /* PROACT_PUSH_* */
    int32_t agent_warps;   /* transfer warps (Table II "transfer thread count" / 32) */
    int32_t block;         /* threads per CTA of fused launches (agent CTAs use the same) */
    uint32_t piece_bytes;  /* agent work unit inside a chunk (multiple of 16, >= 4096) */
    uint32_t watchdog_ms;  /* device spin budget before PROACT_ERR_TIMEOUT */
    int32_t grid_cap;      /* 0 = fill the device share; else max CTAs of a fused launch */
    uint32_t chunk_bytes;  /* preferred chunk size for workload drivers (profiler axis) */
    int32_t discovery;     /* PROACT_DISCOVER_*: how agents find completed chunks (a4) */
    int32_t agent_kernel;  /* PROACT_AGENT_*: where the agent warps run */
} proact_config;

/* Geometry of a registered region as seen by the calling rank. */
typedef struct proact_region_info {
    void *replica_base;      /* local full-extent replica (rank-ordered slice concatenation) */
    uint64_t own_offset;     /* byte offset of my owned slice inside the replica */
    uint64_t own_bytes;
    uint64_t total_bytes;    /* full extent */
    uint64_t chunk_bytes;
    uint32_t n_own_chunks;   /* chunks of my slice (last may be partial) */
    uint32_t n_total_chunks; /* over all ranks */
    uint32_t first_chunk;    /* global id of my first chunk */
    uint32_t generation;     /* completed write generations of this region */
    uint64_t dest_mask;
    uint64_t rank_offset[PROACT_MAX_RANKS + 1]; /* slice offsets, [world] = total */
} proact_region_info;

/* ================================================================ lifecycle ================= */

/* COLLECTIVE.  Bootstrap `ngpus` SPMD ranks (Listing 1 "ngpu = 4").
 * Rank = $PROACT_RANK, else $RANK (torchrun), else the current CUDA device.  Job key =
 * $PROACT_JOB, else "$MASTER_ADDR:$MASTER_PORT" (torchrun), else "default".  Rendezvous goes
 * through a job-keyed /dev/shm segment (no Python, no MPI).  Ranks on one device in one process
 * use direct pointers; ranks on distinct devices of one process enable peer access; ranks in
 * distinct processes map each other's memory with cudaIpcOpenMemHandle.  The calling thread's
 * current CUDA device is the rank's device.  Errors: INVALID (ngpus out of [1,16], rank out
 * of range), STATE (already initialised on this thread), TIMEOUT (peers never arrived), CUDA. */
int proact_init(int ngpus);
/* Same, with explicit rank and job key (for several ranks in one process, one per thread). */
int proact_init_ex(int ngpus, int rank, const char *job);
/* COLLECTIVE.  Drain (BARRIER), unmap peers, free library memory, leave the job. */
int proact_finalize(void);

int proact_rank(void);            /* -1 if not initialised */
int proact_world(void);
int proact_ranks_on_device(void); /* ranks sharing the calling rank's GPU (1 = dedicated) */

const char *proact_error_string(int code);
int proact_last_cuda_error(void); /* last cudaError_t seen by this thread's rank (0 = none) */

/* Tunables for subsequent launches of the calling rank; cfg==NULL restores defaults.  Env
 * overrides applied at init: PROACT_MECH, PROACT_AGENT_WARPS, PROACT_PIECE_BYTES,
 * PROACT_PUSH, PROACT_WATCHDOG_MS. */
int proact_set_config(const proact_config *cfg);
int proact_get_config(proact_config *cfg);

/* ================================================================ regions (a1) ============= */

/* COLLECTIVE.  Make [ptr, ptr+bytes) -- this rank's OWNED slice -- part of a new PROACT-enabled
 * region.  The slice lives inside a caller-allocated full-extent local replica whose layout is
 * the rank-ordered concatenation of all ranks' owned slices (1:1 correspondence, L123): rank p
 * owns [off_p, off_p + bytes_p), off_p = sum of bytes of ranks < p, so the replica base is
 * ptr - off_me and the mirror of my slice on peer p is base_p + off_me.  Chunks are numbered
 * from each slice's start in units of chunk_bytes (the last may be partial) and never straddle
 * owners.  dest_mask bit p = push my chunks to rank p (own bit ignored).  flags: PROACT_REGION_*.
 * Requirements: ptr, bytes, chunk_bytes multiples of 16; chunk_bytes >= 4096 (the paper's
 * smallest granularity, L279, L330) and equal on all ranks; bytes may be 0.  Returns the region
 * id (>= 0, same on all ranks) or INVALID / NOPEER / NOMEM / CUDA / TIMEOUT. */
int proact_register_region(void *ptr, size_t bytes, size_t chunk_bytes, uint64_t dest_mask);
int proact_register_region_ex(void *ptr, size_t bytes, size_t chunk_bytes, uint64_t dest_mask,
                              uint32_t flags);
/* Per-chunk destination override (e.g. Jacobi halo-only: push boundary chunks to neighbours
 * only).  chunk = index within MY slice.  Not collective; takes effect at the next launch.
 * When any chunk of a region has an override, proact::wait_all() is unavailable for it. */
int proact_region_set_chunk_dest(int region, uint32_t chunk, uint64_t mask);
int proact_region_info_get(int region, proact_region_info *out);
/* COLLECTIVE.  Change a region's chunk size (re-allocates its readiness table and flags; the
 * region's generation count is kept).  Used by the profiler to sweep granularity (L93, L112).
 * Must not race with an in-flight launch of the region (synchronise the stream first). */
int proact_region_rechunk(int region, size_t chunk_bytes);

/* ---- NVLS multicast replicas (PAPER.md L137 remote writes, L82 granularity) */
/* 1 if every rank of the job is a thread of this process on its own device and every device
 * supports switch multicast (CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED), else 0. */
int proact_mcast_supported(void);
/* COLLECTIVE.  Allocate a full-extent replica of `bytes` for this rank and return it in *ptr.  If
 * proact_mcast_supported() on every rank, the replicas of all ranks are bound to one multicast
 * object (cuMulticastCreate / AddDevice / BindMem; size rounded up to the multicast granularity)
 * and mapped for unicast access by every device of the job, so that regions registered inside it
 * can be pushed with PROACT_PUSH_MULTICAST; otherwise a plain device allocation.  The caller owns
 * the replica until proact_free_replica (COLLECTIVE), which must precede proact_finalize.
 * Errors: INVALID, STATE, NOMEM, CUDA, TIMEOUT. */
int proact_alloc_replica(size_t bytes, void **ptr);
int proact_free_replica(void *ptr);

/* ================================================================ launch / sync ============= */

/* Launch one producer phase writing `regions` (this launch's new generation of each).
 * `kernel` is a __global__ function whose FIRST parameter is `proact::launch_ctx` by value;
 * args[0] must point to storage for it, which this call fills (epoch, armed regions,
 * generations, mechanism).  grid = producer CTAs wanted (0 = fill the rank's device share);
 * under FUSED/ELIDE the library prepends agent CTAs and clamps the total to the co-resident
 * capacity (cooperative launch on a dedicated GPU), so producer kernels must loop over their
 * tiles with proact::producer_block()/producer_grid().  block = threads per CTA (0 = config).
 * Asynchronous on `stream` (a cudaStream_t); device errors surface at the next sync.
 * INVALID if a region id is unknown or the producer share would be empty. */
int proact_launch(const int *regions, int nregions, const void *kernel, unsigned grid,
                  unsigned block, void **args, size_t smem, void *stream);

/* As proact_launch; `flags` = PROACT_LAUNCH_* capabilities of `kernel`. */
int proact_launch_ex(const int *regions, int nregions, const void *kernel, unsigned grid,
                     unsigned block, void **args, size_t smem, void *stream, unsigned flags);

/* 1 if the next proact_launch of this rank will run tallies and the agent (FUSED with G > 1, or
 * ELIDE), 0 if not (LOCAL / INLINE / BULK, or FUSED on a single rank): lets a workload pick a
 * kernel instantiation without the tally machinery. */
int proact_launch_tallies(void);
/* What the next launch of a kernel that supports PROACT_LAUNCH_TILE_PUSH should instantiate:
 * 0 = plain stores (no tallies), 1 = tallies for a polling agent (FUSED / SEPARATE / ELIDE / DMA),
 * 2 = tile push (PROACT_AGENT_PRODUCER: the kernel's transfer warp pushes its own tiles; launch
 * it with PROACT_LAUNCH_TILE_PUSH). */
int proact_launch_mode(void);

/* Close phase e on `stream` (a8): peers get the credit "rank finished phase e" (write-after-read
 * guard for ping-pong replicas, reading R6), a BULK launch's copies are issued first, and in
 * BARRIER mode the stream also waits for every peer's credit (L125).  Then the rank's epoch
 * advances.  Returns any latched device error (non-blocking check). */
int proact_phase_sync(void *stream, int mode);

/* Global OR of the votes (proact::vote) cast by all ranks in the most recent BARRIER phase,
 * read after the stream is synchronised: 1 = some rank voted.  -1 if not available. */
int proact_last_vote(void);

/* Debug (PROACT_DEBUG=1 at init): copy region `region`'s per-(my chunk, dest) delivery counters
 * (n_own_chunks * world uint32, row-major) to host memory `out` and zero them.  Synchronises
 * the device.  INVALID if debug counters are off or n is too small. */
int proact_region_debug_deliveries(int region, uint32_t *out, size_t n);

/* Debug: protocol state of region `region` as this rank sees it, for post-mortems after a
 * watchdog timeout.  Synchronises the device.  Writes n_own counters, n_own expected, n_own
 * piece counts, n_total arrival flags, 8 queue-control words, 16 credits (done[]) and 16 host
 * words ([0] epoch, [1] generations launched) to `out` (uint32).  INVALID if n is too small. */
int proact_region_debug_state(int region, uint32_t *out, size_t n);

/* Debug (PROACT_DEBUG=2 at init): agent cycle accounting since the last call, 8 counters:
 * [0] discovery-wait cycles, [1] batch-processing cycles, [2] batches, [3] units,
 * [4] TMA push-pipeline cycles, [5] store-drain cycles.  Synchronises the device; resets. */
int proact_debug_agent_prof(unsigned long long *out8);

/* COLLECTIVE host-side barrier of all ranks (no device work): e.g. to read replicas from the
 * host between phases without a peer's next phase overwriting them. */
int proact_host_barrier(void);

/* ---- host-only helpers (no CUDA; also used internally, exposed for tests) --------------- */
/* Slice plan of a region: rank_off[0..world] (prefix sums of bytes[]) and rank_chunk0[0..world]
 * (global id of each rank's first chunk; a rank's chunks are ceil(bytes/chunk_bytes)). */
int proact_plan_slices(int world, const uint64_t *bytes, uint64_t chunk_bytes, uint64_t *rank_off,
                       uint32_t *rank_chunk0);
/* All-gather of n bytes (<= 4096) per rank through the job-keyed /dev/shm rendezvous that
 * proact_init uses (COLLECTIVE over `world` callers with distinct ranks). */
int proact_rdv_allgather(const char *job, int world, int rank, const void *mine, size_t n, void *all);

/* Non-blocking check of the device error word. */
int proact_check(void);
/* Kernels launched by this rank so far (producer/agent grids, sync kernels, helper kernels). */
uint64_t proact_launch_count(void);
uint32_t proact_epoch(void);

/* ================================================================ profiler (a9) ============= */

/* One profiling run: execute a few phases with `cfg` applied and return the measured time in
 * ms (< 0 on failure).  Called on every rank with identical cfg sequences. */
typedef double (*proact_run_fn)(const proact_config *cfg, void *user);

/* COLLECTIVE.  Brute-force sweep (Sec. III-A): mechanism x piece/chunk x
 * agent warps, per `key`; each point's time is the max over ranks; best config returned in
 * *out and cached as JSON in $PROACT_TUNE_CACHE (default ./proact_tune.json) under `key` --
 * a cached key is returned without re-running.  `space` may be NULL (default space: mechanisms
 * FUSED/INLINE/BULK x agent warps 8..64 at the current chunk, piece, push, discovery and agent
 * placement) or a NUL-terminated list such as
 * "mech=0,1,2,5;chunk=65536,1048576;warps=8,32;piece=65536;push=0,1;disc=0,1;akern=0,1". */
int proact_autotune(const char *key, const char *space, proact_run_fn fn, void *user,
                    proact_config *out);

#ifdef __cplusplus
}
#endif
#endif /* PROACT_H */
