/*
 * proact_workloads.h -- C entry points of the producer kernels on the PROACT hot path.
 *
 * Each *_phase call launches ONE producer phase through proact_launch (include/proact.h): it
 * writes the next generation of its output region(s) under the rank's configured mechanism
 * (FUSED agent / INLINE / BULK / LOCAL / ELIDE).  The caller closes the phase with
 * proact_phase_sync().  Regions are the caller's registered replicas; all calls are
 * asynchronous on `stream` (a cudaStream_t) and return PROACT_OK or a PROACT_ERR_* code.
 */
#ifndef PROACT_WORKLOADS_H
#define PROACT_WORKLOADS_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct proact_jacobi_params {
    int region_in, region_out;
    long long N, row0, nrows;
    int rows_per_tile, pad;
} proact_jacobi_params;

typedef struct proact_micro_params {
    int region;
    unsigned phase, seed;
    int K, scattered;
    int verify_region;        /* litmus: region whose current generation must hold phase-1 tags, or -1 */
    unsigned *bad;            /* litmus: device counter of stale / wrong words seen (or NULL) */
} proact_micro_params;

/* Jacobi, 2D 5-point stencil (Sec. IV-C; BASELINE.json configs 1-2; DESIGN.md
 * readings R9/R10).  region_in / region_out: two registered N x N fp32 row-major replicas with
 * identical geometry whose owned slices are whole rows (rank g owns rows
 * [own_offset/(4N), (own_offset+own_bytes)/(4N))).  Reads generation k of region_in (waiting on
 * the neighbours' boundary rows), writes generation k+1 of my rows of region_out:
 * x'[i][j] = 0.25f*((x[i-1][j]+x[i+1][j]) + (x[i][j-1]+x[i][j+1])) in fp32 round-to-nearest
 * without contraction; boundary cells (i or j in {0, N-1}) copied through.  N must be a multiple
 * of 4.  rows_per_tile: band height of a tile (0 = 16); a tile is rows_per_tile x 1024 columns.
 * INVALID on geometry mismatch. */
int proact_jacobi_phase(int region_in, int region_out, long long N, int rows_per_tile, void *stream);

/* Transfer microbenchmark producer (Sec. IV-C, Sec. V-A; reading R14).
 * Writes word k (global word index within the region) of my slice as
 * v = fmix32(k ^ (phase * 0x9E3779B9) ^ seed), then K-1 more fmix32 (MurmurHash3 finaliser).
 * One CTA pass per 4 KiB tile; scattered != 0 permutes the store order inside each tile
 * (position (j*389) mod 1024), which only matters for INLINE (store coalescing, L143, L318). */
int proact_micro_phase(int region, unsigned phase, unsigned seed, int K, int scattered, void *stream);

/* Protocol litmus ("no later than the succeeding global
 * synchronization barrier", L145 visibility): a microbenchmark phase that is also a CONSUMER.
 * Before producing, every CTA waits (proact::wait_range, i.e. the arrival flags or credits of the
 * mechanism that produced it) for the whole current generation of region_in, then checks every
 * word of it against its phase tag -- word k must equal the microbenchmark value of phase
 * `phase - 1` (K = 1) -- and adds the number of words that differ (stale or torn) to *d_bad
 * (device memory, uint32).  It then writes phase `phase` of region_out exactly like
 * proact_micro_phase (K = 1, dense).  region_in / region_out: two registered regions of equal
 * geometry (ping-pong).  phase 0 skips the check. */
int proact_litmus_phase(int region_in, int region_out, unsigned phase, unsigned seed, unsigned *d_bad,
                        void *stream);

/* Fault injection (tests): one launch on `region` whose first producer CTA commits the bytes of my
 * chunk 0 twice, as a producer with a non-deterministic store count would (PAPER.md L129:
 * "a deterministic number of stores" is required).  Under a tallying mechanism (FUSED / ELIDE
 * with G > 1, or DMA) the over-count is detected on the device: the next proact_phase_sync /
 * proact_check returns PROACT_ERR_PROTOCOL (site: commit).  Other chunks are not written. */
int proact_inject_double_commit(int region, void *stream);

/* End-to-end Jacobi through host buffers (the bench's "e2e" path).  COLLECTIVE over the world.
 * h_x0: the full N x N initial grid in host memory (pinned for async copies); h_out: receives
 * this rank's owned rows (row-partitioned like proact_jacobi_phase, rows split as evenly as
 * possible, rank g gets rows [g*N/G, (g+1)*N/G)) at their full-grid position.  Runs `iters`
 * phases with PROACT_SYNC_SIGNAL, BARRIER on the last.  The library allocates (and caches for
 * the next call with the same N and chunk_bytes) the two replicas and registers them, so the
 * first call registers two regions.  Copies in: the full grid (every replica starts identical,
 * reading R16); out: the owned rows.  *bytes_h2d / *bytes_d2h (may be NULL) get the counts. */
int proact_jacobi_solve_host(const float *h_x0, float *h_out, long long N, int iters,
                             size_t chunk_bytes, int rows_per_tile, void *stream,
                             unsigned long long *bytes_h2d, unsigned long long *bytes_d2h);

/* nsolve independent end-to-end solves of the same host input, pipelined (the bench's e2e
 * path): each solve copies h_x0 in (full grid), runs `iters` phases (BARRIER on the last) and
 * copies this rank's rows of its result out to h_outs[k] (nsolve host pointers, pinned), like
 * proact_jacobi_solve_host.  Two library-owned device buffer sets (4 registered regions on the
 * first call), an unregistered H2D staging buffer (moved into the set by a device copy at the
 * start of each solve) and two library copy streams let solve k's phases overlap the H2D of
 * solve k+1 and the D2H of solve k-1, the two copies running at the same time.  Asynchronous: everything is complete when `stream` is.  COLLECTIVE.
 * *bytes_h2d / *bytes_d2h get the per-solve counts. */
int proact_jacobi_solve_host_pipelined(const float *h_x0, float *const *h_outs, int nsolve, long long N,
                                       int iters, size_t chunk_bytes, int rows_per_tile, void *stream,
                                       unsigned long long *bytes_h2d, unsigned long long *bytes_d2h);

/* ---- banded-matrix Jacobi (Sec. IV-C: the paper's own Jacobi) */
typedef struct proact_banded_params {
    int region_in, region_out;
    long long N, w, row0, nrows;
    const float *a;    /* device, DIA layout (2w+1) x N: a[(o+w)*N + i] = A[i][i+o] */
    const float *b;    /* device, N */
} proact_banded_params;

/* One Jacobi sweep of A x = b for my rows (reading R19): x'[i] = (b[i] - sum_{o != 0} A[i][i+o]
 * x[i+o]) / A[i][i], the sum in fp32 in the order o = -w..w, each product rounded before the
 * add, IEEE division.  region_in / region_out: two registered N-float replicas with identical
 * whole-row slices (rank g owns rows [own_offset/4, (own_offset+own_bytes)/4)); a / b: device
 * arrays of the full system (only my rows are read).  Waits for the peers' rows within w of my
 * slice.  w <= 8192.  INVALID on geometry mismatch.  With w <= 4096 and 16-byte aligned a / b
 * the TMA-fed banded_tma_kernel runs (bulk copies of contiguous diagonal slices), otherwise
 * banded_kernel; both give the same bits. */
int proact_banded_phase(int region_in, int region_out, const float *a, const float *b, long long N,
                        long long w, void *stream);

/* ---- graph workloads (Sec. IV-C L265 PageRank, L267 SSSP; configs 3-4) --------- */

/* Destination partition of a graph for G ranks: bounds[0..G] (host array of G+1) receive vertex
 * boundaries, multiples of `align` vertices (use chunk_bytes/4 so that every rank's slice of a
 * replicated 4-byte vertex vector starts on a chunk boundary), chosen so that in-edge counts are
 * as even as possible.  d_dst: device array of E destination ids.  Synchronises `stream`. */
int proact_graph_partition(const uint32_t *d_dst, unsigned long long E, unsigned V, int G, unsigned align,
                           unsigned *bounds, void *stream);

/* Host-only core of proact_graph_partition: bounds from an in-degree histogram (V entries). */
int proact_partition_bounds(const uint32_t *indeg, unsigned V, int G, unsigned align, unsigned *bounds);

/* Build this rank's in-edge CSC for destinations [v0, v1) from a device edge list (d_src,
 * d_dst, optional d_w weights, E edges, V vertices; self loops allowed, duplicates kept) plus the
 * global out-degree.  Library-owned device memory; returns a graph id >= 0 (NOMEM if 4 graphs
 * exist).  The edge list may be freed afterwards.  Synchronises `stream`. */
int proact_graph_build(const uint32_t *d_src, const uint32_t *d_dst, const int32_t *d_w,
                       unsigned long long E, unsigned V, unsigned v0, unsigned v1, void *stream);
/* As proact_graph_build, plus the PageRank hot-source table: the `hot` vertices with the
 * highest global out-degree (ties: smaller id; only vertices with out-edges; at most 45056) are
 * staged in shared memory by every pagerank phase CTA and their in-edges read the table instead of
 * the replica.  hot = 0: no table; hot < 0: env PROACT_GRAPH_HOT, else 8192 (two CTAs per SM).
 * The result is bit-identical either way (exact fixed-point sums).  V < 2^31. */
int proact_graph_build_ex(const uint32_t *d_src, const uint32_t *d_dst, const int32_t *d_w,
                          unsigned long long E, unsigned V, unsigned v0, unsigned v1, int hot, void *stream);
/* Number of hot sources of a graph (0: none) and of my in-edges whose source is hot (either
 * pointer may be NULL). */
int proact_graph_hot(int graph, unsigned *nhot, unsigned long long *e_hot);
int proact_graph_free(int graph);
int proact_graph_info(int graph, unsigned long long *e_own, unsigned *v0, unsigned *nv);

/* PageRank (readings R11/R12).  The replicated region holds contrib[u] = r[u]/out(u) (fp32, 0
 * for dangling u) over all V vertices; its owned slice must be [4*v0, 4*v1).  init writes
 * contrib^0 = fp32(1/V)/out(u) into the WHOLE local replica (identical on every rank).  A phase
 * computes, for my vertices, r'[v] = (float)((1-d)/V + d * sum_{u->v} contrib[u]) with an fp64
 * sum, keeps r' locally and writes contrib'[v] = r'[v]/out(v) into region_out.
 * pagerank_ranks copies my r' (nv floats) to device memory d_out. */
int proact_pagerank_init(int graph, int region, void *stream);
int proact_pagerank_phase(int graph, int region_in, int region_out, double damping, void *stream);
int proact_pagerank_ranks(int graph, float *d_out, void *stream);

/* SSSP, synchronous Bellman-Ford round (reading R13): for my vertices
 * d'[v] = min(d[v], min_{u->v, d[u] != INT32_MAX} d[u] + w), int32, relaxing only sources whose
 * chunk changed in the previous round (all of them when first != 0).  Regions should be
 * registered with PROACT_REGION_SPARSE and chunk_bytes a multiple of 4096.  A round that
 * changes anything casts a proact::vote (read it with a BARRIER phase_sync + proact_last_vote). */
int proact_sssp_phase(int graph, int region_in, int region_out, int first, void *stream);
/* (Same call.)  Weighted graphs also hold my in-edges grouped by source, and each round is either
 * a PULL round (above) or a PUSH round (reading R24, PAPER.md L267's Bellman-Ford with only the
 * sources whose distance changed in the previous round relaxing their edges into my vertices,
 * atomicMin into a private array; identical d').  The choice is made per rank from the out-degree
 * of the vertices this rank changed in the previous round (copied to the host after that round's
 * kernel: call after synchronising with it for a current decision); env PROACT_SSSP_PUSH = 0 / 1
 * forces pull / push, PROACT_SSSP_PUSH_PCT (default 8) is the frontier share of the edges below
 * which a round pushes.  Every rank keeps a private copy of the previous round's input (V ints),
 * refreshed by push rounds and by pull rounds whose frontier is below 4x that share (a round
 * pushes only after a round that refreshed it). */
/* Mode of the graph's last launched SSSP round: 0 pull, 1 push; PROACT_ERR_INVALID for a bad id. */
int proact_sssp_last_mode(int graph);

#ifdef __cplusplus
}
#endif
#endif /* PROACT_WORKLOADS_H */
