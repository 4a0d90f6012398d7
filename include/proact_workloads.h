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
    int K, scattered, pad;
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

#ifdef __cplusplus
}
#endif
#endif /* PROACT_WORKLOADS_H */
