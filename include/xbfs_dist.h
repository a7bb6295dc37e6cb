/*
 * xbfs_dist.h — multi-GPU XBFS: 1D vertex partition, one process per GPU
 * (north_star: "for 2, 4 and 8 GPUs the graph is
 * 1D-partitioned by vertex ... with the direction switch made on globally
 * reduced counts").  The paper runs a single GCD and presents itself as
 * the basis for distributed BFS; the exchange below is this build's.
 *
 * Partition: rank r owns vertices [r*B, min(N, (r+1)*B)), B = 32*ceil(N/(32p)),
 * with the full adjacency row (global neighbour ids) of every owned vertex.
 * Replicated per rank: three N-bit frontier bitmaps (F_k, F_{k+1}, stale).
 * Per level k (the strategy is identical on every rank, chosen from the
 * all-reduced counters by the paper's rule):
 *   BU  phase 0: owned unvisited vertices probe their neighbours in the local
 *       replica of F_k; the owned words of F_{k+1} are stored straight into every
 *       peer's replica (peer memory over NVLink/NVSwitch, CUDA IPC): the
 *       all-gather is fused into the producing kernel.
 *   TD  phase 0: owned frontier vertices expand their rows; an owned neighbour is
 *       claimed locally, a remote one is OR-ed into its owner's inbox bitmap in
 *       peer memory (fire-and-forget RED).  phase 1 (after a barrier): each owner
 *       turns inbox ∧ ¬visited into new frontier vertices, finds each one's parent
 *       with a bottom-up probe against F_k, and stores its owned F_{k+1} words
 *       into every peer's replica.
 * Host barriers and the 4-counter all-reduce between phases are the caller's
 * (torch.distributed), see paper_conf_sc_yangls0w24_b200/xbfs.py DistGraph.
 *
 * Conventions as in xbfs.h (status codes, thread-local error, poisoning).
 */
#ifndef XBFS_DIST_H
#define XBFS_DIST_H

#include <stdint.h>

#include "xbfs.h"

#ifdef __cplusplus
extern "C" {
#endif

#define XBFS_IPC_HANDLE_BYTES 64
#define XBFS_DIST_MAX_RANKS 16
#define XBFS_DIST_NCOUNTS 8   /* length of every counts[] array below */

typedef struct xbfs_dist xbfs_dist;

/* Build rank `rank`'s partition.  Every rank passes the SAME full tuple list
 * (src, dst: num_edges ids of width opts->id_bytes, host or device per opts);
 * the rank keeps the arcs whose source it owns (both directions of every tuple,
 * self-loops and duplicates dropped, rows id-sorted) and re-arranges its rows by
 * neighbour degree, descending, where the degree of a remote
 * neighbour is its tuple-incidence count (reading R-6 in DESIGN.md).
 * Errors: INVALID_ARG (nranks outside [1, XBFS_DIST_MAX_RANKS], rank outside
 * [0, nranks), plus xbfs_build_csr's), OUT_OF_MEMORY, CUDA. */
xbfs_status xbfs_dist_build(const void* src, const void* dst, int64_t num_edges, int64_t num_vertices,
                            int32_t nranks, int32_t rank, const xbfs_build_opts* opts, xbfs_dist** out);

/* Owned range and sizes.  Any out pointer may be NULL. */
xbfs_status xbfs_dist_info(const xbfs_dist* d, int64_t* first, int64_t* count, int64_t* local_arcs,
                           int64_t* num_vertices);

/* IPC handle (XBFS_IPC_HANDLE_BYTES bytes) of this rank's shared region (the
 * three frontier replicas + the inbox); exchange it with every rank. */
xbfs_status xbfs_dist_export(xbfs_dist* d, void* handle_out);

/* Map the peers' shared regions.  handles: nranks * XBFS_IPC_HANDLE_BYTES in
 * rank order (this rank's own entry is ignored).  Call once, after every rank
 * exported; peers may be other GPUs (NVLink P2P) or the same GPU (tests). */
xbfs_status xbfs_dist_attach(xbfs_dist* d, const void* handles);

/* Start a BFS from global vertex `source`: resets this rank's state and writes
 * every element of the caller-owned DEVICE arrays level_local[count] and
 * parent_local[count] (parent values are global ids).  counts[] receives this
 * rank's {owns source, deg(source), tuples of source, non-isolated owned
 * vertices, local arcs, 0, 0, 0}; all-reduce them (sum) and pass the result to
 * xbfs_dist_advance, which also acts as the barrier before the first level. */
xbfs_status xbfs_dist_begin(xbfs_dist* d, int64_t source, int32_t* level_local, int32_t* parent_local,
                            const xbfs_run_opts* opts, int64_t counts[XBFS_DIST_NCOUNTS]);

/* Run phase 0 or 1 of the current level on this rank and synchronise its
 * stream.  After the level's last phase (phase 0 for BU, phase 1 for TD)
 * counts[] = this rank's {new frontier vertices, their degree sum, their tuple
 * count (Graph500 m), arcs probed by BU, 0...}; zeros otherwise.  A caller
 * barrier must separate phase 0 and phase 1 of a TD level; the all-reduce of
 * the counts separates levels. */
xbfs_status xbfs_dist_level(xbfs_dist* d, int32_t phase, int64_t counts[XBFS_DIST_NCOUNTS]);

/* Apply the all-reduced counters (identical on every rank) and choose the next
 * level's strategy.  *done = 1 when the next frontier is empty. */
xbfs_status xbfs_dist_advance(xbfs_dist* d, const int64_t global_counts[XBFS_DIST_NCOUNTS],
                              int32_t* strategy_out, int32_t* done);

/* Per-level log of the last BFS (host arrays of cap entries, NULL to skip);
 * *num_levels = number of levels, *input_edges = Graph500 m (O-6) over all
 * ranks.  Any out pointer may be NULL. */
xbfs_status xbfs_dist_levels(const xbfs_dist* d, int32_t cap, int8_t* strategy, int64_t* frontier_vertices,
                             int64_t* frontier_edges, int32_t* num_levels, int64_t* input_edges);

/* NULL-safe. */
void xbfs_dist_destroy(xbfs_dist* d);

#ifdef __cplusplus
}
#endif
#endif /* XBFS_DIST_H */
