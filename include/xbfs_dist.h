/*
 * xbfs_dist.h — multi-GPU XBFS: 1D vertex partition, one process per GPU on one
 * node (SURVEY §8(a) row a11, §8(b) multi-GPU calls, §8(e); north_star: "for 2, 4
 * and 8 GPUs the graph is 1D-partitioned by vertex ... with the direction switch
 * made on globally reduced counts").  The paper runs a single GCD and
 * presents itself as the basis for distributed BFS; the exchange below is
 * this build's (reading R-10 in DESIGN.md).
 *
 * Partition: rank r owns vertices [r*B, min(N, (r+1)*B)), B = 32*ceil(N/(32p)),
 * with the full adjacency row (global neighbour ids) of every owned vertex, rows
 * re-arranged by neighbour degree descending, ties id ascending (C-12) —
 * the true degrees, so every row is the single-GPU xbfs_reorder row.
 * Replicated per rank: three N-bit frontier bitmaps (F_k, F_{k+1}, stale).
 * Per level k (the strategy is identical on every rank: the paper's rule, P:L87,
 * on the all-reduced counters):
 *   BU  owned unvisited vertices probe their rows against the local replica of
 *       F_k; the owned words of F_{k+1} are stored straight into every peer's
 *       replica (peer memory over NVLink/NVSwitch, CUDA IPC): the all-gather is
 *       fused into the producing kernel.
 *   TD  owned frontier vertices expand their rows; an owned neighbour is claimed
 *       locally, a remote one is OR-ed into its owner's inbox bitmap in peer memory
 *       (fire-and-forget RED); after a barrier each owner turns inbox ∧ ¬visited
 *       into new frontier vertices, gives each the first vertex of its row in F_k
 *       as parent, and stores its owned F_{k+1} words into every replica.
 * The level loop, the barriers and the counter all-reduce run inside
 * xbfs_run_dist (one C call per BFS); the host collectives use the communicator
 * below (a shared-memory segment on the node, no NCCL: reading R-10).
 *
 * Conventions as in xbfs.h (status codes, thread-local error, handle poisoning;
 * every call here is collective unless marked local).
 */
#ifndef XBFS_DIST_H
#define XBFS_DIST_H

#include <stdint.h>

#include "xbfs.h"

#ifdef __cplusplus
extern "C" {
#endif

#define XBFS_UNIQUE_ID_BYTES 128
#define XBFS_DIST_MAX_RANKS 16

typedef struct xbfs_comm xbfs_comm;

/* Local.  A fresh communicator id (128 bytes, the analogue of an ncclUniqueId):
 * rank 0 calls it and broadcasts the bytes to the other ranks (torch.distributed).
 * Errors: INVALID_ARG (NULL). */
xbfs_status xbfs_get_unique_id(uint8_t id[XBFS_UNIQUE_ID_BYTES]);

/* Collective over the nranks processes of one node.  rank 0 creates the shared
 * segment named in `id`, the others attach to it (waiting up to 600 s).  Makes
 * no CUDA call.  Errors: INVALID_ARG (NULL, not an xbfs id, rank outside
 * [0, nranks), nranks outside [1, XBFS_DIST_MAX_RANKS], nranks differing from
 * rank 0's), STATE (segment could not be created / a peer never arrived). */
xbfs_status xbfs_comm_init(const uint8_t id[XBFS_UNIQUE_ID_BYTES], int32_t nranks, int32_t rank, xbfs_comm** out);

/* Collective host-side barrier and int64 sum all-reduce (count <= 512) of the
 * communicator (used inside xbfs_run_dist; exported for the caller's harness and
 * the CPU tests).  Errors: INVALID_ARG, STATE (a peer did not arrive in 600 s). */
xbfs_status xbfs_comm_barrier(xbfs_comm* c);
xbfs_status xbfs_comm_allreduce_i64(xbfs_comm* c, const int64_t* in, int64_t* out, int32_t count);

/* Collective.  Build this rank's partition from ITS OWN share of the input tuples:
 * src/dst hold local_edges ids (width opts->id_bytes; host or device per opts),
 * any split of the M tuples over the ranks (e.g. rank r generates tuples
 * [r*M/p, (r+1)*M/p)).  The library ships every arc (both directions of each
 * tuple) to the owner of its source over peer memory (counts all-gathered first),
 * then each owner sorts, drops self-loops and duplicates (C-3), builds its rows
 * and records per-vertex tuple counts (Graph500 m, O-6); the owned degrees are
 * all-gathered and every row is re-arranged as xbfs_reorder mode 1 does.  The
 * handle runs only with xbfs_run_dist and is freed with xbfs_destroy (local).
 * opts->directed is unsupported (UNSUPPORTED).  Errors: INVALID_ARG (NULL, N out
 * of (0, 2^31), ids >= N on any rank), OUT_OF_MEMORY, CUDA, STATE (comm). */
xbfs_status xbfs_build_csr_dist(xbfs_comm* c, const void* src, const void* dst, int64_t local_edges,
                                int64_t num_vertices, const xbfs_build_opts* opts, xbfs_graph** out);

/* Local.  This rank's owned vertex range [*first, *first + *count). */
xbfs_status xbfs_partition_range(const xbfs_graph* g, int64_t* first, int64_t* count);

/* Collective.  One BFS from global vertex `source`, every level of it:
 * writes every element of the caller-owned DEVICE arrays level_local[count] and
 * parent_local[count] (parent values are global ids; -1 if unreached; semantics
 * of xbfs_run).  opts: strategy parameters as xbfs_run (driver, plan, small_edges,
 * lookahead are ignored).  stats (may be NULL; then the call still synchronises,
 * as the level loop is host-driven): elapsed_ms = this rank's device time from
 * init to the end of the last level (CUDA events; take the max over ranks),
 * num_levels, vertices_reached, arcs_traversed, input_edges_traversed = GLOBAL
 * values, and the per-level arrays (strategy, frontier_vertices, frontier_edges,
 * unvisited, bu_probes) of global counts.  Errors: INVALID_ARG (source outside
 * [0, N), NULL outputs with count > 0), STATE, CUDA. */
xbfs_status xbfs_run_dist(xbfs_graph* g, int64_t source, int32_t* level_local, int32_t* parent_local,
                          const xbfs_run_opts* opts, xbfs_run_stats* stats);

/* Local.  Frees the communicator (NULL-safe); destroy the graphs built on it first. */
void xbfs_comm_destroy(xbfs_comm* c);

#ifdef __cplusplus
}
#endif
#endif /* XBFS_DIST_H */
