/*
 * xbfs.h — C ABI of the B200-native XBFS library (libxbfs.so, sm_100a).
 *
 * Adaptive level-synchronous BFS over a symmetric CSR graph, after
 * "Establish the basis for Breadth-First Search on Frontier System: XBFS on
 * AMD GPUs" (SC'24 workshops; PAPER.md = "P", cited by line).  Each level is
 * expanded by one of three frontier strategies (§III):
 *   0 SF  scan-free top-down    (§III-A)
 *   1 SS  single-scan top-down  (§III-B, incl. No-Frontier-Generation)
 *   2 BU  bottom-up             (§III-C)
 * chosen from ratio_k = edgesF_k / |M| against alpha (alpha = 0.1 P:L347)
 * and the growth of |F| (reading C-10).  Neighbour lists are
 * re-arranged by degree (§IV-B) by xbfs_reorder.
 *
 * Conventions (all entry points):
 *   - extern "C", no exceptions cross the boundary; every call returns an
 *     xbfs_status.  On failure xbfs_last_error() returns a thread-local message.
 *   - A CUDA / NCCL failure poisons the handle: later calls on it return
 *     XBFS_ERR_STATE.  Invalid arguments never poison and write nothing.
 *   - Vertex ids are int32 in [0, N), N < 2^31; edge offsets are int64
 *     (the paper's 8-byte edge / 4-byte vertex indices).
 *   - The handle owns every device buffer it allocates (CSR, bitmaps, queues,
 *     counters); xbfs_destroy frees them.  Output arrays are caller-owned.
 *   - Work is enqueued on the handle's stream (xbfs_build_opts.stream);
 *     xbfs_run with stats == NULL returns without synchronising.
 *   - A handle is not thread-safe; distinct handles are independent.
 */
#ifndef XBFS_H
#define XBFS_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    XBFS_OK = 0,
    XBFS_ERR_INVALID_ARG = 1,   /* null pointer, N out of range, id out of range, bad source */
    XBFS_ERR_OUT_OF_MEMORY = 2, /* cudaMalloc / host allocation failed */
    XBFS_ERR_CUDA = 3,          /* CUDA runtime error (handle poisoned) */
    XBFS_ERR_NCCL = 4,          /* NCCL error (handle poisoned) */
    XBFS_ERR_STATE = 5,         /* handle poisoned by an earlier failure, or wrong mode */
    XBFS_ERR_UNSUPPORTED = 6    /* feature not built / not available */
} xbfs_status;

enum { XBFS_SF = 0, XBFS_SS = 1, XBFS_BU = 2 };

typedef struct xbfs_graph xbfs_graph;

/* Options for xbfs_build_csr.  Zero-initialised means: device 0 (current),
 * default stream, uint32 ids, host-resident edges, dedup on. */
typedef struct {
    int32_t device;          /* CUDA device ordinal the handle lives on (-1 = current) */
    int32_t id_bytes;        /* width of src/dst elements: 4 (uint32) or 8 (int64); 0 = 4 */
    void* stream;            /* cudaStream_t for all work of this handle; NULL = legacy default */
    int32_t edges_on_device; /* 1: src/dst are device pointers; 0: host pointers */
    int32_t keep_duplicates; /* 0 (default): drop duplicate arcs (reading C-3) */
    int32_t directed;        /* 1: tuple (i,j) is the arc i -> j only (reading R-9): top-down
                                steps follow out-arcs, bottom-up steps search in-arcs (a second, transposed
                                CSR), BU candidates are vertices with in-degree > 0.  Runs on the persistent
                                driver only (driver 0/3, no look-ahead); 0 (default): symmetric graph */
} xbfs_build_opts;

/* Options for xbfs_run.  xbfs_run_opts_default() fills the paper's values. */
typedef struct {
    double alpha;            /* BU iff edgesF_k / A > alpha; the paper uses 0.1 (MI250X);
                                default 0.04, re-tuned on B200 (reading C-13) */
    double grow;             /* SS iff |F_k| > grow * |F_{k-1}| and ratio > ratio_min (C-10) */
    double ratio_min;        /*   "                                                    */
    double bu_stay;          /* >0: stay BU while |U_k| * bu_stay < edgesF_k (C-11); default 1.0, 0 = paper rule */
    int32_t force_strategy;  /* -1 adaptive; 0 SF, 1 SS, 2 BU on every level (tests, Fig 7 sweep) */
    int32_t driver;          /* 0 auto (= 3), 1 host loop (one sync per level), 2 CUDA-graph device
                                loop, 3 persistent kernel (one cooperative launch per BFS, grid
                                barriers between levels).  Per-launch profiling and plans always
                                use the host loop. */
    int32_t small_edges;     /* SF levels with edgesF_k <= this run inside one thread-block cluster
                                (small-frontier mode); default 65536, 0 = off, max 73728 */
    int32_t plan_len;        /* > 0: strategy plan for levels [0, plan_len) (host-loop driver only) */
    const int8_t* plan;      /* host array: plan[k] in {-1 selector, 0 SF, 1 SS, 2 BU} overrides the
                                strategy of level k (forced-strategy studies, Tab VI) */
    int32_t lookahead;       /* 1: bottom-up look-ahead ("proactive") update, SURVEY f1:
                                a BU step also sets to level k+2 every candidate whose whole row has
                                no F_k vertex but a vertex this same pass already put in F_{k+1}.
                                Levels stay exact; parents of those vertices are that neighbour.
                                Persistent driver only (driver 0 / 3, no plan, no per-launch
                                profiling): XBFS_ERR_INVALID_ARG otherwise.  Default 0. */
} xbfs_run_opts;

/* Per-run statistics; filled when a non-NULL pointer is passed (xbfs_run then
 * synchronises its stream).  The per-level arrays are optional caller-owned
 * HOST arrays of level_capacity entries (NULL to skip). */
typedef struct {
    float elapsed_ms;              /* device time from init to the last level (CUDA events) */
    int32_t num_levels;            /* max level + 1 */
    int64_t vertices_reached;      /* sum_k |F_k| */
    int64_t arcs_traversed;        /* sum_k edgesF_k = sum of deg over reached (paper TEPS numerator, C-4) */
    int64_t input_edges_traversed; /* Graph500 m = sum of tuple counts over reached (O-6) */
    uint32_t kernel_launches;      /* library kernels launched by this run (device-counted) */
    int32_t level_capacity;
    int8_t* strategy;              /* [level_capacity] strategy used at level k */
    int64_t* frontier_vertices;    /* |F_k| */
    int64_t* frontier_edges;       /* edgesF_k */
    int64_t* unvisited;            /* |U_k| non-isolated unvisited before step k */
    int64_t* bu_probes;            /* arcs probed by BU at level k (0 for TD levels) */
    /* Per-launch timing (measurement only): when kernel_capacity > 0 the host-loop
     * driver brackets every kernel with CUDA events on the handle's stream and
     * fills up to kernel_capacity entries (caller-owned host arrays). */
    int32_t kernel_capacity;       /* at most 4096 launches are recorded (event pool made at build time) */
    int32_t num_kernels;           /* launches recorded */
    int32_t* kernel_id;            /* XBFS_K_* */
    int32_t* kernel_level;         /* level k the launch belongs to (-1 = init) */
    float* kernel_ms;              /* event-timed duration */
    /* [level_capacity] device time of level k in ms (persistent driver: %globaltimer
     * stamps at the grid barrier ending each level; 0 under the other drivers) */
    float* level_ms;
    /* [level_capacity] vertices step k set to level k+2 through the BU look-ahead (0 if off) */
    int64_t* lookahead_found;
    /* persistent driver: device time (%globaltimer) from the kernel's first CTA entry to the end of
     * the per-BFS init + seed phase; 0 under the other drivers */
    float init_ms;
} xbfs_run_stats;

/* kernel ids reported in xbfs_run_stats.kernel_id */
enum { XBFS_K_INIT = 0, XBFS_K_SEED = 1, XBFS_K_GENERATE_PRE = 2, XBFS_K_TD_SF = 3, XBFS_K_TD_SS = 4,
       XBFS_K_GENERATE_POST = 5, XBFS_K_BU = 6, XBFS_K_SELECT = 7, XBFS_K_SMALL = 8,
       XBFS_K_SS_COUNT = 9 };

/* Fill opts with the defaults (alpha 0.04, grow 2.0, ratio_min 1e-3, bu_stay 1, adaptive). */
void xbfs_run_opts_default(xbfs_run_opts* opts);

/* Build the symmetric CSR (Graph500 "kernel 1"; P:L358 layout) from M input
 * tuples (src[e], dst[e]) over N vertices: both arcs per tuple, self-loops and
 * duplicate arcs dropped, rows sorted by neighbour id.  Also records per-vertex
 * tuple counts (Graph500 m, O-6) and the non-isolated bitmap.
 *   src, dst : M ids each, width opts->id_bytes, host or device per opts.
 *              Borrowed for the call only.
 *   out      : receives a new handle (NULL on failure).
 * Errors: INVALID_ARG if out/src/dst NULL (with M > 0), N <= 0, N >= 2^31,
 * M < 0, or any id >= N; OUT_OF_MEMORY; CUDA.  Synchronises the stream. */
xbfs_status xbfs_build_csr(const void* src, const void* dst, int64_t num_edges, int64_t num_vertices,
                           const xbfs_build_opts* opts, xbfs_graph** out);

/* Degree-aware neighbour re-arrangement (§IV-B): mode 1 sorts every
 * row by neighbour degree descending, ties by id ascending (reading C-12);
 * mode 0 restores id order.  Levels are invariant; parents and BU probe
 * counts change.  Idempotent.  Errors: INVALID_ARG (mode), STATE, CUDA. */
xbfs_status xbfs_reorder(xbfs_graph* g, int32_t mode);

/* One BFS from `source` (v0 seeds level 0).  Writes every element of
 * the caller-owned DEVICE arrays level[N] and parent[N] (int32):
 *   level[v]  = hop distance from source, -1 if unreached (C-1)
 *   parent[v] = a neighbour of v with level[v]-1 (any valid one, C-14);
 *               parent[source] = source; -1 if unreached.
 * opts may be NULL (defaults).  stats may be NULL (no synchronisation).
 * Errors: INVALID_ARG (NULL g/level/parent, source outside [0,N)), STATE, CUDA. */
xbfs_status xbfs_run(xbfs_graph* g, int64_t source, int32_t* level, int32_t* parent,
                     const xbfs_run_opts* opts, xbfs_run_stats* stats);

/* Same as xbfs_run but level/parent are HOST arrays of N int32: the BFS runs
 * into the handle's device scratch and the result is copied back (D2H inside
 * the call).  Synchronises.  Used for the end-to-end (e2e) measurement. */
xbfs_status xbfs_run_host(xbfs_graph* g, int64_t source, int32_t* level_host, int32_t* parent_host,
                          const xbfs_run_opts* opts, xbfs_run_stats* stats);

/* Graph500-style multi-root run (TEPS over many roots) with HOST
 * outputs: one BFS per sources[i], i < count, each exactly as xbfs_run.  The
 * result of sources[i] lands in level_host/parent_host + (i % host_slots) * N
 * (host_slots >= 1; host_slots == count keeps every result; pinned host memory
 * gives full PCIe speed).  Pipelined: BFS i+1 runs on the handle's stream while
 * the D2H copies of BFS i run on a second stream (two device output slots,
 * allocated on first use, 16N bytes), so the call costs ~max(compute, copy)
 * per root instead of their sum.  Synchronises before returning.
 * Errors: INVALID_ARG (NULL pointer, count < 0, host_slots < 1, any source
 * outside [0,N): checked before anything is enqueued), STATE, CUDA. */
xbfs_status xbfs_run_host_batch(xbfs_graph* g, const int64_t* sources, int32_t count, int32_t host_slots,
                                int32_t* level_host, int32_t* parent_host, const xbfs_run_opts* opts);

/* Graph facts: N, stored arcs A, input tuples M, max degree.  Any out pointer
 * may be NULL. */
xbfs_status xbfs_graph_info(const xbfs_graph* g, int64_t* n, int64_t* arcs, int64_t* input_edges,
                            int32_t* max_degree);

/* Copy the CSR to host arrays row_ptr[N+1] (int64) and col[A] (int32).
 * Test/inspection only.  Synchronises. */
xbfs_status xbfs_copy_csr(const xbfs_graph* g, int64_t* row_ptr_host, int32_t* col_host);

/* Free the handle and all device memory it owns.  NULL-safe. */
void xbfs_destroy(xbfs_graph* g);

/* Thread-local message of the last failing call on this thread ("" if none). */
const char* xbfs_last_error(void);

/* Library build facts: compute capability compiled for (e.g. 100 for sm_100a). */
int32_t xbfs_compiled_arch(void);

#ifdef __cplusplus
}
#endif
#endif /* XBFS_H */
