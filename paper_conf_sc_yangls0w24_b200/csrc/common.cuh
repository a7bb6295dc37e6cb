// common.cuh — internal types of libxbfs (B200 / sm_100a).  Not part of the ABI.
//
// Layout in HBM:
//   row_ptr  int64[N+1]   col int32[A]      (8-byte edge, 4-byte vertex ids)
//   tcount   int32[N]     tuples per first endpoint (Graph500 m, O-6)
//   visited  uint32[W]    W = ceil(N/32); isolated vertices pre-set (never candidates)
//   fb[3]    uint32[W]    frontier bitmaps, rotated: level k reads fb[k%3] (F_k),
//                         writes fb[(k+1)%3] (F_{k+1}), clears fb[(k+2)%3] (F_{k-1})
//   queue[3] {qv int32, qoff int64, qdelta int64}[N] + tile_first int32[A/TILE+2]
//            qoff = exclusive prefix of degrees over the queue (edge-balanced tiles),
//            qdelta = row_ptr[v] - qoff, so arc a of the frontier is col[a + qdelta[j]].
//   DevState (device) + HostCtl (pinned, mapped) per handle.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <vector>

#include "xbfs.h"

namespace xbfs {

// L2 eviction-priority hints (B200 A/B, round 2): the outputs' lines are kept in L2 so
// the scattered level / parent stores of the levels merge there instead of costing a
// DRAM read-modify-write; streaming CSR reads may be marked evict-first.
#ifndef XBFS_OUT_KEEP
#define XBFS_OUT_KEEP 0
#endif
#ifndef XBFS_STREAM_HINT
#define XBFS_STREAM_HINT 0      // bit 0: head32, bit 1: col, bit 2: row_ptr -> L2 evict_first
#endif
__device__ __forceinline__ unsigned long long l2_policy_last() {
    unsigned long long p;
    asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ unsigned long long l2_policy_first() {
    unsigned long long p;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
// an output store (level / parent)
__device__ __forceinline__ void st_out(int* p, int v) {
#if XBFS_OUT_KEEP
    asm volatile("st.global.L2::cache_hint.b32 [%0], %1, %2;" ::"l"(p), "r"(v), "l"(l2_policy_last()) : "memory");
#else
    *p = v;
#endif
}
// read-only streaming loads: head32 (bit 0), col (bit 1), row_ptr (bit 2)
template <int BIT>
__device__ __forceinline__ unsigned ld_ro32(const unsigned* p) {
    if constexpr ((XBFS_STREAM_HINT & BIT) != 0) {
        unsigned v;
        asm volatile("ld.global.nc.L2::cache_hint.b32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(l2_policy_first()));
        return v;
    } else {
        return __ldg(p);
    }
}
template <int BIT>
__device__ __forceinline__ int ld_ro32(const int* p) {
    return (int)ld_ro32<BIT>(reinterpret_cast<const unsigned*>(p));
}
template <int BIT>
__device__ __forceinline__ long long ld_ro64(const long long* p) {
    if constexpr ((XBFS_STREAM_HINT & BIT) != 0) {
        long long v;
        asm volatile("ld.global.nc.L2::cache_hint.b64 %0, [%1], %2;" : "=l"(v) : "l"(p), "l"(l2_policy_first()));
        return v;
    } else {
        return *p;
    }
}

constexpr int kTile = 2048;          // frontier arcs per td_expand tile
constexpr int kExpandThreads = 512;  // td_expand block
constexpr int kBuThreads = 256;      // bu_traverse block (8 warps)
constexpr int kBuChunkWords = 8;     // bitmap words (256 vertices) per warp chunk
#ifndef XBFS_BU_BATCH
#define XBFS_BU_BATCH 4
#endif
constexpr int kBuBatch = XBFS_BU_BATCH;  // arcs probed per lane step (B200 A/B s24: 2 / 3 / 4 / 6 / 8 / 16 -> 796 / 815 / 825 / 822 / 818 / 784 GTEPS)
#ifndef XBFS_BU_HARD_MIN
#define XBFS_BU_HARD_MIN 256
#endif
constexpr int kBuHardMin = XBFS_BU_HARD_MIN;  // unresolved rows with more arcs left go warp-cooperative
#ifndef XBFS_BU_FIRST_ILP
#define XBFS_BU_FIRST_ILP 5
#endif
constexpr int kBuFirstIlp = XBFS_BU_FIRST_ILP;  // first probes in flight per lane (B200 A/B s24 48 roots, round 2: 4 / 5 / 6 -> 826 / 830 / 825 GTEPS)
constexpr int kGenThreads = 256;
constexpr int kSmallThreads = 512;   // small-frontier cluster kernel: threads per CTA
constexpr int kSmallCluster = 8;     // CTAs per cluster (portable size)
constexpr int kSmallInline = 8;      // frontier vertices with deg <= this are expanded by one thread
constexpr int kSmallBig = 8192;      // per-CTA list of higher-degree vertices (warp-cooperative)
constexpr long long kSmallEdgesMax = 9LL * kSmallBig;  // guarantees the big list never overflows
constexpr int kSmallMaxDeg = 512;    // frontier max degree allowed in the small mode (warp steps <= 16)
constexpr int kLogCap = 1 << 16;     // per-level log entries kept on the device
constexpr int kProfLaunches = 4096;  // per-launch timing: launches recorded at most
#ifndef XBFS_PERSIST_THREADS
#define XBFS_PERSIST_THREADS 1024
#endif
#ifndef XBFS_PERSIST_BLOCKS
#define XBFS_PERSIST_BLOCKS 1
#endif
constexpr int kPersistThreads = XBFS_PERSIST_THREADS; // persistent (one launch per BFS) driver: threads per CTA
constexpr int kPersistBlocks = XBFS_PERSIST_BLOCKS;   // ... CTAs per SM (64 registers per thread)

struct LevelRec {
    long long fsize, fedges, unvisited, probes;
    long long la_found;        // vertices this step set to level k+2 (BU look-ahead)
    int strategy, pad;
    unsigned long long t_ns;   // %globaltimer at the end of the level (persistent driver; 0 otherwise)
};

// Mirror of the scalars the host loop needs after each select (pinned + mapped).
struct HostCtl {
    int k, strategy, queue_valid, done;
    long long fsize, fedges;   // |F_k|, edgesF_k of the level about to run
    unsigned fmaxdeg;          // max degree over F_k
    int prev_small;            // level k-1 was a small SF level (small-mode entry gate)
};

struct DevState {
    int k;                  // level being processed
    int strategy;           // strategy chosen for level k
    int queue_valid;        // queue buffer k&1 holds F_k
    int done;
    unsigned long long qctr[3];  // packed (count << dbits) + degree sum of the queue of F_k in
                                 // slot k%3; level k zeroes slot (k+2)%3 (one barrier per level)
    unsigned qmax[3];            // max degree over the same queue (small-frontier mode gate)
    unsigned fmaxdeg;            // max degree over F_k
    long long fsize, fedges;     // |F_k|, edgesF_k
    long long fprev;             // |F_{k-1}|
    long long unvisited;         // U_k (non-isolated, unvisited)
    unsigned long long acc_found[3], acc_edges[3], acc_probes[3];  // BU / SS-count accumulators:
                                 // level k adds into slot k%3; slot (k+1)%3 is zeroed before level k+1
    unsigned long long acc_la_found[3], acc_la_edges[3];  // BU look-ahead (level k+2) discoveries, same slots
    unsigned long long td_ctr[3];     // step tickets of a dynamically scheduled top-down step, same slots
    unsigned long long acc_zero[3];   // SF winners with out-degree 0 (directed sinks), same slots: counted
                                      // in |F_{k+1}| but never queued (a tile's queue range stays <= its arcs)
    long long reached, arcs_traversed;
    unsigned int launches;       // library kernels launched (device-counted)
    int nlevels;
    // selection parameters (copied from xbfs_run_opts)
    double alpha, grow, ratio_min, bu_stay;
    int force, prev_strategy;
    long long source;
    long long small_edges;       // SF levels with edgesF_k <= this run in the cluster kernel (0 = off)
    int advanced;                // k_small already advanced the level state: k_select only mirrors it
    int prev_small;              // level k-1 was a small SF level (small-mode entry gate)
    int mirror_host;             // host-loop driver: mirror the level state into HostCtl
    int lookahead;               // BU look-ahead (persistent driver)
    unsigned long long t_start;  // %globaltimer after init + seed (persistent driver)
    unsigned long long t_enter;  // earliest CTA entry of the persistent kernel (atomicMin; host sets ~0)
    int* out_level;              // the run's output arrays (set per run with the parameters; the
    int* out_parent;             // per-level kernels read them here, so one CUDA graph serves any outputs)
    // persistent driver: grid-barrier arrival counter, alone on its 128-byte line
    // (zeroed with the rest of the state before every run)
    alignas(128) unsigned bar_count;
    unsigned bar_pad_[31];
};

// Arguments shared by all level kernels (static per handle => graph-capturable).
struct KArgs {
    const long long* row_ptr;
    const int* col;
    int* level;
    int* parent;
    const unsigned long long* head;  // per vertex: deg << 32 | first stored neighbour
    const unsigned* head32;          // per vertex: min(deg, dmax) << idbits | first neighbour (BU first probe)
    int idbits;                      // bits of a vertex id in head32 (bitlen(N-1))
    unsigned int* visited;
    unsigned int* fb[3];
    unsigned int* la;       // look-ahead bitmap: level-(k+2) vertices found by BU step k
    int* qv[3];
    long long* qoff[3];
    long long* qdelta[3];
    int* tile_first[3];
    DevState* st;
    HostCtl* hctl;          // device alias of the mapped host struct
    LevelRec* log;
    long long n;
    long long words;        // ceil(N/32)
    long long arcs;         // A
    int dbits;              // low bits of qctr holding the degree sum
    int track_max;          // keep qmax (frontier max degree) for the small-mode gate
    // the CSR bottom-up steps search: the same as row_ptr/col/head32 on a symmetric
    // graph, the transposed (in-arc) CSR on a directed one (reading R-9)
    const long long* bu_row_ptr;
    const int* bu_col;
    const unsigned* bu_head32;
    int directed;
};

}  // namespace xbfs

struct xbfs_graph {
    int device = 0;
    cudaStream_t stream = nullptr;
    bool poisoned = false;
    long long n = 0, arcs = 0, m_input = 0;
    int max_deg = 0;
    int reorder_mode = 0;
    int num_sms = 148;
    // CSR
    long long* row_ptr = nullptr;
    int* col = nullptr;
    int* tcount = nullptr;
    unsigned int* nonisolated = nullptr; // BU candidates: degree > 0 (in-degree > 0 when directed)
    // directed graphs (f4): transposed CSR searched by bottom-up steps
    int directed = 0;
    long long* in_row_ptr = nullptr;
    int* in_col = nullptr;
    unsigned* in_head32 = nullptr;
    unsigned long long* head = nullptr;  // deg << 32 | col[row_ptr[v]] (rebuilt by every reorder)
    unsigned* head32 = nullptr;          // the same in 4 bytes (degree capped, see k_head)
    int idbits = 32;
    long long nonisolated_count = 0;
    // BFS work state
    unsigned int* visited = nullptr;
    unsigned int* fb = nullptr;          // 4 * stride words: 3 frontier maps + the look-ahead map
    int* qv = nullptr;                   // 3 * N (queue of F_k in buffer k%3)
    long long* qoff = nullptr;           // 3 * N
    long long* qdelta = nullptr;         // 3 * N
    int* tile_first = nullptr;           // 3 * tiles_cap
    long long tiles_cap = 0;
    xbfs::DevState* st = nullptr;
    xbfs::LevelRec* log = nullptr;
    xbfs::HostCtl* hctl = nullptr;       // pinned host
    xbfs::HostCtl* hctl_dev = nullptr;   // its device alias
    // pinned staging ring of the per-run state: the H2D copy that resets the device state
    // stays asynchronous (from pageable memory the driver may wait for the stream first,
    // so the launch that follows was issued only once the GPU had gone idle)
    static constexpr int kStageSlots = 4;
    xbfs::DevState* hstage = nullptr;
    cudaEvent_t ev_stage[kStageSlots] = {nullptr, nullptr, nullptr, nullptr};
    int stage_next = 0;
    unsigned long long* red_scratch = nullptr;  // reductions for stats
    int* scratch_level = nullptr;        // xbfs_run_host device scratch: 2 slots of N (batch pipelining)
    int* scratch_parent = nullptr;
    cudaStream_t copy_stream = nullptr;  // D2H of xbfs_run_host_batch
    cudaEvent_t ev_done[2] = {nullptr, nullptr}, ev_copied[2] = {nullptr, nullptr};
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
    int dbits = 40;
    cudaGraphExec_t loop_exec = nullptr;   // CUDA-graph device loop: one per handle, built with it
    std::vector<cudaEvent_t> prof_events;  // per-launch timing pool (2 * kProfLaunches, built with it)
    struct xbfs_dist_part* dist = nullptr; // multi-GPU partition (xbfs_build_csr_dist); NULL = single GPU
    xbfs::KArgs kargs() const;
};

struct xbfs_comm;
namespace xbfs {
// driver state created at build / re-arrangement time (bfs.cu)
xbfs_status prepare_drivers(xbfs_graph* g);
// multi-GPU (comm.cu host collectives; dist.cu partition)
constexpr int kMaxCommRanks = 16;
xbfs_status comm_barrier(xbfs_comm* c);
xbfs_status comm_allgather(xbfs_comm* c, const void* mine, size_t bytes, void* all);
xbfs_status comm_allreduce_sum(xbfs_comm* c, const int64_t* in, int64_t* out, int n);
int comm_rank(const xbfs_comm* c);
int comm_size(const xbfs_comm* c);
void dist_destroy(struct xbfs_dist_part* d);
// error plumbing (api.cu)
xbfs_status set_error(xbfs_status s, const char* fmt, ...);
xbfs_status cuda_fail(xbfs_graph* g, cudaError_t e, const char* what);
}  // namespace xbfs

#define XBFS_CUDA(g, call)                                                  \
    do {                                                                    \
        cudaError_t _e = (call);                                            \
        if (_e != cudaSuccess) return ::xbfs::cuda_fail((g), _e, #call);    \
    } while (0)
