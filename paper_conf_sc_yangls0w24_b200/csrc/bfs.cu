// bfs.cu — the XBFS level kernels for sm_100a and the level-loop drivers.
//
// Per level k (§III):
//   SF  td_expand<SF>: atomic test-and-set on the visited bitmap;
//                    the winner writes level/parent and is appended to the next
//                    queue with ONE packed 64-bit atomic per warp that returns
//                    both its slot and its degree offset (edge-balanced tiles).
//   SS [generate if the queue is missing] + td_expand<SS> (plain
//                    level/parent stores, no status atomics; next-frontier bit
//                    set with a fire-and-forget RED) + generate (one scan of the
//                    next-frontier bitmap builds the next queue).  When a queue
//                    already exists (after SF/SS) the first generate is skipped:
//                    No-Frontier-Generation.
//   BU bu_traverse: each warp takes 32 bitmap words (1024
//                    vertices), compacts the unvisited ones with ballot/popc
//                    (the paper's count + prefix-sum + queue-write "double scan"
//                    folded into registers and shared memory), then each lane
//                    walks one candidate's (degree-ordered) row and stops
//                    at the first neighbour in the current frontier bitmap.
//   select (1 thread): consolidates the counters, logs the level, and picks the
//                    next strategy: BU iff edgesF/A > alpha, else
//                    SS/SF by frontier growth (reading C-10).
#include <stdio.h>
#include <string.h>

#include <cooperative_groups.h>

#include <algorithm>
#include <type_traits>

#include "common.cuh"
#include "bu_core.cuh"

namespace cg = cooperative_groups;

namespace xbfs {

constexpr unsigned FULL = 0xffffffffu;

// output fill with 256-bit stores (A/B)
#ifndef XBFS_FILL256
#define XBFS_FILL256 1
#endif

// output fill with L2 evict_last (init_body)
#ifndef XBFS_FILL_HINT
#define XBFS_FILL_HINT 1
#endif
constexpr long long kFillKeepBytes = 192LL << 20;

// BU first probe from the 4-byte head32[] (1) or the 8-byte head[] (0; A/B only)
#ifndef XBFS_BU_H32
#define XBFS_BU_H32 1
#endif

__device__ __forceinline__ void count_launch(DevState* st) {
    if (blockIdx.x == 0 && threadIdx.x == 0) atomicAdd(&st->launches, 1u);
}

// Clear the stale frontier bitmap fb[(k+2)%3] (it held F_{k-1}); it becomes the
// "next" bitmap of level k+1.  Grid-stride, vectorised.
__device__ __forceinline__ void clear_stale(const KArgs& a, int k) {
    unsigned int* z = a.fb[(k + 2) % 3];
    const long long w4 = a.words / 4;
    uint4* z4 = reinterpret_cast<uint4*>(z);
    const long long tid = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    const long long nth = (long long)gridDim.x * blockDim.x;
    for (long long i = tid; i < w4; i += nth) z4[i] = make_uint4(0, 0, 0, 0);
    for (long long i = w4 * 4 + tid; i < a.words; i += nth) z[i] = 0;
}

// Max-degree tracking without hammering one L2 address: most calls see a value
// that is already large enough and skip the atomic.
__device__ __forceinline__ void atomic_max_if_greater(unsigned* p, unsigned v) {
    if (v > __ldcg(p)) atomicMax(p, v);
}

// Frontier max degree only gates the small-frontier cluster mode of the
// per-level drivers; the persistent driver skips the tracking (KArgs.track_max).

// Warp-reduce a per-lane max and publish it (call with the whole warp converged).
__device__ __forceinline__ void flush_max(unsigned* p, unsigned lmax) {
    const unsigned w = __reduce_max_sync(FULL, lmax);
    if ((threadIdx.x & 31) == 0 && w) atomic_max_if_greater(p, w);
}

// Warp-aggregated enqueue of the lanes with `win` set: one 64-bit atomicAdd on
// the packed counter returns both the queue slot base (high bits) and the degree
// offset base (low dbits), so qoff is an exact exclusive prefix sum of degrees
// over the queue, in slot order.  Every tile start (multiple of kTile) that falls
// inside a vertex's arc range records that vertex's slot in tile_first.
// lmax accumulates the lane's max enqueued degree; the kernel publishes it once
// at the end with flush_max (no extra round trip inside the hot loop).
__device__ __forceinline__ void enqueue_warp(bool win, int v, long long rs, long long deg,
                                             unsigned long long* ctr, unsigned& lmax, int dbits, int* qv,
                                             long long* qoff, long long* qdelta, int* tile_first) {
    const unsigned mask = __ballot_sync(FULL, win);
    if (mask == 0) return;
    const int lane = threadIdx.x & 31;
    if (win) lmax = max(lmax, (unsigned)deg);
    const int rank = __popc(mask & ((1u << lane) - 1u));
    long long d = win ? deg : 0;
    long long incl = d;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        long long t = __shfl_up_sync(FULL, incl, o);
        if (lane >= o) incl += t;
    }
    const long long total = __shfl_sync(FULL, incl, 31);
    unsigned long long base = 0;
    if (lane == 0)
        base = atomicAdd(ctr, ((unsigned long long)__popc(mask) << dbits) + (unsigned long long)total);
    base = __shfl_sync(FULL, base, 0);
    if (win) {
        const long long slot = (long long)(base >> dbits) + rank;
        const long long off = (long long)(base & ((1ull << dbits) - 1ull)) + incl - d;
        qv[slot] = v;
        qoff[slot] = off;
        qdelta[slot] = rs - off;
        if (deg > 0) {
            const long long t0 = (off + kTile - 1) / kTile, t1 = (off + deg - 1) / kTile;
            for (long long t = t0; t <= t1; ++t) tile_first[t] = (int)slot;
        }
    }
}

// Same as enqueue_warp for up to R winners per lane (one atomic per warp).
template <int R>
__device__ __forceinline__ void enqueue_warp_multi(const bool (&win)[R], const int (&v)[R], const long long (&rs)[R],
                                                   const long long (&deg)[R], unsigned long long* ctr, unsigned& lmax,
                                                   int dbits, int* qv, long long* qoff, long long* qdelta,
                                                   int* tile_first) {
    int cnt = 0;
    long long dsum = 0;
#pragma unroll
    for (int i = 0; i < R; ++i)
        if (win[i]) { ++cnt; dsum += deg[i]; lmax = max(lmax, (unsigned)deg[i]); }
    if (!__any_sync(FULL, cnt > 0)) return;
    const int lane = threadIdx.x & 31;
    int ic = cnt;
    long long id = dsum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const int tc = __shfl_up_sync(FULL, ic, o);
        const long long td = __shfl_up_sync(FULL, id, o);
        if (lane >= o) { ic += tc; id += td; }
    }
    const int wc = __shfl_sync(FULL, ic, 31);
    const long long wd = __shfl_sync(FULL, id, 31);
    unsigned long long base = 0;
    if (lane == 0) base = atomicAdd(ctr, ((unsigned long long)wc << dbits) + (unsigned long long)wd);
    base = __shfl_sync(FULL, base, 0);
    long long slot = (long long)(base >> dbits) + ic - cnt;
    long long off = (long long)(base & ((1ull << dbits) - 1ull)) + id - dsum;
#pragma unroll
    for (int i = 0; i < R; ++i) {
        if (!win[i]) continue;
        qv[slot] = v[i];
        qoff[slot] = off;
        qdelta[slot] = rs[i] - off;
        if (deg[i] > 0) {
            const long long t0 = (off + kTile - 1) / kTile, t1 = (off + deg[i] - 1) / kTile;
            for (long long t = t0; t <= t1; ++t) tile_first[t] = (int)slot;
        }
        ++slot;
        off += deg[i];
    }
}

// The host-loop driver reads the level state from pinned, mapped host memory:
// one 32-byte store per level (skipped by the CUDA-graph driver).
__device__ __forceinline__ void mirror_host(const KArgs& a, const DevState* st) {
    if (!st->mirror_host) return;
    HostCtl h;
    h.k = st->k;
    h.strategy = st->strategy;
    h.queue_valid = st->queue_valid;
    h.done = st->done;
    h.fsize = st->fsize;
    h.fedges = st->fedges;
    h.fmaxdeg = st->fmaxdeg;
    h.prev_small = st->prev_small;
    *a.hctl = h;
}

// ---------------------------------------------------------------- init
// src >= 0 (persistent driver): the thread that fills the source's element writes
// its seed values instead (level 0, parent = itself, visited and F_0 bits), so the
// seed needs no barrier of its own after the fill.
__device__ __forceinline__ void init_body(const KArgs& a, int* __restrict__ level, int* __restrict__ parent,
                                          const unsigned int* __restrict__ nonisolated, long long src = -1,
                                          bool clear_la = false) {
    const long long tid = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    const long long nth = (long long)gridDim.x * blockDim.x;
    const long long n4 = a.n / 4;
    int4* l4 = reinterpret_cast<int4*>(level);
    int4* p4 = reinterpret_cast<int4*>(parent);
    const int4 m1 = make_int4(-1, -1, -1, -1);
#if XBFS_FILL256
    if ((((uintptr_t)level | (uintptr_t)parent) & 31) == 0) {
        // one 32-byte store per sector (STG.256).  Outputs of at most kFillKeepBytes are written
        // with L2 evict_last: their lines stay in L2, where the levels' scattered 4-byte
        // level / parent stores then merge instead of each costing a DRAM sector
        // read-modify-write (B200 A/B: s24 855 vs 829 GTEPS, s24d 730 vs 713, s20 / grid equal;
        // s27, whose 1 GB of outputs cannot stay: 1024 vs 1038 with the hint, hence the bound;
        // evict_first on the fill: 812; evict_last on the scattered stores themselves: 838;
        // evict_first on the head32 / col / row_ptr reads: equal or worse)
        const bool keep = XBFS_FILL_HINT && 8 * a.n <= kFillKeepBytes;
        const long long n8 = a.n / 8;
        const long long sc = src >= 0 ? src / 8 : -1;
        for (long long i = tid; i < n8; i += nth) {
            if (keep) {
                asm volatile("st.global.L1::no_allocate.L2::evict_last.v8.b32 [%0], {%1,%1,%1,%1,%1,%1,%1,%1};" ::"l"(level + 8 * i), "r"(-1) : "memory");
                asm volatile("st.global.L1::no_allocate.L2::evict_last.v8.b32 [%0], {%1,%1,%1,%1,%1,%1,%1,%1};" ::"l"(parent + 8 * i), "r"(-1) : "memory");
            } else {
                asm volatile("st.global.v8.b32 [%0], {%1,%1,%1,%1,%1,%1,%1,%1};" ::"l"(level + 8 * i), "r"(-1) : "memory");
                asm volatile("st.global.v8.b32 [%0], {%1,%1,%1,%1,%1,%1,%1,%1};" ::"l"(parent + 8 * i), "r"(-1) : "memory");
            }
            if (i == sc) { level[src] = 0; parent[src] = (int)src; }
        }
        for (long long i = n8 * 8 + tid; i < a.n; i += nth) {
            level[i] = i == src ? 0 : -1;
            parent[i] = i == src ? (int)src : -1;
        }
    } else
#endif
    if ((((uintptr_t)level | (uintptr_t)parent) & 15) == 0) {
        const long long sc = src >= 0 ? src / 4 : -1;
        for (long long i = tid; i < n4; i += nth) {
            l4[i] = m1;
            p4[i] = m1;
            if (i == sc) { level[src] = 0; parent[src] = (int)src; }
        }
        for (long long i = n4 * 4 + tid; i < a.n; i += nth) {
            level[i] = i == src ? 0 : -1;
            parent[i] = i == src ? (int)src : -1;
        }
    } else {
        for (long long i = tid; i < a.n; i += nth) {
            level[i] = i == src ? 0 : -1;
            parent[i] = i == src ? (int)src : -1;
        }
    }
    // isolated vertices are pre-marked visited: never BU candidates (reading C-27)
    const long long sw = src >= 0 ? src >> 5 : -1;
    const unsigned sbit = src >= 0 ? 1u << (src & 31) : 0u;
    for (long long w = tid; w < a.words; w += nth) {
        a.visited[w] = ~nonisolated[w] | (w == sw ? sbit : 0u);
        a.fb[0][w] = w == sw ? sbit : 0u;
        a.fb[1][w] = 0;
        a.fb[2][w] = 0;
        if (clear_la) a.la[w] = 0;   // (look-ahead map: the LA instantiation only)
    }
}

__global__ __launch_bounds__(256) void k_init_fill(KArgs a, const unsigned int* __restrict__ nonisolated) {
    count_launch(a.st);
    init_body(a, a.st->out_level, a.st->out_parent, nonisolated);
}

__device__ int choose_strategy(const DevState* st, long long arcs, long long fsize, long long fprev,
                               long long fedges, long long unvisited, int prev) {
    if (st->force >= 0) return st->force;
    // ratio = edgesF / A compared as edgesF > alpha * A (no division on the critical path)
    const double e = (double)fedges, A = (double)arcs;
    if (arcs > 0 && e > st->alpha * A) return XBFS_BU;                        // P:L87, strict (C-8)
    if (st->bu_stay > 0.0 && prev == XBFS_BU && (double)unvisited * st->bu_stay < e)
        return XBFS_BU;                                                       // C-11 (optional)
    if ((double)fsize > st->grow * (double)fprev && arcs > 0 && e > st->ratio_min * A) return XBFS_SS;  // C-10
    return XBFS_SF;
}

// Seed the source (the source holds level 0) and reset the level state.
// One thread.
// bits_done: init_body(src) already wrote the source's level/parent and bits.
__device__ __forceinline__ void seed_body(const KArgs& a, int* level, int* parent, long long nonisolated_count,
                                          const unsigned int* __restrict__ nonisolated, bool bits_done) {
    DevState* st = a.st;
    const long long s = st->source;   // per-run parameter copied in before init
    const long long rs = a.row_ptr[s], deg = a.row_ptr[s + 1] - rs;
    const unsigned sbit = 1u << (s & 31);
    // the source is a BU candidate (counted in U_0) iff it is not pre-set visited
    const bool s_cand = (nonisolated[s >> 5] & sbit) != 0;
    if (!bits_done) {
        level[s] = 0;
        parent[s] = (int)s;
        atomicOr(a.visited + (s >> 5), sbit);
        atomicOr(a.fb[0] + (s >> 5), sbit);
    }
    a.qv[0][0] = (int)s;
    a.qoff[0][0] = 0;
    a.qdelta[0][0] = rs;
    if (deg > 0) {
        const long long t1 = (deg - 1) / kTile;
        for (long long t = 0; t <= t1; ++t) a.tile_first[0][t] = 0;
    }
    st->k = 0;
    st->qctr[0] = (1ull << a.dbits) + (unsigned long long)deg;
    st->qctr[1] = 0;
    st->qctr[2] = 0;
    st->qmax[0] = (unsigned)deg;
    st->qmax[1] = 0;
    st->qmax[2] = 0;
    st->fmaxdeg = (unsigned)deg;
    st->prev_small = 0;
    st->queue_valid = 1;
    st->done = 0;
    st->fsize = 1;
    st->fedges = deg;
    st->fprev = 0;
    st->unvisited = nonisolated_count - (s_cand ? 1 : 0);
    for (int i = 0; i < 3; ++i) {
        st->acc_found[i] = st->acc_edges[i] = st->acc_probes[i] = st->acc_zero[i] = st->td_ctr[i] = 0;
        st->acc_la_found[i] = st->acc_la_edges[i] = 0;
    }
    st->reached = 0;
    st->arcs_traversed = 0;
    st->nlevels = 0;
    st->source = s;
    st->prev_strategy = -1;
    st->strategy = choose_strategy(st, a.arcs, 1, 0, deg, st->unvisited, -1);
}

__global__ void k_seed(KArgs a, long long nonisolated_count, const unsigned int* __restrict__ nonisolated) {
    count_launch(a.st);
    seed_body(a, a.st->out_level, a.st->out_parent, nonisolated_count, nonisolated, false);
    mirror_host(a, a.st);
}

// ------------------------------------------------------------- select
// The level state the selector evolves (one copy per CTA in the persistent
// driver, where every CTA computes the same decision from the same counters).
struct SelState {
    int k, strategy, queue_valid, done, prev_strategy, nlevels, prev_small, prefill, qreset, pad_;
    long long fsize, fedges, fprev, unvisited, reached, arcs_traversed;
    long long la_cf, la_ce;    // look-ahead vertices (count, degree sum) merged into F_{k+1} before level k
    unsigned fmaxdeg;
};

// End of level k: consolidate the counters of F_{k+1} (acc slot k%3 after BU / SS,
// queue counter (k+1)%3 after SF), log the level (if `log_it`), choose the
// strategy of level k+1 (P:L87 rule + readings C-10/C-11).  All counter reads go
// through L2.
__device__ __forceinline__ void select_step(const KArgs& a, SelState& s, bool log_it, unsigned long long t_ns) {
    const DevState* st = a.st;
    const int k = s.k;
    const int strat = s.strategy;
    long long nf, ne;
    if (strat == XBFS_BU || strat == XBFS_SS) {   // counted by k_bu_traverse / k_ss_count; no queue
        nf = (long long)__ldcg(&st->acc_found[k % 3]);
        ne = (long long)__ldcg(&st->acc_edges[k % 3]);
        s.queue_valid = 0;
    } else {
        const unsigned long long q = __ldcg(&st->qctr[(k + 1) % 3]);
        nf = (long long)(q >> a.dbits);
        ne = (long long)(q & ((1ull << a.dbits) - 1ull));
        if (a.directed) nf += (long long)__ldcg(&st->acc_zero[k % 3]);   // unqueued sinks
        s.queue_valid = 1;
    }
    // look-ahead (persistent driver): vertices of F_{k+1} that BU step k-1 already
    // set (level k+1) were merged into the F_{k+1} bitmap before this level; the
    // count pass of SS saw them, the BU / SF counters did not, and an SF queue
    // lacks them.
    const long long carry_f = s.la_cf;
    s.qreset = 0;
    if (carry_f) {
        if (strat != XBFS_SS) { nf += carry_f; ne += s.la_ce; }
        s.queue_valid = 0;
        // an SF step filled queue slot (k+1)%3 without the carried vertices; the
        // queue is regenerated into that slot, whose counter must restart at 0
        s.qreset = strat == XBFS_SF;
    }
    long long laf = 0, lae = 0;
    if (strat == XBFS_BU && st->lookahead) {
        laf = (long long)__ldcg(&st->acc_la_found[k % 3]);
        lae = (long long)__ldcg(&st->acc_la_edges[k % 3]);
    }
    if (log_it && k < kLogCap) {
        LevelRec r;
        r.fsize = s.fsize;
        r.fedges = s.fedges;
        r.unvisited = s.unvisited;
        r.probes = strat == XBFS_BU ? (long long)__ldcg(&st->acc_probes[k % 3]) : 0;
        r.la_found = laf;
        r.strategy = strat;
        r.pad = 0;
        r.t_ns = t_ns;
        a.log[k] = r;
    }
    // enter the small-frontier mode only after one small SF level has already run
    // through the level kernels (a single small level does not pay for the switch)
    s.prev_small = strat == XBFS_SF && s.fedges <= st->small_edges && s.fmaxdeg <= (unsigned)kSmallMaxDeg;
    s.reached += s.fsize;
    s.arcs_traversed += s.fedges;
    s.fprev = s.fsize;
    s.fsize = nf;
    s.fedges = ne;
    s.unvisited -= nf - carry_f + laf;   // newly visited during level k
    s.la_cf = laf;
    s.la_ce = lae;
    s.prefill = laf > 0;
    s.prev_strategy = strat;
    s.k = k + 1;
    s.fmaxdeg = __ldcg(&st->qmax[(k + 1) % 3]);
    if (nf == 0) {
        s.done = 1;
        s.nlevels = k + 1;
    } else {
        s.strategy = choose_strategy(st, a.arcs, nf, s.fprev, ne, s.unvisited, strat);
    }
}

__device__ __forceinline__ void sel_load(const DevState* st, SelState& s) {
    s.k = __ldcg(&st->k);
    s.strategy = __ldcg(&st->strategy);
    s.queue_valid = __ldcg(&st->queue_valid);
    s.done = __ldcg(&st->done);
    s.prev_strategy = __ldcg(&st->prev_strategy);
    s.nlevels = __ldcg(&st->nlevels);
    s.prev_small = __ldcg(&st->prev_small);
    s.fsize = __ldcg(&st->fsize);
    s.fedges = __ldcg(&st->fedges);
    s.fprev = __ldcg(&st->fprev);
    s.unvisited = __ldcg(&st->unvisited);
    s.reached = __ldcg(&st->reached);
    s.arcs_traversed = __ldcg(&st->arcs_traversed);
    s.fmaxdeg = __ldcg(&st->fmaxdeg);
    s.prefill = 0;
    s.qreset = 0;
    s.la_cf = s.la_ce = 0;   // look-ahead runs only in the persistent driver, whose state never leaves the kernel
}

__device__ __forceinline__ void sel_store(DevState* st, const SelState& s) {
    st->k = s.k;
    st->strategy = s.strategy;
    st->queue_valid = s.queue_valid;
    st->done = s.done;
    st->prev_strategy = s.prev_strategy;
    st->nlevels = s.nlevels;
    st->prev_small = s.prev_small;
    st->fsize = s.fsize;
    st->fedges = s.fedges;
    st->fprev = s.fprev;
    st->unvisited = s.unvisited;
    st->reached = s.reached;
    st->arcs_traversed = s.arcs_traversed;
    st->fmaxdeg = s.fmaxdeg;
}

// Per-level kernels: one thread reads the state, steps it, writes it back and
// zeroes the slots level k+1 accumulates into (qctr/qmax (k+2)%3, acc (k+1)%3).
// Fusing it into the last block of the level kernels was measured slower: it
// raised their register pressure (spills).
__device__ void select_body(const KArgs& a) {
    DevState* st = a.st;
    SelState s;
    sel_load(st, s);
    const int k = s.k;
    select_step(a, s, true, 0ull);
    st->qctr[(k + 2) % 3] = 0;   // counter of the queue built during level k+1
    st->qmax[(k + 2) % 3] = 0;
    st->acc_found[(k + 1) % 3] = st->acc_edges[(k + 1) % 3] = st->acc_probes[(k + 1) % 3] = 0;
    st->acc_zero[(k + 1) % 3] = 0;
    st->td_ctr[(k + 1) % 3] = 0;
    st->acc_la_found[(k + 1) % 3] = st->acc_la_edges[(k + 1) % 3] = 0;
    sel_store(st, s);
    mirror_host(a, st);
}

// Profiling build (XBFS_TL_PROF=1): per level, min / max over CTAs of %globaltimer at
// the level's start, when the CTA's work is done, after its release fence and when it
// leaves the level's last barrier; per warp, stamps inside the scan-free expansion of
// levels < 8 (printed to stderr after a run with stats).
#ifndef XBFS_TL_PROF
#define XBFS_TL_PROF 0
#endif
#if XBFS_TL_PROF
constexpr int kTlLevels = 64;
constexpr int kTlwLevels = 8, kTlwWarps = 8192;
__device__ unsigned long long g_tl[kTlLevels][8][2];   // phases 0-3 last barrier, 5-7 a mid-level one
__device__ unsigned long long g_tlw[kTlwLevels][5][kTlwWarps];   // SF sub-phases per warp (lane 0)
__device__ __forceinline__ void tlw_rec(int k, int ph) {
    const long long gwarp = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
    if ((threadIdx.x & 31) == 0 && k < kTlwLevels && gwarp < kTlwWarps) {
        unsigned long long t;
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
        g_tlw[k][ph][gwarp] = t;
    }
}
__device__ __forceinline__ void tl_rec(int k, int ph, unsigned long long t) {
    if (k >= 0 && k < kTlLevels) {
        atomicMin(&g_tl[k][ph][0], t);
        atomicMax(&g_tl[k][ph][1], t);
    }
}
#define XBFS_TLW(k, ph) tlw_rec(k, ph)
#else
#define XBFS_TLW(k, ph) ((void)0)
#endif

// ----------------------------------------------------------- top-down
// One tile = kTile consecutive frontier arcs; tile_first gives the first queue
// entry overlapping it, so tiles are balanced regardless of the degree mix
// (hubs span many tiles, small vertices share one).  Arc a of the frontier is
// col[a + qdelta[j]] for its owner j (binary search of qoff in shared memory).
// TPT base tiles form one CTA step of the persistent kernel (more arcs in flight
// per thread when its CTAs are 1024 threads wide); the per-level kernels use 1.
// B200 A/B (1024 x 1 persistent CTAs, s24): SS 2 / SF 1 = 334 us per BFS,
// 1/1 = 342, 2/2 = 345, 4/1 = 347 (SF's enqueue registers spill at R = 4).
template <int TPT>
struct TdSmemT {
    long long off[TPT * kTile + 1];
    long long delta[TPT * kTile + 1];
    int v[TPT * kTile + 1];
    long long next;   // dynamic scheduling: the CTA's next step
};
using TdSmem = TdSmemT<1>;

#ifndef XBFS_SS_TPT
#define XBFS_SS_TPT 2
#endif
#ifndef XBFS_SF_TPT
#define XBFS_SF_TPT 1
#endif

#ifndef XBFS_SS_CLAIM
#define XBFS_SS_CLAIM 0
#endif

#ifndef XBFS_TD_DYN
#define XBFS_TD_DYN 1
#endif
#ifndef XBFS_SPLIT_MAX
#define XBFS_SPLIT_MAX 4
#endif
constexpr long long kSplitMax = XBFS_SPLIT_MAX;   // parts per base tile when tiles are fewer than CTAs (0: off; B200 A/B grid 4096^2: 2 / 4 / 8 / 32 -> 0.627 / 0.656 / 0.645 / 0.600 GTEPS, s20 and s24 flat)
#ifndef XBFS_SPLIT_MIN_ARCS
#define XBFS_SPLIT_MIN_ARCS 64
#endif
constexpr long long kSplitMinArcs = XBFS_SPLIT_MIN_ARCS;            // ... each of at least this many arcs

#ifndef XBFS_SF_PRECHECK_MIN
#define XBFS_SF_PRECHECK_MIN 65536
#endif
constexpr long long kSfPrecheckMin = XBFS_SF_PRECHECK_MIN;   // edgesF_k above which SF probes before claiming

// The top-down probe of visited may go through L1 (XBFS_TD_VIS_L1): within a level the
// bits only go 0 -> 1, so a stale line can only report a vertex of F_{k+1} as unvisited,
// which costs SF an atomic that then fails and SS a second store of the same level with
// another valid parent (C-26); vertices of earlier levels are always seen, because the
// grid barrier's acquire invalidates L1 (CCTL.IVALL) before every level.
#ifndef XBFS_TD_VIS_L1
#define XBFS_TD_VIS_L1 1
#endif
// (SS: a vertex found earlier in the same level is seen as visited only through L2, where
// the REDs land; a stale L1 line costs four scattered writes)
#ifndef XBFS_SS_VIS_L1
#define XBFS_SS_VIS_L1 0
#endif
__device__ __forceinline__ unsigned ld_vis(const unsigned* p) {
#if XBFS_TD_VIS_L1
    return __ldca(p);
#else
    return __ldcg(p);
#endif
}

// DIR: directed graph (f4, R-9): out-degree-0 winners are counted, not queued.
template <int MODE, int THREADS, int TPT = 1, bool DIR = false>
__device__ __forceinline__ void td_expand_body(const KArgs& a, int k, int* __restrict__ level,
                                               int* __restrict__ parent, TdSmemT<TPT>& sm, long long Fs = -1,
                                               long long Ts = -1) {
    clear_stale(a, k);
    const int in = k % 3, ob = (k + 1) % 3;
    long long F = Fs, T = Ts;   // |F_k|, edgesF_k: from the caller's selector state when it has them
    if (F < 0) {
        const unsigned long long q = __ldcg(&a.st->qctr[k % 3]);
        F = (long long)(q >> a.dbits);
        T = (long long)(q & ((1ull << a.dbits) - 1ull));
    }
    if (F == 0 || T == 0) return;
    // small scan-free levels claim with the atomic directly (one round trip less
    // per arc chain); large ones probe first so that arcs to visited vertices,
    // the majority there, cost no atomic
    const bool precheck = MODE != XBFS_SF || T > kSfPrecheckMin;
    const long long ntiles = (T + kTile - 1) / kTile;
    const int* __restrict__ qv = a.qv[in];
    const long long* __restrict__ qoff = a.qoff[in];
    const long long* __restrict__ qdelta = a.qdelta[in];
    const int* __restrict__ tfirst = a.tile_first[in];
    unsigned int* __restrict__ visited = a.visited;
    unsigned int* __restrict__ next = a.fb[(k + 1) % 3];
    const int lvl = k + 1;
    long long* s_off = sm.off;
    long long* s_delta = sm.delta;
    int* s_v = sm.v;
    unsigned lmax = 0;

    // Scan-free levels with fewer tiles than CTAs (small frontiers: the first levels, the
    // tail, many-level graphs): every base tile is split into S equal parts (>= 64 arcs
    // each; single-scan steps keep whole tiles: B200 A/B s24, its hub level 260 -> 295 us
    // with the split code in its loop), so that the
    // scattered claims, stores and row_ptr reads of a small level are spread over up to
    // every SM instead of queueing in the few that hold a 2048-arc tile (one SM issues
    // ~1 scattered sector per clock: a tile of winners alone took 7-12 us).
    const long long nsteps_full = (ntiles + TPT - 1) / TPT;
    const long long S = (MODE != XBFS_SF || nsteps_full >= gridDim.x || kSplitMax == 0)
                            ? 0
                            : max(1LL, min(min((long long)gridDim.x / ntiles, (long long)kSplitMax),
                                           T / (ntiles * kSplitMinArcs)));
    const long long nsteps = S ? ntiles * S : nsteps_full;
    // Large single-scan steps take their steps from a ticket counter instead of
    // round-robin: the cost of a step varies with how many of its arcs discover a vertex,
    // and the static deal left the CTAs of a hub level finishing 25-35 us apart (level
    // timeline, s24).  Thread 0 holds the ticket of the step after next, so the atomic's
    // round trip hides behind a whole step.
    const bool dyn = XBFS_TD_DYN && MODE == XBFS_SS && nsteps >= 2 * (long long)gridDim.x;
    unsigned long long* tctr = &a.st->td_ctr[k % 3];
    unsigned long long tk = 0;
    if (dyn && threadIdx.x == 0) tk = gridDim.x + atomicAdd(tctr, 1ull);
    for (long long t = blockIdx.x; t < nsteps;) {
        long long a0, a1, i0, i1;
        if (S) {
            const long long Sd = S > 0 ? S : 1;   // (S == 0 is a compile-time constant for SS)
            const long long bt = t / Sd, p = t - bt * Sd;
            const long long b0 = bt * kTile, bl = min(b0 + kTile, T) - b0;
            a0 = b0 + bl * p / Sd;
            a1 = b0 + bl * (p + 1) / Sd;
            i0 = __ldcg(tfirst + bt);
            i1 = (bt + 1 < ntiles) ? (long long)__ldcg(tfirst + bt + 1) : F - 1;
        } else {
            a0 = t * TPT * kTile;
            a1 = min(a0 + (long long)(TPT * kTile), T);
            i0 = __ldcg(tfirst + t * TPT);
            i1 = (t * TPT + TPT < ntiles) ? (long long)__ldcg(tfirst + t * TPT + TPT) : F - 1;
        }
        const int nv = (int)(i1 - i0 + 1);
        __syncthreads();
        if (dyn && threadIdx.x == 0) {
            sm.next = (long long)tk;
            tk = gridDim.x + atomicAdd(tctr, 1ull);
        }
        for (int i = threadIdx.x; i < nv; i += THREADS) {
            s_off[i] = __ldcg(qoff + i0 + i);
            s_delta[i] = __ldcg(qdelta + i0 + i);
            s_v[i] = __ldcg(qv + i0 + i);
        }
        __syncthreads();
        const long long t_next = dyn ? sm.next : t + gridDim.x;
        if (MODE == XBFS_SF) XBFS_TLW(k, 0);
        // R arcs per thread (stride THREADS: coalesced col reads), processed
        // stage by stage so the R dependent load chains are in flight together.
        constexpr int R = TPT * kTile / THREADS;
        int v[R], u[R];
        unsigned vis[R];
        bool valid[R], win[R];
        long long rs[R], deg[R];
#pragma unroll
        for (int i = 0; i < R; ++i) {
            const long long arc = a0 + i * THREADS + threadIdx.x;
            valid[i] = arc < a1;
            v[i] = 0;
            u[i] = 0;
            if (valid[i]) {
                // owner: last j with s_off[j] <= arc
                int lo = 0, hi = nv - 1;
                while (lo < hi) {
                    const int mid = (lo + hi + 1) >> 1;
                    if (s_off[mid] <= arc) lo = mid; else hi = mid - 1;
                }
                v[i] = ld_ro32<2>(a.col + arc + s_delta[lo]);
                u[i] = s_v[lo];
            }
        }
#pragma unroll
        for (int i = 0; i < R; ++i)
            vis[i] = !valid[i] ? FULL
                               : (!precheck ? 0u
                                            : ((MODE == XBFS_SF || XBFS_SS_VIS_L1) ? ld_vis(visited + (v[i] >> 5))
                                                                                   : __ldcg(visited + (v[i] >> 5))));
        if (MODE == XBFS_SF) {
            unsigned old[R];
#pragma unroll
            for (int i = 0; i < R; ++i) {
                const unsigned bit = 1u << (v[i] & 31);
                old[i] = (vis[i] & bit) ? bit : atomicOr(visited + (v[i] >> 5), bit);
            }
#if XBFS_TL_PROF
            {   // stamp once the claims have returned
                unsigned x = 0;
#pragma unroll
                for (int i = 0; i < R; ++i) x |= old[i];
                if (x == 0x12345678u) __nanosleep(1);
                XBFS_TLW(k, 1);
            }
#endif
#pragma unroll
            for (int i = 0; i < R; ++i) {
                const unsigned bit = 1u << (v[i] & 31);
                win[i] = valid[i] && !(old[i] & bit);
                rs[i] = 0;
                deg[i] = 0;
                if (win[i]) {
                    st_out(level + v[i], lvl);
                    st_out(parent + v[i], u[i]);
                    atomicOr(next + (v[i] >> 5), bit);
                    rs[i] = a.row_ptr[v[i]];
                    deg[i] = a.row_ptr[v[i] + 1];
                }
            }
#pragma unroll
            for (int i = 0; i < R; ++i) deg[i] -= rs[i];
            XBFS_TLW(k, 2);
            if constexpr (DIR) {
                int zc = 0;     // winners without out-arcs (directed sinks) are counted, not queued
#pragma unroll
                for (int i = 0; i < R; ++i)
                    if (win[i] && deg[i] == 0) { ++zc; win[i] = false; }
                if (__any_sync(FULL, zc)) {
                    zc = __reduce_add_sync(FULL, (unsigned)zc);
                    if ((threadIdx.x & 31) == 0) atomicAdd(&a.st->acc_zero[k % 3], (unsigned long long)zc);
                }
            }
            enqueue_warp_multi<R>(win, v, rs, deg, &a.st->qctr[(k + 1) % 3], lmax, a.dbits, a.qv[ob],
                                  a.qoff[ob], a.qdelta[ob], a.tile_first[ob]);
            XBFS_TLW(k, 3);
        } else {
            // single-scan: no status atomics; two threads that both see the bit
            // clear write the same level value (benign race; either parent is
            // valid, C-26).  Both bitmaps get fire-and-forget REDs, so later arcs
            // of this level mostly see the vertex as visited (one probe per arc).
#if XBFS_SS_CLAIM
            // (variant) the visited RED returns the old word: only the first writer stores
            unsigned old[R];
#pragma unroll
            for (int i = 0; i < R; ++i) {
                const unsigned bit = 1u << (v[i] & 31);
                old[i] = (valid[i] && !(vis[i] & bit)) ? atomicOr(visited + (v[i] >> 5), bit) : FULL;
            }
#pragma unroll
            for (int i = 0; i < R; ++i) {
                const unsigned bit = 1u << (v[i] & 31);
                if (!(old[i] & bit)) {
                    level[v[i]] = lvl;
                    parent[v[i]] = u[i];
                    atomicOr(next + (v[i] >> 5), bit);
                }
            }
#else
#pragma unroll
            for (int i = 0; i < R; ++i) {
                const unsigned bit = 1u << (v[i] & 31);
                if (valid[i] && !(vis[i] & bit)) {
                    st_out(level + v[i], lvl);
                    st_out(parent + v[i], u[i]);
                    atomicOr(next + (v[i] >> 5), bit);
                    atomicOr(visited + (v[i] >> 5), bit);
                }
            }
#endif
        }
        t = t_next;
    }
    if (MODE == XBFS_SF) XBFS_TLW(k, 4);
    if (MODE == XBFS_SF && a.track_max) flush_max(&a.st->qmax[(k + 1) % 3], lmax);
}

template <int MODE>
__global__ __launch_bounds__(kExpandThreads, 2) void k_td_expand(KArgs a) {
    count_launch(a.st);
    __shared__ TdSmem sm;
    td_expand_body<MODE, kExpandThreads>(a, a.st->k, a.st->out_level, a.st->out_parent, sm);
}

// -------------------------------------------------------------- generate
// Single-scan's one scan over the status, here the N-bit next-frontier
// bitmap: it yields the counters the selector needs (|F_{k+1}|, edgesF_{k+1},
// max degree, from the dense head[] array) into acc slot k%3.  The queue itself
// is materialised by generate (role 0) only if the next level is top-down; a
// bottom-up next level never needs it (the bitmap is its input).  visited
// already holds F_{k+1}: the expansion set it with REDs.
__device__ __forceinline__ void ss_count_body(const KArgs& a, int k) {
    const unsigned int* __restrict__ bm = a.fb[(k + 1) % 3];
    unsigned long long found = 0, edges = 0;
    unsigned gmax = 0;
    for (long long w = blockIdx.x * (long long)blockDim.x + threadIdx.x; w < a.words;
         w += (long long)gridDim.x * blockDim.x) {
        unsigned word = __ldcg(bm + w);
        if (!word) continue;
        found += __popc(word);
        // up to 8 head32[] loads in flight per step (a dense frontier word holds several
        // bits); the 4-byte word halves the bytes of the 8-byte head[] (a saturated degree
        // field, deg >= dmax, falls back to the row_ptr pair)
        const unsigned dmax = a.idbits >= 32 ? 0u : (0xffffffffu >> a.idbits);
        while (word) {
            unsigned hv[8];
            int vx[8];
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                hv[i] = 0u;
                vx[i] = -1;
                if (word) {
                    vx[i] = (int)(w * 32 + __ffs(word) - 1);
                    hv[i] = __ldg(a.head32 + vx[i]);
                    word &= word - 1;
                }
            }
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                unsigned d = a.idbits >= 32 ? dmax : hv[i] >> a.idbits;
                if (vx[i] >= 0 && d >= dmax) d = (unsigned)(a.row_ptr[vx[i] + 1] - a.row_ptr[vx[i]]);
                edges += d;
                gmax = max(gmax, d);
            }
        }
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        found += __shfl_xor_sync(FULL, found, o);
        edges += __shfl_xor_sync(FULL, edges, o);
    }
    if ((threadIdx.x & 31) == 0 && found) {
        atomicAdd(&a.st->acc_found[k % 3], found);
        atomicAdd(&a.st->acc_edges[k % 3], edges);
    }
    if (a.track_max) flush_max(&a.st->qmax[(k + 1) % 3], gmax);
}

__global__ __launch_bounds__(kGenThreads) void k_ss_count(KArgs a) {
    count_launch(a.st);
    ss_count_body(a, a.st->k);
}

// Bitmap -> queue (the single-scan generation pass, over the N-bit frontier
// bitmap instead of the 4N-byte status array).  role 0: F_k from fb[k%3] into
// queue slot k%3 (queue missing after a BU / SS level).  role 1: F_{k+1} from
// fb[(k+1)%3] into slot (k+1)%3 and visited |= F_{k+1}.
__device__ __forceinline__ void generate_body(const KArgs& a, int k, int role) {
    const unsigned int* __restrict__ bm = role == 0 ? a.fb[k % 3] : a.fb[(k + 1) % 3];
    const int ob = role == 0 ? k % 3 : (k + 1) % 3;
    unsigned long long* ctr = &a.st->qctr[role == 0 ? k % 3 : (k + 1) % 3];
    const long long nth = (long long)gridDim.x * blockDim.x;
    const long long base_tid = blockIdx.x * (long long)blockDim.x + (threadIdx.x & ~31);
    const int lane = threadIdx.x & 31;
    unsigned gmax = 0;
    for (long long w0 = base_tid; w0 < a.words; w0 += nth) {
        const long long w = w0 + lane;
        unsigned word = w < a.words ? __ldcg(bm + w) : 0u;
        if (role == 1 && word) a.visited[w] = __ldcg(a.visited + w) | word;
        // pass 1: count and degree sum of this lane's vertices; vertices without
        // (out-)arcs are not queued (directed sinks: nothing to expand, and a tile's
        // queue range must stay within its arcs)
        int cnt = 0;
        long long dsum = 0;
        for (unsigned b = word; b; b &= b - 1) {
            const long long v = w * 32 + __ffs(b) - 1;
            const long long d = a.row_ptr[v + 1] - a.row_ptr[v];
            dsum += d;
            cnt += d > 0;
            gmax = max(gmax, (unsigned)d);
        }
        int ic = cnt;
        long long id = dsum;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int tc = __shfl_up_sync(FULL, ic, o);
            const long long td = __shfl_up_sync(FULL, id, o);
            if (lane >= o) { ic += tc; id += td; }
        }
        const int wc = __shfl_sync(FULL, ic, 31);
        if (wc == 0) continue;
        const long long wd = __shfl_sync(FULL, id, 31);
        unsigned long long base = 0;
        if (lane == 0) base = atomicAdd(ctr, ((unsigned long long)wc << a.dbits) + (unsigned long long)wd);
        base = __shfl_sync(FULL, base, 0);
        long long slot = (long long)(base >> a.dbits) + ic - cnt;
        long long off = (long long)(base & ((1ull << a.dbits) - 1ull)) + id - dsum;
        int* qv = a.qv[ob];
        long long* qoff = a.qoff[ob];
        long long* qdelta = a.qdelta[ob];
        int* tf = a.tile_first[ob];
        for (unsigned b = word; b; b &= b - 1) {
            const long long v = w * 32 + __ffs(b) - 1;
            const long long rs = a.row_ptr[v], deg = a.row_ptr[v + 1] - rs;
            if (deg == 0) continue;
            qv[slot] = (int)v;
            qoff[slot] = off;
            qdelta[slot] = rs - off;
            if (deg > 0) {
                const long long t0 = (off + kTile - 1) / kTile, t1 = (off + deg - 1) / kTile;
                for (long long t = t0; t <= t1; ++t) tf[t] = (int)slot;
            }
            ++slot;
            off += deg;
        }
    }
    if (a.track_max) flush_max(&a.st->qmax[role == 0 ? k % 3 : (k + 1) % 3], gmax);
}

__global__ __launch_bounds__(kGenThreads) void k_generate(KArgs a, int role) {
    count_launch(a.st);
    generate_body(a, a.st->k, role);
}

// ------------------------------------------------------------- bottom-up
// Candidates U_k = not visited (isolated vertices are pre-marked visited).
// A candidate v is found iff some neighbour is in F_k = fb[k%3] (never a bit set
// in this same pass: reading C-9), giving level k+1 and that neighbour as parent.
// kp: where k lives (DevState or the persistent CTA's selector copy); it is
// re-read for the epilogue instead of keeping k live across the traversal
// (one register less: the per-level kernel runs at 48 without spills).
#ifndef XBFS_BU_ALT
#define XBFS_BU_ALT 1
#endif
#if XBFS_BU_PROF
__device__ unsigned long long g_bu_prof[8];   // profiling build: BU phase cycles of the dense steps
#endif

template <int WARPS, bool LA, class Smem, bool DIR = false>
__device__ __forceinline__ void bu_body(const KArgs& a, const int* kp, int* __restrict__ level,
                                        int* __restrict__ parent, Smem& sm, bool prefill, long long U) {
    int k = *(const volatile int*)kp;
    clear_stale(a, k);
    const unsigned int* __restrict__ cur = a.fb[k % 3];
    unsigned int* __restrict__ next = a.fb[(k + 1) % 3];
    const int lvl = k + 1;
    unsigned long long found = 0, edges = 0, probes = 0;
    unsigned fmax = 0;
    BuLa la;
    BuView b;
    b.cur = cur;
    b.nxt = next;
    b.visited = a.visited;
    b.words = a.words;
    b.head = a.head;
    b.head32 = DIR ? a.bu_head32 : a.head32;   // in-arc CSR on a directed graph (f4, R-9)
    b.idbits = a.idbits;
    b.row_ptr = DIR ? a.bu_row_ptr : a.row_ptr;
    b.col = DIR ? a.bu_col : a.col;
    b.level = level;
    b.parent = parent;
    b.lvl = lvl;
    // consecutive BU steps sweep in opposite directions; even levels (the first BU step is
    // usually level 2) walk downwards, starting where the grid-stride output fill ended
    // (B200 A/B s24: even-down 862 vs odd-down 856 GTEPS)
    b.reverse = XBFS_BU_ALT && !(k & 1);
#if XBFS_BU_PROF
    b.prof = U * 16 >= a.n ? g_bu_prof : nullptr;   // the dense steps only
#endif
    // prefill: F_{k+1} already holds look-ahead vertices of step k-1 (OR into it)
    const bool pf = LA && prefill;
    unsigned long long oedges = 0;   // DIR: out-degrees of the found vertices, summed where they are published
    bu_chunks<WARPS, LA, XBFS_BU_H32>(b, sm, [&](long long w, unsigned vis, unsigned f, unsigned lf) {
        if (pf) f |= __ldcg(next + w);
        if (f) next[w] = f;
        a.visited[w] = vis | f | lf;
        if (LA && lf) a.la[w] = lf;
        if constexpr (DIR) {
            for (unsigned bits = f; bits;) {
                unsigned long long hv[8];
#pragma unroll
                for (int i = 0; i < 8; ++i) {
                    hv[i] = 0ull;
                    if (bits) {
                        hv[i] = __ldg(a.head + w * 32 + __ffs(bits) - 1);
                        bits &= bits - 1;
                    }
                }
#pragma unroll
                for (int i = 0; i < 8; ++i) oedges += hv[i] >> 32;
            }
        }
    }, found, edges, probes, fmax, la);
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int o = 16; o; o >>= 1) {
        found += __shfl_xor_sync(FULL, found, o);
        edges += __shfl_xor_sync(FULL, edges, o);
        probes += __shfl_xor_sync(FULL, probes, o);
        if (LA) {
            la.found += __shfl_xor_sync(FULL, la.found, o);
            la.edges += __shfl_xor_sync(FULL, la.edges, o);
        }
    }
    k = *(const volatile int*)kp;
    // directed graph: the BU rows are in-arc rows, whose lengths are not the out-degrees
    // edgesF_{k+1} needs; those were summed from the out-arc head[] at publication
    if (DIR) {
        edges = oedges;
#pragma unroll
        for (int o = 16; o; o >>= 1) edges += __shfl_xor_sync(FULL, edges, o);
    }
    if (lane == 0 && (found | edges | probes)) {
        atomicAdd(&a.st->acc_found[k % 3], found);
        atomicAdd(&a.st->acc_edges[k % 3], edges);
        atomicAdd(&a.st->acc_probes[k % 3], probes);
    }
    if (LA && lane == 0 && la.found) {
        atomicAdd(&a.st->acc_la_found[k % 3], la.found);
        atomicAdd(&a.st->acc_la_edges[k % 3], la.edges);
    }
    if (a.track_max) {
        fmax = __reduce_max_sync(FULL, fmax);
        if (lane == 0 && fmax) atomic_max_if_greater(&a.st->qmax[(k + 1) % 3], fmax);
    }
}

// Look-ahead merge (persistent driver, after a BU step with look-ahead
// discoveries): F_{k+2} |= la, la = 0.  F_{k+2}'s bitmap was cleared during step
// k (the stale-map clear); the grid barrier that follows orders it before step k+1.
__device__ __forceinline__ void la_merge(const KArgs& a, int knext) {
    unsigned int* f2 = a.fb[(knext + 1) % 3];
    for (long long w = blockIdx.x * (long long)blockDim.x + threadIdx.x; w < a.words;
         w += (long long)gridDim.x * blockDim.x) {
        const unsigned x = __ldcg(a.la + w);
        if (x) {
            f2[w] = __ldcg(f2 + w) | x;
            a.la[w] = 0;
        }
    }
}

__global__ __launch_bounds__(kBuThreads, 4) void k_bu_traverse(KArgs a) {
    count_launch(a.st);
    __shared__ BuSmem<kBuThreads / 32> sm;
    bu_body<kBuThreads / 32, false>(a, &a.st->k, a.st->out_level, a.st->out_parent, sm, false, a.st->unvisited);
}

// ---------------------------------------------------------------- select
template <bool kGraph>
__global__ void k_select(KArgs a, cudaGraphConditionalHandle h_while) {
    count_launch(a.st);
    DevState* st = a.st;
    if (st->advanced) {             // k_small already ran its levels and advanced the state
        st->advanced = 0;
        if (kGraph) cudaGraphSetConditional(h_while, st->done ? 0u : 1u);
        return;
    }
    select_body(a);
    if (kGraph) cudaGraphSetConditional(h_while, st->done ? 0u : 1u);
}

// Small-frontier cluster mode gate: a scan-free level whose frontier has at most
// small_edges arcs and no vertex above kSmallMaxDeg (a hub would serialise a warp).
__host__ __device__ __forceinline__ bool small_gate(long long small_edges, int strategy, int queue_valid,
                                                    long long fedges, unsigned maxdeg) {
    return strategy == XBFS_SF && queue_valid && fedges <= small_edges && maxdeg <= (unsigned)kSmallMaxDeg;
}

__device__ __forceinline__ bool small_mode(const DevState* st, int strategy, int queue_valid, long long fedges,
                                           unsigned maxdeg) {
    return small_gate(st->small_edges, strategy, queue_valid, fedges, maxdeg);
}

// Device loop: map (strategy, queue_valid) of level k to a SWITCH branch.
__global__ void k_plan(KArgs a, cudaGraphConditionalHandle h_switch) {
    count_launch(a.st);
    const int s = a.st->strategy, qv = a.st->queue_valid;
    unsigned br = s == XBFS_BU ? 4u : (s == XBFS_SF ? (qv ? 0u : 1u) : (qv ? 2u : 3u));
    if (a.st->prev_small && small_mode(a.st, s, qv, a.st->fedges, a.st->fmaxdeg)) br = 5u;
    cudaGraphSetConditional(h_switch, br);
}

// --------------------------------------------------- small-frontier mode
// One thread-block cluster (kSmallCluster CTAs x 1024 threads) runs consecutive
// scan-free levels while edgesF_k <= small_edges: the level
// barrier is a cluster barrier (~hundreds of ns) instead of a kernel boundary +
// host round trip, which is what bounds the many tiny levels of a grid graph
// (small/many-level graphs are dominated by CPU-GPU interaction).
// Vertex-per-thread for deg <= kSmallInline (all arcs' loads in flight at once),
// warp-per-vertex (32 arcs per step) for the rest.  The frontier bitmaps keep the
// level kernels' invariant exactly but cheaply: winners RED their bit into
// fb[(k+1)%3], and the stale F_{k-1} bits are unset one by one from its queue
// (buffer (k+2)%3, untouched during level k) instead of clearing N/8 bytes.
__device__ __forceinline__ bool sf_claim(unsigned int* visited, int v) {
    const unsigned bit = 1u << (v & 31);
    if (__ldcg(visited + (v >> 5)) & bit) return false;
    return !(atomicOr(visited + (v >> 5), bit) & bit);
}

__global__ void __cluster_dims__(kSmallCluster, 1, 1) __launch_bounds__(kSmallThreads, 1) k_small_sf(KArgs a) {
    count_launch(a.st);
    int* __restrict__ level = a.st->out_level;
    int* __restrict__ parent = a.st->out_parent;
    cg::cluster_group cl = cg::this_cluster();
    const int crank = (int)cl.block_rank(), csize = (int)cl.num_blocks();
    DevState* st = a.st;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nwarps = blockDim.x >> 5;
    __shared__ int s_big[kSmallBig];
    __shared__ int s_nbig;
    int k = st->k;
    long long fsize = st->fsize, fedges = st->fedges, fprev = st->fprev, unvisited = st->unvisited;
    long long reached = st->reached, arcs_tr = st->arcs_traversed;
    unsigned fmaxdeg = st->fmaxdeg;
    bool done = false;
    int next_strat = XBFS_SF;
    const long long tid = (long long)crank * blockDim.x + threadIdx.x;
    const long long nth = (long long)csize * blockDim.x;
    cl.sync();                      // every CTA has read the state before CTA 0 touches it
    for (;;) {
        const int in = k % 3, ob = (k + 1) % 3;
        unsigned long long* octr = &st->qctr[(k + 1) % 3];
        unsigned* omax = &st->qmax[(k + 1) % 3];
        unsigned lmax = 0;
        unsigned int* next = a.fb[(k + 1) % 3];
        if (crank == 0 && threadIdx.x == 0) {
            st->qctr[(k + 2) % 3] = 0;
            st->qmax[(k + 2) % 3] = 0;
        }
        if (threadIdx.x == 0) s_nbig = 0;
        {   // unset the stale F_{k-1} bits (its queue is buffer (k+2)%3)
            unsigned int* stale = a.fb[(k + 2) % 3];
            const int* pq = a.qv[(k + 2) % 3];
            for (long long j = tid; j < fprev; j += nth) {
                const int v = pq[j];
                atomicAnd(stale + (v >> 5), ~(1u << (v & 31)));
            }
        }
        __syncthreads();
        const int* qv = a.qv[in];
        const long long* qoff = a.qoff[in];
        const long long* qdelta = a.qdelta[in];
        const int lvl = k + 1;
        const long long rounds = (fsize + nth - 1) / nth;
        for (long long r = 0; r < rounds; ++r) {
            const long long j = r * nth + tid;
            int u = 0;
            long long rs = 0, d = 0;
            if (j < fsize) {
                u = qv[j];
                const long long o = qoff[j];
                rs = o + qdelta[j];
                d = (j + 1 < fsize ? qoff[j + 1] : fedges) - o;
                if (d > kSmallInline) {
                    s_big[atomicAdd(&s_nbig, 1)] = (int)j;   // cannot overflow: small_edges <= 9*kSmallBig
                    d = 0;
                }
            }
            int v[kSmallInline];
            bool win[kSmallInline];
            long long vrs[kSmallInline], vdeg[kSmallInline];
#pragma unroll
            for (int i = 0; i < kSmallInline; ++i) v[i] = i < d ? __ldg(a.col + rs + i) : -1;
#pragma unroll
            for (int i = 0; i < kSmallInline; ++i) {
                win[i] = v[i] >= 0 && sf_claim(a.visited, v[i]);
                vrs[i] = 0;
                vdeg[i] = 0;
                if (win[i]) {
                    level[v[i]] = lvl;
                    parent[v[i]] = u;
                    atomicOr(next + (v[i] >> 5), 1u << (v[i] & 31));
                    vrs[i] = a.row_ptr[v[i]];
                    vdeg[i] = a.row_ptr[v[i] + 1];
                }
            }
#pragma unroll
            for (int i = 0; i < kSmallInline; ++i) vdeg[i] -= vrs[i];
            enqueue_warp_multi<kSmallInline>(win, v, vrs, vdeg, octr, lmax, a.dbits, a.qv[ob], a.qoff[ob], a.qdelta[ob],
                                             a.tile_first[ob]);
        }
        __syncthreads();
        const int nbig = s_nbig;
        for (int b = wid; b < nbig; b += nwarps) {
            const long long j = s_big[b];
            const int bu = qv[j];
            const long long o = qoff[j];
            const long long rs = o + qdelta[j];
            const long long d = (j + 1 < fsize ? qoff[j + 1] : fedges) - o;
            for (long long base = 0; base < d; base += 32) {
                const long long p = base + lane;
                const int v = p < d ? __ldg(a.col + rs + p) : -1;
                const bool w = v >= 0 && sf_claim(a.visited, v);
                long long vrs = 0, vdeg = 0;
                if (w) {
                    level[v] = lvl;
                    parent[v] = bu;
                    atomicOr(next + (v >> 5), 1u << (v & 31));
                    vrs = a.row_ptr[v];
                    vdeg = a.row_ptr[v + 1] - vrs;
                }
                enqueue_warp(w, v, vrs, vdeg, octr, lmax, a.dbits, a.qv[ob], a.qoff[ob], a.qdelta[ob],
                             a.tile_first[ob]);
            }
        }
        flush_max(omax, lmax);
        cl.sync();                  // level barrier: all claims and enqueues of level k are visible
        const unsigned long long q = atomicAdd(octr, 0ull);
        const unsigned nmax = atomicOr(omax, 0u);
        const long long nf = (long long)(q >> a.dbits);
        const long long ne = (long long)(q & ((1ull << a.dbits) - 1ull));
        if (crank == 0 && threadIdx.x == 0 && k < kLogCap) {
            LevelRec rec;
            rec.fsize = fsize;
            rec.fedges = fedges;
            rec.unvisited = unvisited;
            rec.probes = 0;
            rec.la_found = 0;
            rec.strategy = XBFS_SF;
            rec.pad = 0;
            rec.t_ns = 0;            // (no %globaltimer stamps outside the persistent driver)
            a.log[k] = rec;
        }
        reached += fsize;
        arcs_tr += fedges;
        fprev = fsize;
        unvisited -= nf;
        fsize = nf;
        fedges = ne;
        fmaxdeg = nmax;
        ++k;
        if (nf == 0) { done = true; break; }
        next_strat = choose_strategy(st, a.arcs, nf, fprev, ne, unvisited, XBFS_SF);
        if (!small_mode(st, next_strat, 1, ne, nmax)) break;
    }
    if (crank == 0 && threadIdx.x == 0) {
        st->k = k;
        st->strategy = next_strat;
        st->queue_valid = 1;
        st->done = done ? 1 : 0;
        if (done) st->nlevels = k;
        st->fsize = fsize;
        st->fedges = fedges;
        st->fprev = fprev;
        st->unvisited = unvisited;
        st->reached = reached;
        st->arcs_traversed = arcs_tr;
        st->prev_strategy = XBFS_SF;
        for (int i = 0; i < 3; ++i) st->acc_found[i] = st->acc_edges[i] = st->acc_probes[i] = st->acc_zero[i] = st->td_ctr[i] = 0;
        st->fmaxdeg = fmaxdeg;
        st->advanced = st->mirror_host ? 0 : 1;   // graph driver: its k_select node only mirrors
        st->prev_small = 1;
        mirror_host(a, st);
    }
}

// Graph500 m (O-6) = sum of tuple counts over reached vertices; untimed.
__global__ __launch_bounds__(256) void k_count_m(const int* __restrict__ level, const int* __restrict__ tcount,
                                                 long long n, unsigned long long* out) {
    unsigned long long s = 0;
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < n;
         v += (long long)gridDim.x * blockDim.x)
        if (level[v] >= 0) s += (unsigned long long)tcount[v];
    for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(FULL, s, o);
    if ((threadIdx.x & 31) == 0 && s) atomicAdd(out, s);
}

// ------------------------------------------------- persistent driver
// One cooperative launch per BFS: init, seed and every level run inside one
// kernel whose CTAs are all co-resident (cudaLaunchCooperativeKernel checks it),
// separated by grid barriers instead of kernel boundaries.  The level loop's
// fixed cost (~20 us per level through launches + a 1-thread select kernel, both
// for the host loop and the CUDA-graph loop, tools/level_floor.py) becomes one
// or two grid barriers.  Every CTA steps its own copy of the selector state from
// the same counters (deterministic), so the decision needs no extra barrier;
// CTA 0 also logs the level and its %globaltimer stamp.
__device__ __forceinline__ unsigned long long globaltimer() {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

// 1: release-add arrival + relaxed polling with backoff + one acquire fence
// (A/B: grid 77.2 vs 74.8 ms, s24 equal, so the SC-fence version stays default)
#ifndef XBFS_BARRIER_V2
#define XBFS_BARRIER_V2 0
#endif

__device__ __forceinline__ unsigned ld_acquire(const unsigned* p) {
    unsigned v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

// Grid barrier: monotonic arrival counter (zeroed with the state before the
// run); barrier e completes when it reaches e * gridDim.x.  __syncthreads +
// the release fence before the arrival and the acquire load after it order
// every write of the phase before every read of the next (mutable state is
// read through L2 everywhere).  A barrier that does not complete within 100 s
// traps: the run fails with a CUDA error (handle poisoned) instead of hanging.
__device__ __forceinline__ void grid_sync(unsigned* ctr, unsigned& epoch, int tl = -1, int ph0 = 0) {
    __syncthreads();
#if XBFS_TL_PROF
    if (threadIdx.x == 0) tl_rec(tl, ph0 + 1, globaltimer());
#else
    (void)tl;
#endif
    if (threadIdx.x == 0) {
        ++epoch;
        const unsigned target = epoch * gridDim.x;
#if XBFS_BARRIER_V2
        // arrival with release semantics (orders this CTA's phase writes, which
        // __syncthreads made visible to this thread, before the count); relaxed
        // polling (no L1 invalidation per poll); one acquire fence after it
        asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(ctr) : "memory");
        unsigned v;
        asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
        if ((int)(v - target) < 0) {
            const unsigned long long t0 = globaltimer();
            int polls = 0;
            do {
                if (++polls > 256) __nanosleep(256);
                if (globaltimer() - t0 > 100000000000ull) __trap();
                asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(ctr) : "memory");
            } while ((int)(v - target) < 0);
        }
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
#else
        __threadfence();
#if XBFS_TL_PROF
        tl_rec(tl, ph0 + 2, globaltimer());
#endif
        atomicAdd(ctr, 1u);
        if ((int)(ld_acquire(ctr) - target) < 0) {
            const unsigned long long t0 = globaltimer();
            while ((int)(ld_acquire(ctr) - target) < 0)
                if (globaltimer() - t0 > 100000000000ull) __trap();
        }
#endif
#if XBFS_TL_PROF
        tl_rec(tl, ph0 + 3, globaltimer());
#endif
    }
    __syncthreads();
}

// ------------------------------------------- tiny-frontier mode (f3)
// SURVEY §8(f) f3 inside the persistent driver: while a scan-free level's frontier
// is tiny (edgesF_k <= kTinyEdges, |F_k| <= kTinyCap), CTA 0 alone runs the
// consecutive levels with the queue of F_k in SHARED memory and __syncthreads as
// the level barrier; the other CTAs wait at one grid barrier and reload the
// selector state CTA 0 leaves behind.  A level then costs its own dependent
// round trips (col -> claim -> row_ptr) instead of those plus the global queue
// staging, the grid barrier and the counter read (small levels
// are dominated by synchronisation).  The bitmap invariant of the level loop is
// kept without N/8-byte clears: F_{k-1}'s bits are unset from its queue.
constexpr int kTinyCap = 2048;       // frontier vertices held in shared memory
constexpr int kTinyMaxDeg = 64;      // graphs up to this max degree run the TINY instantiation
constexpr int kTinyEdges = 2048;     // frontier arcs: one or two per thread of the 1024-thread CTA
constexpr int kTinyDbits = 44;       // packed smem counter: count << 44 | degree sum
// only from level 16 on: many-level graphs (grids, roads: P:L356) gain (B200, 4096^2 grid:
// 0.570 vs 0.561 GTEPS), while on Kronecker graphs (7-9 levels) the mode's entry and exit
// cost about what its few tiny levels save (s24 2x48 roots with it from level 0: 788 vs 800)
constexpr int kTinyMinLevel = 16;

struct TinySmem {
    int v[2][kTinyCap];
    long long rs[2][kTinyCap];
    long long off[2][kTinyCap + 1];  // exclusive prefix of degrees; off[F] = edgesF
    unsigned long long ctr;
};

__device__ __forceinline__ bool tiny_gate(const DevState* st, const SelState& s) {
    return s.k >= kTinyMinLevel && s.strategy == XBFS_SF && s.queue_valid && st->small_edges > 0 &&
           s.fedges <= kTinyEdges &&
           s.fedges <= st->small_edges && s.fsize <= kTinyCap;
}

// CTA 0 only (blockDim = kPersistThreads).  Entry: F_k in the global queue slot k%3.
// Exit (the gate fails or the BFS ends): the unexpanded F_k back in slot k%3, every
// other counter slot zeroed, the selector state stored for the other CTAs.
__device__ void tiny_levels(const KArgs& a, SelState& s, TinySmem& tm, int* __restrict__ level,
                            int* __restrict__ parent) {
    DevState* st = a.st;
    const int tid = threadIdx.x, lane = tid & 31;
    const unsigned lt = (1u << lane) - 1u;
    constexpr int NT = kPersistThreads;
    int k = s.k;
    int c = 0;
    {   // load F_k into buffer 0
        const int in = k % 3;
        const long long F = s.fsize;
        for (long long j = tid; j < F; j += NT) {
            tm.v[0][j] = __ldcg(a.qv[in] + j);
            const long long o = __ldcg(a.qoff[in] + j);
            tm.off[0][j] = o;
            tm.rs[0][j] = o + __ldcg(a.qdelta[in] + j);
        }
        if (tid == 0) tm.off[0][F] = s.fedges;
        // the stale map fb[(k+2)%3] holds F_{k-1}: unset from its queue (a top-down level
        // leaves it in slot (k+2)%3), else clear it whole (after a bottom-up level)
        if (k > 0) {
            unsigned* stale = a.fb[(k + 2) % 3];
            if (s.prev_strategy != XBFS_BU && s.fprev <= 8 * kTinyCap) {
                const int* pq = a.qv[(k + 2) % 3];
                for (long long j = tid; j < s.fprev; j += NT) {
                    const int v = __ldcg(pq + j);
                    atomicAnd(stale + (v >> 5), ~(1u << (v & 31)));
                }
            } else {
                uint4* z4 = reinterpret_cast<uint4*>(stale);
                for (long long i = tid; i < a.words / 4; i += NT) z4[i] = make_uint4(0, 0, 0, 0);
                for (long long i = a.words / 4 * 4 + tid; i < a.words; i += NT) stale[i] = 0;
            }
        }
    }
    __syncthreads();
    for (;;) {
        const long long F = s.fsize, T = s.fedges;
        const int lvl = k + 1;
        unsigned int* next = a.fb[(k + 1) % 3];
        if (tid == 0) tm.ctr = 0;
        __syncthreads();
        // expand: arc a of F_k owned by the last j with off[j] <= a (binary search in smem)
        constexpr int R = kTinyEdges / NT;
        bool win[R];
        int v[R], u[R];
        long long rs[R], deg[R];
#pragma unroll
        for (int i = 0; i < R; ++i) {
            const long long arc = tid + (long long)i * NT;
            v[i] = -1;
            u[i] = 0;
            if (arc < T) {
                int lo = 0, hi = (int)F - 1;
                while (lo < hi) {
                    const int mid = (lo + hi + 1) >> 1;
                    if (tm.off[c][mid] <= arc) lo = mid; else hi = mid - 1;
                }
                u[i] = tm.v[c][lo];
                v[i] = __ldg(a.col + tm.rs[c][lo] + (arc - tm.off[c][lo]));
            }
        }
        unsigned old[R];
#pragma unroll
        for (int i = 0; i < R; ++i) old[i] = v[i] >= 0 ? atomicOr(a.visited + (v[i] >> 5), 1u << (v[i] & 31)) : ~0u;
#pragma unroll
        for (int i = 0; i < R; ++i) {
            win[i] = v[i] >= 0 && !((old[i] >> (v[i] & 31)) & 1u);
            rs[i] = 0;
            deg[i] = 0;
            if (win[i]) {
                level[v[i]] = lvl;
                parent[v[i]] = u[i];
                atomicOr(next + (v[i] >> 5), 1u << (v[i] & 31));
                rs[i] = a.row_ptr[v[i]];
                deg[i] = a.row_ptr[v[i] + 1];
            }
        }
        // warp-aggregated append to the shared next queue: one smem atomic per warp on the
        // packed (count, degree sum) counter gives slots and exact degree offsets
        int cnt = 0;
        long long dsum = 0;
#pragma unroll
        for (int i = 0; i < R; ++i) {
            deg[i] -= rs[i];
            if (win[i]) { ++cnt; dsum += deg[i]; }
        }
        if (__any_sync(FULL, cnt > 0)) {
            int ic = cnt;
            long long id = dsum;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int tc = __shfl_up_sync(FULL, ic, o);
                const long long td = __shfl_up_sync(FULL, id, o);
                if (lane >= o) { ic += tc; id += td; }
            }
            const int wc = __shfl_sync(FULL, ic, 31);
            const long long wd = __shfl_sync(FULL, id, 31);
            unsigned long long base = 0;
            if (lane == 31) base = atomicAdd(&tm.ctr, ((unsigned long long)wc << kTinyDbits) + (unsigned long long)wd);
            base = __shfl_sync(FULL, base, 31);
            int slot = (int)(base >> kTinyDbits) + ic - cnt;
            long long off = (long long)(base & ((1ull << kTinyDbits) - 1ull)) + id - dsum;
#pragma unroll
            for (int i = 0; i < R; ++i) {
                if (!win[i]) continue;
                tm.v[c ^ 1][slot] = v[i];
                tm.rs[c ^ 1][slot] = rs[i];
                tm.off[c ^ 1][slot] = off;
                ++slot;
                off += deg[i];
            }
        }
        (void)lt;
        __syncthreads();
        const unsigned long long q = tm.ctr;
        const long long nf = (long long)(q >> kTinyDbits), ne = (long long)(q & ((1ull << kTinyDbits) - 1ull));
        // F_k's bits leave fb[k%3] now (nobody reads F_k's map at level k+1; it is that level's stale map)
        for (long long j = tid; j < F; j += NT) {
            const int w = tm.v[c][j];
            atomicAnd(a.fb[k % 3] + (w >> 5), ~(1u << (w & 31)));
        }
        if (tid == 0) {
            tm.off[c ^ 1][nf] = ne;
            if (k < kLogCap) {
                LevelRec r;
                r.fsize = F;
                r.fedges = T;
                r.unvisited = s.unvisited;
                r.probes = 0;
                r.la_found = 0;
                r.strategy = XBFS_SF;
                r.pad = 0;
                r.t_ns = globaltimer();
                a.log[k] = r;
            }
            s.reached += F;
            s.arcs_traversed += T;
            s.fprev = F;
            s.fsize = nf;
            s.fedges = ne;
            s.unvisited -= nf;
            s.prev_strategy = XBFS_SF;
            s.prev_small = 0;
            s.queue_valid = 1;
            s.k = k + 1;
            if (nf == 0) {
                s.done = 1;
                s.nlevels = k + 1;
            } else {
                s.strategy = choose_strategy(st, a.arcs, nf, F, ne, s.unvisited, XBFS_SF);
            }
        }
        __syncthreads();
        k = s.k;
        c ^= 1;
        if (s.done || !tiny_gate(st, s)) break;
    }
    // exit: the unexpanded F_k (buffer c) into the global queue slot k%3 for the level kernels
    if (!s.done) {
        const int ob = k % 3;
        const long long F = s.fsize;
        for (long long j = tid; j < F; j += NT) {
            const long long o = tm.off[c][j], d = tm.off[c][j + 1] - o;
            a.qv[ob][j] = tm.v[c][j];
            a.qoff[ob][j] = o;
            a.qdelta[ob][j] = tm.rs[c][j] - o;
            if (d > 0) {
                const long long t0 = (o + kTile - 1) / kTile, t1 = (o + d - 1) / kTile;
                for (long long t = t0; t <= t1; ++t) a.tile_first[ob][t] = (int)j;
            }
        }
    }
    if (tid == 0) {
        for (int i = 0; i < 3; ++i) {
            st->qctr[i] = i == k % 3 ? ((unsigned long long)s.fsize << a.dbits) + (unsigned long long)s.fedges : 0ull;
            st->qmax[i] = 0;
            st->acc_found[i] = st->acc_edges[i] = st->acc_probes[i] = st->acc_zero[i] = st->td_ctr[i] = 0;
            st->acc_la_found[i] = st->acc_la_edges[i] = 0;
        }
        sel_store(st, s);
    }
}

template <bool LA>
union PersistSmem {
    TinySmem tiny;
    TdSmemT<(XBFS_SS_TPT > XBFS_SF_TPT ? XBFS_SS_TPT : XBFS_SF_TPT)> td;
    typename std::conditional<LA, BuSmemLa<kPersistThreads / 32>, BuSmem<kPersistThreads / 32>>::type bu;
};

// LA: the BU look-ahead variant (a separate instantiation, so the default kernel
// carries none of its registers).
// DIR: directed graph (f4, reading R-9; also a separate instantiation).
// (level / parent are kernel parameters here, not loads from the state: parameters
// live in the constant bank, registers would be held across the whole kernel)
// TINY: the tiny-frontier mode is a separate instantiation, launched for graphs whose
// max degree is <= kTinyMaxDeg (grids, road-like graphs: the many-level ones); its mere
// presence in the Kronecker kernel cost 2.5 % (B200 A/B s24 2x48 roots: 788 vs 808
// GTEPS, code layout) although it never triggers there.
template <bool LA, bool DIR, bool TINY = false>
__global__ __launch_bounds__(kPersistThreads, kPersistBlocks) void k_persist(
    KArgs a, int* __restrict__ level, int* __restrict__ parent, const unsigned int* __restrict__ nonisolated,
    long long nonisolated_count) {
    extern __shared__ __align__(16) unsigned char dsm[];
    PersistSmem<LA>& sm = *reinterpret_cast<PersistSmem<LA>*>(dsm);
    __shared__ SelState s;
    unsigned epoch = 0;
    unsigned* bar = &a.st->bar_count;
    if (threadIdx.x == 0) atomicMin(&a.st->t_enter, globaltimer());
    count_launch(a.st);
    // the source's entries are written by the fill itself and the seed state by one
    // thread alongside it: one barrier for both
    init_body(a, level, parent, nonisolated, *(const volatile long long*)&a.st->source, LA);
    if (blockIdx.x == 0 && threadIdx.x == 0) seed_body(a, level, parent, nonisolated_count, nonisolated, true);
    grid_sync(bar, epoch);
    if (blockIdx.x == 0 && threadIdx.x == 0) a.st->t_start = globaltimer();
    if (threadIdx.x == 0) sel_load(a.st, s);
    __syncthreads();
    for (;;) {
        const int k = s.k, strat = s.strategy, qvalid = s.queue_valid;
        if (s.done) break;
#if XBFS_TL_PROF
        if (threadIdx.x == 0) tl_rec(k, 0, globaltimer());
#endif
        if (TINY && !LA && !DIR && tiny_gate(a.st, s)) {
            // tiny-frontier mode (f3): CTA 0 runs the levels, the others wait here once
            if (blockIdx.x == 0) tiny_levels(a, s, sm.tiny, level, parent);
            grid_sync(bar, epoch);
            if (threadIdx.x == 0 && blockIdx.x != 0) sel_load(a.st, s);
            __syncthreads();
            continue;
        }
        if (blockIdx.x == 0 && threadIdx.x == 0) {
            // slots nobody touches during level k (see select_body)
            a.st->qctr[(k + 2) % 3] = 0;
            a.st->qmax[(k + 2) % 3] = 0;
            a.st->acc_found[(k + 1) % 3] = a.st->acc_edges[(k + 1) % 3] = a.st->acc_probes[(k + 1) % 3] = 0;
            a.st->acc_zero[(k + 1) % 3] = 0;
            a.st->td_ctr[(k + 1) % 3] = 0;
            a.st->acc_la_found[(k + 1) % 3] = a.st->acc_la_edges[(k + 1) % 3] = 0;
        }
        if (strat != XBFS_BU && !qvalid) {
            generate_body(a, k, 0);
            grid_sync(bar, epoch);
        }
        if (strat == XBFS_SF) {
            // (directed: the queue holds |F_k| minus the sinks; read its own count)
            td_expand_body<XBFS_SF, kPersistThreads, XBFS_SF_TPT, DIR>(
                a, k, level, parent, *reinterpret_cast<TdSmemT<XBFS_SF_TPT>*>(&sm.td), DIR ? -1 : s.fsize,
                s.fedges);
        } else if (strat == XBFS_SS) {
            td_expand_body<XBFS_SS, kPersistThreads, XBFS_SS_TPT, DIR>(
                a, k, level, parent, *reinterpret_cast<TdSmemT<XBFS_SS_TPT>*>(&sm.td), DIR ? -1 : s.fsize,
                s.fedges);
            grid_sync(bar, epoch, k, 4);
            ss_count_body(a, k);
        } else {
            // (directed: bu_body sums edgesF_{k+1} over out-arcs itself)
            bu_body<kPersistThreads / 32, LA, decltype(sm.bu), DIR>(a, &s.k, level, parent, sm.bu, s.prefill,
                                                                   s.unvisited);
        }
        grid_sync(bar, epoch, k);
        if (threadIdx.x == 0) select_step(a, s, blockIdx.x == 0, blockIdx.x == 0 ? globaltimer() : 0ull);
        __syncthreads();
        if (LA && s.la_cf > 0) {    // look-ahead vertices of step k join F_{k+2} before step k+1
            la_merge(a, s.k);
            grid_sync(bar, epoch);
        }
        if (LA && s.qreset) {       // the regenerated queue of F_{k+1} restarts its counter
            if (blockIdx.x == 0 && threadIdx.x == 0) a.st->qctr[s.k % 3] = 0;
            grid_sync(bar, epoch);
        }
    }
    if (blockIdx.x == 0 && threadIdx.x == 0) sel_store(a.st, s);
}

// ------------------------------------------------------------- drivers
namespace {

struct Grids {
    int init, expand, gen, bu;
};

// One wave of resident blocks per kernel (grid-stride loops inside), sized from
// the occupancy calculator once per device.
Grids grids_for(const xbfs_graph* g) {
    static int occ[4] = {0, 0, 0, 0};
    if (!occ[0]) {
        int o = 0;
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, k_init_fill, 256, 0);
        occ[0] = std::max(o, 1);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, k_td_expand<XBFS_SF>, kExpandThreads, 0);
        occ[1] = std::max(o, 1);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, k_generate, kGenThreads, 0);
        occ[2] = std::max(o, 1);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, k_bu_traverse, kBuThreads, 0);
        occ[3] = std::max(o, 1);
    }
    // XBFS_GRID_{EXPAND,GEN,BU}: blocks per SM override (tuning experiments only)
    static int ov[3] = {-1, -1, -1};
    if (ov[0] < 0) {
        const char* names[3] = {"XBFS_GRID_EXPAND", "XBFS_GRID_GEN", "XBFS_GRID_BU"};
        for (int i = 0; i < 3; ++i) {
            const char* e = getenv(names[i]);
            ov[i] = e ? atoi(e) : 0;
        }
    }
    Grids r;
    r.init = g->num_sms * std::max(occ[0], 8);   // streaming fill: as many threads as fit
    r.expand = g->num_sms * (ov[0] > 0 ? ov[0] : occ[1]);
    r.gen = g->num_sms * (ov[1] > 0 ? ov[1] : occ[2]);
    r.bu = g->num_sms * (ov[2] > 0 ? ov[2] : occ[3]);
    return r;
}

// Optional per-launch event timing (xbfs_run_stats.kernel_capacity > 0), from the
// event pool the handle created at build time (at most kProfLaunches launches).
struct Prof {
    xbfs_graph* g = nullptr;
    xbfs_run_stats* st = nullptr;
    int n = 0;
    bool on() const {
        return st && st->kernel_capacity > 0 && n < st->kernel_capacity && 2 * (n + 1) <= (int)g->prof_events.size();
    }
    xbfs_status before() {
        if (!on()) return XBFS_OK;
        XBFS_CUDA(g, cudaEventRecord(g->prof_events[2 * n], g->stream));
        return XBFS_OK;
    }
    xbfs_status after(int id, int level) {
        if (!on()) return XBFS_OK;
        XBFS_CUDA(g, cudaEventRecord(g->prof_events[2 * n + 1], g->stream));
        if (st->kernel_id) st->kernel_id[n] = id;
        if (st->kernel_level) st->kernel_level[n] = level;
        ++n;
        return XBFS_OK;
    }
    xbfs_status finish() {
        if (!st || st->kernel_capacity <= 0) return XBFS_OK;
        st->num_kernels = n;
        for (int i = 0; i < n; ++i) {
            float ms = 0.f;
            XBFS_CUDA(g, cudaEventElapsedTime(&ms, g->prof_events[2 * i], g->prof_events[2 * i + 1]));
            if (st->kernel_ms) st->kernel_ms[i] = ms;
        }
        return XBFS_OK;
    }
};

#define XBFS_TRY(expr)                          \
    do {                                        \
        xbfs_status _s = (expr);                \
        if (_s != XBFS_OK) return _s;           \
    } while (0)

#define XBFS_LAUNCH(prof, id, lvl, launch)      \
    do {                                        \
        XBFS_TRY((prof).before());              \
        launch;                                 \
        XBFS_CUDA((prof).g, cudaGetLastError()); \
        XBFS_TRY((prof).after((id), (lvl)));    \
    } while (0)

// Enqueue one level given the host-known strategy / queue state.
xbfs_status launch_level(xbfs_graph* g, const KArgs& a, int k, int strat, int queue_valid, long long fedges,
                         unsigned maxdeg, int prev_small, long long small_edges, Prof& P) {
    const Grids G = grids_for(g);
    cudaStream_t s = g->stream;
    // The small-frontier kernel advances the level state itself (no k_select).
    if (prev_small && small_gate(small_edges, strat, queue_valid, fedges, maxdeg)) {
        XBFS_LAUNCH(P, XBFS_K_SMALL, k, (k_small_sf<<<kSmallCluster, kSmallThreads, 0, s>>>(a)));
        return XBFS_OK;
    }
    if (strat != XBFS_BU && !queue_valid)
        XBFS_LAUNCH(P, XBFS_K_GENERATE_PRE, k, (k_generate<<<G.gen, kGenThreads, 0, s>>>(a, 0)));
    if (strat == XBFS_SF) {
        XBFS_LAUNCH(P, XBFS_K_TD_SF, k, (k_td_expand<XBFS_SF><<<G.expand, kExpandThreads, 0, s>>>(a)));
    } else if (strat == XBFS_SS) {
        XBFS_LAUNCH(P, XBFS_K_TD_SS, k, (k_td_expand<XBFS_SS><<<G.expand, kExpandThreads, 0, s>>>(a)));
        XBFS_LAUNCH(P, XBFS_K_SS_COUNT, k, (k_ss_count<<<G.gen, kGenThreads, 0, s>>>(a)));
    } else {
        XBFS_LAUNCH(P, XBFS_K_BU, k, (k_bu_traverse<<<G.bu, kBuThreads, 0, s>>>(a)));
    }
    XBFS_LAUNCH(P, XBFS_K_SELECT, k, (k_select<false><<<1, 1, 0, s>>>(a, 0)));
    return XBFS_OK;
}

xbfs_status run_host_loop(xbfs_graph* g, const KArgs& a, long long small_edges, const int8_t* plan, int plan_len,
                          Prof& P) {
    // k_seed wrote hctl; wait for it, then one sync per level (P:L151's
    // host/device crossing, kept as the debug / measurement driver).
    XBFS_CUDA(g, cudaStreamSynchronize(g->stream));
    for (;;) {
        volatile HostCtl* h = g->hctl;
        if (h->done) break;
        int strat = h->strategy, prev_small = h->prev_small;
        const int k = h->k;
        if (k < plan_len) {
            prev_small = 0;   // planned levels always run through the level kernels
            if (plan[k] >= 0 && plan[k] != strat) {
                strat = plan[k];
                XBFS_CUDA(g, cudaMemcpyAsync(&g->st->strategy, &strat, sizeof(int), cudaMemcpyHostToDevice,
                                             g->stream));
            }
        }
        XBFS_TRY(launch_level(g, a, k, strat, h->queue_valid, h->fedges, h->fmaxdeg, prev_small, small_edges, P));
        XBFS_CUDA(g, cudaStreamSynchronize(g->stream));
    }
    return XBFS_OK;
}

// ------------------------------------------------- CUDA-graph device loop
// One graph per handle: init -> seed -> WHILE(!done) { plan -> SWITCH{SF | gen+SF |
// SS+count | gen+SS+count | BU | small} -> select }.  The kernels take
// the run's parameters and output pointers from the device state, so the graph is
// instantiated once (xbfs_build_csr / xbfs_reorder), never inside xbfs_run.  The
// strategy decision never leaves the device: one launch per BFS instead of one
// host/device crossing per level (the paper's P:L151 cost).
xbfs_status add_kernel(xbfs_graph* g, cudaGraph_t gr, cudaGraphNode_t* out, const cudaGraphNode_t* dep,
                       void* fn, int grid, int block, void** args) {
    cudaKernelNodeParams p = {};
    p.func = fn;
    p.gridDim = dim3(grid);
    p.blockDim = dim3(block);
    p.sharedMemBytes = 0;
    p.kernelParams = args;
    p.extra = nullptr;
    XBFS_CUDA(g, cudaGraphAddKernelNode(out, gr, dep, dep ? 1 : 0, &p));
    return XBFS_OK;
}

xbfs_status build_loop_graph(xbfs_graph* g) {
    if (g->loop_exec) {
        cudaGraphExecDestroy(g->loop_exec);
        g->loop_exec = nullptr;
    }
    const Grids G = grids_for(g);
    KArgs a = g->kargs();
    const unsigned int* noniso = g->nonisolated;
    long long nic = g->nonisolated_count;
    cudaGraph_t top = nullptr;
    XBFS_CUDA(g, cudaGraphCreate(&top, 0));
    struct Del { cudaGraph_t& t; ~Del() { if (t) cudaGraphDestroy(t); } } del{top};
    cudaGraphNode_t n_init, n_seed, n_while, n_plan, n_sw, n_sel, x, y;
    {
        void* args[] = {&a, &noniso};
        XBFS_TRY(add_kernel(g, top, &n_init, nullptr, (void*)k_init_fill, G.init, 256, args));
    }
    {
        void* args[] = {&a, &nic, &noniso};
        XBFS_TRY(add_kernel(g, top, &n_seed, &n_init, (void*)k_seed, 1, 1, args));
    }
    cudaGraphConditionalHandle h_while, h_switch;
    XBFS_CUDA(g, cudaGraphConditionalHandleCreate(&h_while, top, 1, cudaGraphCondAssignDefault));
    cudaGraphNodeParams wp = {};
    wp.type = cudaGraphNodeTypeConditional;
    wp.conditional.handle = h_while;
    wp.conditional.type = cudaGraphCondTypeWhile;
    wp.conditional.size = 1;
    XBFS_CUDA(g, cudaGraphAddNode(&n_while, top, &n_seed, 1, &wp));
    cudaGraph_t body = wp.conditional.phGraph_out[0];
    XBFS_CUDA(g, cudaGraphConditionalHandleCreate(&h_switch, body, 0, cudaGraphCondAssignDefault));
    {
        void* args[] = {&a, &h_switch};
        XBFS_TRY(add_kernel(g, body, &n_plan, nullptr, (void*)k_plan, 1, 1, args));
    }
    cudaGraphNodeParams sp = {};
    sp.type = cudaGraphNodeTypeConditional;
    sp.conditional.handle = h_switch;
    sp.conditional.type = cudaGraphCondTypeSwitch;
    sp.conditional.size = 6;
    XBFS_CUDA(g, cudaGraphAddNode(&n_sw, body, &n_plan, 1, &sp));
    cudaGraph_t* br = sp.conditional.phGraph_out;
    int role0 = 0;
    void* a_exp[] = {&a};
    void* a_gen0[] = {&a, &role0};
    void* f_sf = (void*)k_td_expand<XBFS_SF>;
    void* f_ss = (void*)k_td_expand<XBFS_SS>;
    void* f_gen = (void*)k_generate;
    void* f_cnt = (void*)k_ss_count;
    // 0: SF (queue valid)
    XBFS_TRY(add_kernel(g, br[0], &x, nullptr, f_sf, G.expand, kExpandThreads, a_exp));
    // 1: generate + SF
    XBFS_TRY(add_kernel(g, br[1], &x, nullptr, f_gen, G.gen, kGenThreads, a_gen0));
    XBFS_TRY(add_kernel(g, br[1], &y, &x, f_sf, G.expand, kExpandThreads, a_exp));
    // 2: SS + count (No-Frontier-Generation: the queue exists)
    XBFS_TRY(add_kernel(g, br[2], &x, nullptr, f_ss, G.expand, kExpandThreads, a_exp));
    XBFS_TRY(add_kernel(g, br[2], &y, &x, f_cnt, G.gen, kGenThreads, a_exp));
    // 3: generate + SS + count
    XBFS_TRY(add_kernel(g, br[3], &x, nullptr, f_gen, G.gen, kGenThreads, a_gen0));
    XBFS_TRY(add_kernel(g, br[3], &y, &x, f_ss, G.expand, kExpandThreads, a_exp));
    XBFS_TRY(add_kernel(g, br[3], &x, &y, f_cnt, G.gen, kGenThreads, a_exp));
    // 4: BU
    XBFS_TRY(add_kernel(g, br[4], &x, nullptr, (void*)k_bu_traverse, G.bu, kBuThreads, a_exp));
    // 5: small-frontier cluster mode (cluster dims are compiled into the kernel)
    XBFS_TRY(add_kernel(g, br[5], &x, nullptr, (void*)k_small_sf, kSmallCluster, kSmallThreads, a_exp));
    {
        void* args[] = {&a, &h_while};
        XBFS_TRY(add_kernel(g, body, &n_sel, &n_sw, (void*)k_select<true>, 1, 1, args));
    }
    XBFS_CUDA(g, cudaGraphInstantiate(&g->loop_exec, top, 0));
    return XBFS_OK;
}

xbfs_status launch_persist(xbfs_graph* g, const KArgs& a, int* level, int* parent, bool lookahead) {
    static int occ[4][64];
    static bool init[4][64] = {{false}};
    const bool tiny = !lookahead && !g->directed && g->max_deg <= kTinyMaxDeg;
    const int dev = g->device & 63, v = lookahead ? 1 : (g->directed ? 2 : (tiny ? 3 : 0));
    void* fn = lookahead ? (void*)k_persist<true, false>
                         : (g->directed ? (void*)k_persist<false, true>
                                        : (tiny ? (void*)k_persist<false, false, true> : (void*)k_persist<false, false>));
    const size_t smem = lookahead ? sizeof(PersistSmem<true>) : sizeof(PersistSmem<false>);
    if (!init[v][dev]) {
        XBFS_CUDA(g, cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
        int o = 0;
        XBFS_CUDA(g, cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, fn, kPersistThreads, smem));
        occ[v][dev] = o;
        init[v][dev] = true;
    }
    if (occ[v][dev] < 1) return set_error(XBFS_ERR_UNSUPPORTED, "persistent driver: k_persist does not fit on an SM");
    const int grid = g->num_sms * std::min(occ[v][dev], kPersistBlocks);
    const unsigned int* noniso = g->nonisolated;
    long long nic = g->nonisolated_count;
    KArgs ka = a;
    ka.track_max = 0;   // no small-frontier mode inside the persistent kernel
    void* args[] = {&ka, &level, &parent, &noniso, &nic};
    XBFS_CUDA(g, cudaLaunchCooperativeKernel(fn, dim3(grid), dim3(kPersistThreads), args, smem, g->stream));
    return XBFS_OK;
}

}  // namespace

// Everything a run needs beyond the CSR, created at build time so that xbfs_run
// never allocates: the CUDA-graph device loop (re-instantiated after
// every re-arrangement, which may move col), the host-output scratch slots and
// copy stream, and the per-launch profiling event pool.
xbfs_status prepare_drivers(xbfs_graph* g) {
    XBFS_TRY(build_loop_graph(g));
    if (!g->scratch_level) {
        XBFS_CUDA(g, cudaMalloc(&g->scratch_level, 2 * g->n * sizeof(int)));
        XBFS_CUDA(g, cudaMalloc(&g->scratch_parent, 2 * g->n * sizeof(int)));
    }
    if (!g->copy_stream) {
        XBFS_CUDA(g, cudaStreamCreateWithFlags(&g->copy_stream, cudaStreamNonBlocking));
        for (int s = 0; s < 2; ++s) {
            XBFS_CUDA(g, cudaEventCreateWithFlags(&g->ev_done[s], cudaEventDisableTiming));
            XBFS_CUDA(g, cudaEventCreateWithFlags(&g->ev_copied[s], cudaEventDisableTiming));
        }
    }
    while ((int)g->prof_events.size() < 2 * kProfLaunches) {
        cudaEvent_t e;
        XBFS_CUDA(g, cudaEventCreate(&e));
        g->prof_events.push_back(e);
    }
    return XBFS_OK;
}

}  // namespace xbfs

using namespace xbfs;

static xbfs_status run_impl(xbfs_graph* g, int64_t source, int32_t* level, int32_t* parent,
                            const xbfs_run_opts* opts, xbfs_run_stats* stats) {
    if (!g) return set_error(XBFS_ERR_INVALID_ARG, "xbfs_run: NULL handle");
    if (g->dist) return set_error(XBFS_ERR_STATE, "xbfs_run: a distributed handle runs with xbfs_run_dist");
    if (!level || !parent) return set_error(XBFS_ERR_INVALID_ARG, "xbfs_run: NULL level/parent");
    if (source < 0 || source >= g->n)
        return set_error(XBFS_ERR_INVALID_ARG, "xbfs_run: source %lld outside [0, %lld)", (long long)source, g->n);
    if (g->poisoned) return set_error(XBFS_ERR_STATE, "handle poisoned by an earlier failure");
    xbfs_run_opts o;
    xbfs_run_opts_default(&o);
    if (opts) o = *opts;
    if (o.force_strategy < -1 || o.force_strategy > 2)
        return set_error(XBFS_ERR_INVALID_ARG, "force_strategy must be -1..2");
    if (o.driver < 0 || o.driver > 3) return set_error(XBFS_ERR_INVALID_ARG, "driver must be 0..3");
    XBFS_CUDA(g, cudaSetDevice(g->device));

    KArgs a = g->kargs();
    const bool host_only = (stats && stats->kernel_capacity > 0) || (o.plan && o.plan_len > 0);
    const bool use_persist = (o.driver == 0 || o.driver == 3) && !host_only;
    const bool use_graph = o.driver == 2 && !host_only;
    if (g->directed && (!use_persist || o.lookahead))
        return set_error(XBFS_ERR_UNSUPPORTED,
                         "directed graphs run on the persistent driver only (driver 0/3, no plan, no per-launch "
                         "profiling, no look-ahead)");
    if (o.lookahead && !use_persist)
        return set_error(XBFS_ERR_INVALID_ARG, "lookahead needs the persistent driver (driver 0/3, no plan/profiling)");
    // selection parameters and output pointers live in the device state
    {
        // a pinned slot whose previous copy has executed (the ring is 4 runs deep)
        const int slot = g->stage_next;
        g->stage_next = (slot + 1) % xbfs_graph::kStageSlots;
        XBFS_CUDA(g, cudaEventSynchronize(g->ev_stage[slot]));
        DevState& hs = g->hstage[slot];
        memset(&hs, 0, sizeof(hs));
        hs.alpha = o.alpha;
        hs.grow = o.grow;
        hs.ratio_min = o.ratio_min;
        hs.bu_stay = o.bu_stay;
        hs.force = o.force_strategy;
        hs.source = source;
        hs.small_edges = std::min<long long>(std::max(o.small_edges, 0), kSmallEdgesMax);
        hs.mirror_host = (use_graph || use_persist) ? 0 : 1;
        hs.lookahead = o.lookahead ? 1 : 0;
        hs.out_level = level;
        hs.out_parent = parent;
        hs.t_enter = ~0ull;
        XBFS_CUDA(g, cudaMemcpyAsync(g->st, &hs, sizeof(hs), cudaMemcpyHostToDevice, g->stream));
        XBFS_CUDA(g, cudaEventRecord(g->ev_stage[slot], g->stream));
    }
    const Grids G = grids_for(g);
    Prof P;
    P.g = g;
    P.st = stats;
    if (use_persist) {
        XBFS_CUDA(g, cudaEventRecord(g->ev0, g->stream));
        XBFS_TRY(launch_persist(g, a, level, parent, o.lookahead != 0));
        XBFS_CUDA(g, cudaEventRecord(g->ev1, g->stream));
    } else if (use_graph) {
        XBFS_CUDA(g, cudaEventRecord(g->ev0, g->stream));
        XBFS_CUDA(g, cudaGraphLaunch(g->loop_exec, g->stream));
        XBFS_CUDA(g, cudaEventRecord(g->ev1, g->stream));
    } else {
        XBFS_CUDA(g, cudaEventRecord(g->ev0, g->stream));
        XBFS_LAUNCH(P, XBFS_K_INIT, -1, (k_init_fill<<<G.init, 256, 0, g->stream>>>(a, g->nonisolated)));
        XBFS_LAUNCH(P, XBFS_K_SEED, -1,
                    (k_seed<<<1, 1, 0, g->stream>>>(a, g->nonisolated_count, g->nonisolated)));
        XBFS_TRY(run_host_loop(g, a, std::min<long long>(std::max(o.small_edges, 0), kSmallEdgesMax), o.plan,
                               o.plan ? std::max(o.plan_len, 0) : 0, P));
        XBFS_CUDA(g, cudaEventRecord(g->ev1, g->stream));
    }

    if (stats) {
        XBFS_CUDA(g, cudaMemsetAsync(g->red_scratch, 0, sizeof(unsigned long long), g->stream));
        k_count_m<<<G.init, 256, 0, g->stream>>>(level, g->tcount, g->n, g->red_scratch);
        XBFS_CUDA(g, cudaGetLastError());
        DevState hs;
        unsigned long long m = 0;
        XBFS_CUDA(g, cudaMemcpyAsync(&hs, g->st, sizeof(hs), cudaMemcpyDeviceToHost, g->stream));
        XBFS_CUDA(g, cudaMemcpyAsync(&m, g->red_scratch, sizeof(m), cudaMemcpyDeviceToHost, g->stream));
        XBFS_CUDA(g, cudaStreamSynchronize(g->stream));
        float ms = 0.f;
        XBFS_CUDA(g, cudaEventElapsedTime(&ms, g->ev0, g->ev1));
        stats->elapsed_ms = ms;
        stats->num_levels = hs.nlevels;
        stats->vertices_reached = hs.reached;
        stats->arcs_traversed = hs.arcs_traversed;
        stats->input_edges_traversed = (int64_t)m;
        stats->kernel_launches = hs.launches;
#if XBFS_TL_PROF
        {
            unsigned long long tl[kTlLevels][8][2];
            cudaMemcpyFromSymbol(tl, g_tl, sizeof(tl));
            for (int k = 0; k < std::min(hs.nlevels, kTlLevels); ++k) {
                auto us = [&](unsigned long long t) { return t == ~0ull || t == 0 ? -1.0 : (double)(t - hs.t_start) * 1e-3; };
                fprintf(stderr, "TL %d start %.2f %.2f done %.2f %.2f fence %.2f %.2f pass %.2f %.2f", k,
                        us(tl[k][0][0]), us(tl[k][0][1]), us(tl[k][1][0]), us(tl[k][1][1]), us(tl[k][2][0]),
                        us(tl[k][2][1]), us(tl[k][3][0]), us(tl[k][3][1]));
                if (tl[k][5][1])
                    fprintf(stderr, " | mid done %.2f %.2f fence %.2f %.2f pass %.2f %.2f", us(tl[k][5][0]),
                            us(tl[k][5][1]), us(tl[k][6][0]), us(tl[k][6][1]), us(tl[k][7][0]), us(tl[k][7][1]));
                fprintf(stderr, "\n");
            }
            for (int k = 0; k < kTlLevels; ++k)
                for (int p = 0; p < 8; ++p) { tl[k][p][0] = ~0ull; tl[k][p][1] = 0; }
            cudaMemcpyToSymbol(g_tl, tl, sizeof(tl));
            static unsigned long long tw[kTlwLevels][5][kTlwWarps];
            cudaMemcpyFromSymbol(tw, g_tlw, sizeof(tw));
            for (int k = 0; k < std::min(hs.nlevels, kTlwLevels); ++k) {
                fprintf(stderr, "TLW %d", k);
                for (int p = 0; p < 5; ++p) {
                    unsigned long long mx = 0;
                    int arg = -1;
                    for (int w = 0; w < kTlwWarps; ++w)
                        if (tw[k][p][w] > mx && tw[k][p][w] >= hs.t_start) { mx = tw[k][p][w]; arg = w; }
                    fprintf(stderr, " p%d %.2f (w%d)", p, mx ? (double)(mx - hs.t_start) * 1e-3 : -1.0, arg);
                }
                fprintf(stderr, "\n");
            }
            memset(tw, 0, sizeof(tw));
            cudaMemcpyToSymbol(g_tlw, tw, sizeof(tw));
        }
#endif
#if XBFS_BU_PROF
        {
            unsigned long long pr[8];
            cudaMemcpyFromSymbol(pr, g_bu_prof, sizeof(pr));
            fprintf(stderr, "BUPROF scan %llu first %llu miss %llu hard %llu publish %llu nmiss %llu warps %llu maxwarp %llu\n",
                    pr[0], pr[1], pr[2], pr[3], pr[4], pr[5], pr[6], pr[7]);
            memset(pr, 0, sizeof(pr));
            cudaMemcpyToSymbol(g_bu_prof, pr, sizeof(pr));
        }
#endif
        // persistent driver: first CTA entry .. end of init + seed (%globaltimer)
        stats->init_ms = (use_persist && hs.t_enter != ~0ull && hs.t_start >= hs.t_enter)
                             ? (float)((hs.t_start - hs.t_enter) * 1e-6) : 0.f;
        XBFS_TRY(P.finish());
        const int nl = std::min(hs.nlevels, std::min(stats->level_capacity, kLogCap));
        if (nl > 0 && (stats->strategy || stats->frontier_vertices || stats->frontier_edges ||
                       stats->unvisited || stats->bu_probes || stats->level_ms || stats->lookahead_found)) {
            // the log is copied in slices through a fixed host buffer (no allocation per run)
            LevelRec rec[256];
            for (int i0 = 0; i0 < nl; i0 += 256) {
                const int cnt = std::min(256, nl - i0);
                XBFS_CUDA(g, cudaMemcpy(rec, g->log + i0, cnt * sizeof(LevelRec), cudaMemcpyDeviceToHost));
                for (int j = 0; j < cnt; ++j) {
                    const int i = i0 + j;
                    const LevelRec& r = rec[j];
                    if (stats->strategy) stats->strategy[i] = (int8_t)r.strategy;
                    if (stats->frontier_vertices) stats->frontier_vertices[i] = r.fsize;
                    if (stats->frontier_edges) stats->frontier_edges[i] = r.fedges;
                    if (stats->unvisited) stats->unvisited[i] = r.unvisited;
                    if (stats->bu_probes) stats->bu_probes[i] = r.probes;
                    if (stats->lookahead_found) stats->lookahead_found[i] = r.la_found;
                    if (stats->level_ms) {
                        unsigned long long t0 = hs.t_start;
                        if (i > 0) {
                            LevelRec prev;
                            if (j > 0) prev = rec[j - 1];
                            else XBFS_CUDA(g, cudaMemcpy(&prev, g->log + i - 1, sizeof(LevelRec), cudaMemcpyDeviceToHost));
                            t0 = prev.t_ns;
                        }
                        stats->level_ms[i] = (use_persist && r.t_ns >= t0 && t0) ? (float)((r.t_ns - t0) * 1e-6) : 0.f;
                    }
                }
            }
        }
    }
    return XBFS_OK;
}

extern "C" xbfs_status xbfs_run(xbfs_graph* g, int64_t source, int32_t* level, int32_t* parent,
                                const xbfs_run_opts* opts, xbfs_run_stats* stats) {
    return run_impl(g, source, level, parent, opts, stats);
}

// A failing host-output call must not return while copies it enqueued can still
// write into the caller's host buffers: drain both streams first (best effort).
static xbfs_status drain(xbfs_graph* g, xbfs_status s) {
    if (g->copy_stream) cudaStreamSynchronize(g->copy_stream);
    if (g->stream) cudaStreamSynchronize(g->stream);
    return s;
}

extern "C" xbfs_status xbfs_run_host_batch(xbfs_graph* g, const int64_t* sources, int32_t count, int32_t host_slots,
                                           int32_t* level_host, int32_t* parent_host, const xbfs_run_opts* opts) {
    if (!g) return set_error(XBFS_ERR_INVALID_ARG, "xbfs_run_host_batch: NULL handle");
    if (g->dist) return set_error(XBFS_ERR_STATE, "xbfs_run_host_batch: distributed handle");
    if (count < 0 || host_slots < 1) return set_error(XBFS_ERR_INVALID_ARG, "xbfs_run_host_batch: count < 0 or host_slots < 1");
    if (count == 0) return XBFS_OK;
    if (!sources || !level_host || !parent_host)
        return set_error(XBFS_ERR_INVALID_ARG, "xbfs_run_host_batch: NULL sources/level/parent");
    for (int32_t i = 0; i < count; ++i)
        if (sources[i] < 0 || sources[i] >= g->n)
            return set_error(XBFS_ERR_INVALID_ARG, "xbfs_run_host_batch: sources[%d] = %lld outside [0, %lld)", i,
                             (long long)sources[i], g->n);
    if (g->poisoned) return set_error(XBFS_ERR_STATE, "handle poisoned by an earlier failure");
    XBFS_CUDA(g, cudaSetDevice(g->device));
    const size_t bytes = (size_t)g->n * sizeof(int);
    for (int32_t i = 0; i < count; ++i) {
        const int s = i & 1;
        int* lv = g->scratch_level + (size_t)s * g->n;
        int* pa = g->scratch_parent + (size_t)s * g->n;
        cudaError_t e = cudaSuccess;
        // slot s is free once the D2H copies of BFS i-2 have drained
        if (i >= 2) e = cudaStreamWaitEvent(g->stream, g->ev_copied[s], 0);
        if (e != cudaSuccess) return drain(g, cuda_fail(g, e, "cudaStreamWaitEvent"));
        xbfs_status st = run_impl(g, sources[i], lv, pa, opts, nullptr);
        if (st != XBFS_OK) return drain(g, st);
        const size_t off = (size_t)(i % host_slots) * g->n;
        if ((e = cudaEventRecord(g->ev_done[s], g->stream)) != cudaSuccess ||
            (e = cudaStreamWaitEvent(g->copy_stream, g->ev_done[s], 0)) != cudaSuccess ||
            (e = cudaMemcpyAsync(level_host + off, lv, bytes, cudaMemcpyDeviceToHost, g->copy_stream)) != cudaSuccess ||
            (e = cudaMemcpyAsync(parent_host + off, pa, bytes, cudaMemcpyDeviceToHost, g->copy_stream)) != cudaSuccess ||
            (e = cudaEventRecord(g->ev_copied[s], g->copy_stream)) != cudaSuccess)
            return drain(g, cuda_fail(g, e, "xbfs_run_host_batch copy-back"));
    }
    XBFS_CUDA(g, cudaStreamSynchronize(g->copy_stream));
    XBFS_CUDA(g, cudaStreamSynchronize(g->stream));
    return XBFS_OK;
}

extern "C" xbfs_status xbfs_run_host(xbfs_graph* g, int64_t source, int32_t* level_host, int32_t* parent_host,
                                     const xbfs_run_opts* opts, xbfs_run_stats* stats) {
    if (!g) return set_error(XBFS_ERR_INVALID_ARG, "xbfs_run_host: NULL handle");
    if (g->dist) return set_error(XBFS_ERR_STATE, "xbfs_run_host: distributed handle");
    if (!level_host || !parent_host) return set_error(XBFS_ERR_INVALID_ARG, "xbfs_run_host: NULL level/parent");
    if (g->poisoned) return set_error(XBFS_ERR_STATE, "handle poisoned by an earlier failure");
    XBFS_CUDA(g, cudaSetDevice(g->device));
    xbfs_status s = run_impl(g, source, g->scratch_level, g->scratch_parent, opts, stats);
    if (s != XBFS_OK) return drain(g, s);
    XBFS_CUDA(g, cudaMemcpyAsync(level_host, g->scratch_level, g->n * sizeof(int), cudaMemcpyDeviceToHost, g->stream));
    XBFS_CUDA(g, cudaMemcpyAsync(parent_host, g->scratch_parent, g->n * sizeof(int), cudaMemcpyDeviceToHost, g->stream));
    XBFS_CUDA(g, cudaStreamSynchronize(g->stream));
    return XBFS_OK;
}
