// dist.cu — multi-GPU XBFS (include/xbfs_dist.h): 1D vertex partition, one
// process per GPU, the frontier exchange fused into the producing kernels as
// stores to peer memory (CUDA IPC; NVLink/NVSwitch between GPUs), the level loop
// and the per-level counter all-reduce inside xbfs_run_dist (comm.cu's host
// collectives; reading R-10).
//
// Per rank: owned rows [lo, lo+count) with global neighbour ids, a local visited
// bitmap over the owned range, three replicated N-bit frontier bitmaps and an
// inbox bitmap over the owned range (the last two live in one shared region that
// every peer maps).  Levels follow SURVEY §8(e); the per-level strategy rule is
// the paper's, evaluated on all-reduced counters so every rank agrees.
#include <cub/cub.cuh>

#include <algorithm>
#include <new>
#include <vector>

#include "bu_core.cuh"
#include "common.cuh"
#include "xbfs_dist.h"

#define XBFS_TRY_D(expr)                        \
    do {                                        \
        xbfs_status _s = (expr);                \
        if (_s != XBFS_OK) return _s;           \
    } while (0)

namespace xbfs {
namespace dist {

constexpr unsigned FULL = 0xffffffffu;
constexpr int kB = 256;
constexpr int kChunkArcs = 1024;     // TD work item: one vertex, up to 1024 arcs
constexpr unsigned long long kFirst = 1ull << 63;   // build key flag: the tuple's first endpoint is the row
constexpr unsigned long long kDrop = ~0ull;         // build key of a self-loop (sorted last, dropped)

struct DAcc {
    unsigned long long found, edges, m, probes;
    unsigned long long items;         // TD work items generated for the current level
    unsigned long long pad[3];
};

// Arguments of every dist kernel (flat, by value).
struct DArgs {
    const long long* row_ptr;        // local rows [count+1]
    const int* col;                  // global neighbour ids
    const unsigned long long* head;  // local: deg << 32 | first stored neighbour
    const int* tcount;               // local: tuples whose first endpoint is the vertex
    const unsigned* noniso;          // local words
    unsigned* vis;                   // local words (owned range)
    unsigned* fb[3];                 // local replicas, full N bits each
    unsigned* inbox;                 // local inbox (owned range)
    unsigned* peer_fb[XBFS_DIST_MAX_RANKS][3];
    unsigned* peer_inbox[XBFS_DIST_MAX_RANKS];
    unsigned long long* items;       // TD work items (v_local << 32 | chunk)
    DAcc* acc;
    int* level;                      // local
    int* parent;                     // local (global ids)
    long long n, lo, count, lo_w, cw, fwords, blk, blk_w;
    int rank, nranks;
};

__device__ __forceinline__ bool test_bit(const unsigned* bm, long long v) {
    return (__ldcg(bm + (v >> 5)) >> (v & 31)) & 1u;
}

__global__ __launch_bounds__(kB) void k_init(DArgs a) {
    const long long tid = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    const long long nth = (long long)gridDim.x * blockDim.x;
    for (long long i = tid; i < a.count; i += nth) { a.level[i] = -1; a.parent[i] = -1; }
    for (long long w = tid; w < a.cw; w += nth) { a.vis[w] = ~a.noniso[w]; a.inbox[w] = 0; }
    for (long long w = tid; w < a.fwords; w += nth) { a.fb[0][w] = 0; a.fb[1][w] = 0; a.fb[2][w] = 0; }
    if (tid == 0) *a.acc = DAcc{};
}

__global__ void k_seed(DArgs a, long long s) {
    a.fb[0][s >> 5] |= 1u << (s & 31);
    if (s >= a.lo && s < a.lo + a.count) {
        const long long vl = s - a.lo;
        a.level[vl] = 0;
        a.parent[vl] = (int)s;
        a.vis[vl >> 5] |= 1u << (vl & 31);
    }
}

// Store one owned word of F_{k+1} into every replica (local + peers): the
// all-gather, fused into the kernel that produced the word.
__device__ __forceinline__ void publish_word(const DArgs& a, int slot, long long w_local, unsigned word) {
    const long long gw = a.lo_w + w_local;
    a.fb[slot][gw] = word;
    for (int p = 0; p < a.nranks; ++p)
        if (p != a.rank) a.peer_fb[p][slot][gw] = word;
}

// First stored neighbour of local vertex vl that is in F_k (bitmap cur), or -1.
// probes counts arcs inspected (P:L131 early termination).
__device__ __forceinline__ int find_parent(const DArgs& a, const unsigned* cur, long long vl,
                                           unsigned long long& probes) {
    const unsigned long long hd = __ldg(a.head + vl);
    const long long d = (long long)(hd >> 32);
    if (d == 0) return -1;
    const int fu = (int)(unsigned)hd;
    if (test_bit(cur, fu)) { probes += 1; return fu; }
    const long long rs = a.row_ptr[vl];
    for (long long p = rs + 1; p < rs + d; p += 8) {
        int u[8];
#pragma unroll
        for (int j = 0; j < 8; ++j) u[j] = p + j < rs + d ? __ldg(a.col + p + j) : -1;
#pragma unroll
        for (int j = 0; j < 8; ++j)
            if (u[j] >= 0 && test_bit(cur, u[j])) { probes += (unsigned long long)(p + j - rs + 1); return u[j]; }
    }
    probes += (unsigned long long)d;
    return -1;
}

// ---------------------------------------------------------------- BU
// The single-GPU bottom-up core (bu_core.cuh) over the owned words; each owned
// word of F_{k+1} is published to every replica by the lane that owns it.
__global__ __launch_bounds__(kBuThreads, 4) void k_bu(DArgs a, int k) {
    const int slot = (k + 1) % 3;
    unsigned long long found = 0, edges = 0, m = 0, probes = 0;
    unsigned fmax = 0;
    // stale replica clear (F_{k-1}), full N bits, local only
    for (long long w = blockIdx.x * (long long)blockDim.x + threadIdx.x; w < a.fwords;
         w += (long long)gridDim.x * blockDim.x)
        a.fb[(k + 2) % 3][w] = 0;
    BuView b;
    b.cur = a.fb[k % 3];
    b.nxt = nullptr;
    b.visited = a.vis;
    b.words = a.cw;
    b.head = a.head;
    b.head32 = nullptr;
    b.idbits = 32;
    b.row_ptr = a.row_ptr;
    b.col = a.col;
    b.level = a.level;
    b.parent = a.parent;
    b.lvl = k + 1;
    b.reverse = false;
#if XBFS_BU_PROF
    b.prof = nullptr;
#endif
    __shared__ BuSmem<kBuThreads / 32> sm;
    BuLa la_unused;
    bu_chunks<kBuThreads / 32, false, false>(b, sm, [&](long long w, unsigned vis, unsigned f, unsigned) {
        publish_word(a, slot, w, f);
        if (f) {
            a.vis[w] = vis | f;
            for (unsigned bits = f; bits; bits &= bits - 1) m += (unsigned long long)a.tcount[w * 32 + __ffs(bits) - 1];
        }
    }, found, edges, probes, fmax, la_unused);
    for (int o = 16; o; o >>= 1) {
        found += __shfl_xor_sync(FULL, found, o);
        edges += __shfl_xor_sync(FULL, edges, o);
        m += __shfl_xor_sync(FULL, m, o);
        probes += __shfl_xor_sync(FULL, probes, o);
    }
    if ((threadIdx.x & 31) == 0 && (found | probes)) {
        atomicAdd(&a.acc->found, found);
        atomicAdd(&a.acc->edges, edges);
        atomicAdd(&a.acc->m, m);
        atomicAdd(&a.acc->probes, probes);
    }
}

// ---------------------------------------------------------------- TD
// Work items from the owned words of F_k: one item per 1024-arc chunk of a row.
__global__ __launch_bounds__(kB) void k_items(DArgs a, int k) {
    const unsigned* cur = a.fb[k % 3];
    const int lane = threadIdx.x & 31;
    const long long nth = (long long)gridDim.x * blockDim.x;
    for (long long w0 = blockIdx.x * (long long)blockDim.x + (threadIdx.x & ~31); w0 < a.cw; w0 += nth) {
        const long long w = w0 + lane;
        const unsigned word = w < a.cw ? __ldcg(cur + a.lo_w + w) : 0u;
        int cnt = 0;
        for (unsigned b = word; b; b &= b - 1) {
            const long long d = (long long)(__ldg(a.head + w * 32 + __ffs(b) - 1) >> 32);
            cnt += (int)((d + kChunkArcs - 1) / kChunkArcs);
        }
        int incl = cnt;
        for (int o = 1; o < 32; o <<= 1) {
            const int t = __shfl_up_sync(FULL, incl, o);
            if (lane >= o) incl += t;
        }
        const int tot = __shfl_sync(FULL, incl, 31);
        if (tot == 0) continue;
        unsigned long long base = 0;
        if (lane == 0) base = atomicAdd(&a.acc->items, (unsigned long long)tot);
        base = __shfl_sync(FULL, base, 0);
        unsigned long long pos = base + incl - cnt;
        for (unsigned b = word; b; b &= b - 1) {
            const long long vl = w * 32 + __ffs(b) - 1;
            const long long d = (long long)(__ldg(a.head + vl) >> 32);
            for (long long c = 0; c * kChunkArcs < d; ++c) a.items[pos++] = ((unsigned long long)vl << 32) | c;
        }
    }
}

// Warp per work item: owned neighbours are claimed with plain stores + RED
// (single-scan style); remote ones are OR-ed into the owner's inbox.
__global__ __launch_bounds__(kB) void k_td(DArgs a, int k) {
    const int lane = threadIdx.x & 31;
    const long long gw = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
    const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    const long long nitems = (long long)a.acc->items;
    unsigned* next = a.fb[(k + 1) % 3];
    const int lvl = k + 1;
    for (long long w = blockIdx.x * (long long)blockDim.x + threadIdx.x; w < a.fwords;
         w += (long long)gridDim.x * blockDim.x)
        a.fb[(k + 2) % 3][w] = 0;
    for (long long it = gw; it < nitems; it += nw) {
        const unsigned long long item = a.items[it];
        const long long ul = (long long)(item >> 32), c = (long long)(item & 0xffffffffu);
        const int ug = (int)(a.lo + ul);
        const long long rs = a.row_ptr[ul], re = a.row_ptr[ul + 1];
        const long long b0 = rs + c * kChunkArcs, b1 = min(re, b0 + kChunkArcs);
        for (long long p = b0 + lane; p < b1; p += 32) {
            const int v = __ldg(a.col + p);
            const unsigned bit = 1u << (v & 31);
            const long long vl = (long long)v - a.lo;
            if (vl >= 0 && vl < a.count) {
                if (!(__ldcg(a.vis + (vl >> 5)) & bit)) {
                    a.level[vl] = lvl;
                    a.parent[vl] = ug;
                    atomicOr(a.vis + (vl >> 5), bit);
                    atomicOr(next + (v >> 5), bit);
                }
            } else {
                const int o = (int)(v / a.blk);
                atomicOr(a.peer_inbox[o] + ((v >> 5) - (long long)o * a.blk_w), bit);
            }
        }
    }
}

// TD phase 1: inbox ∧ ¬visited are new owned frontier vertices; each finds its
// parent with a bottom-up probe against F_k (the first vertex of its row in F_k),
// then the owned F_{k+1} words go to every replica and are counted.
__global__ __launch_bounds__(kB) void k_merge(DArgs a, int k) {
    const unsigned* cur = a.fb[k % 3];
    const int slot = (k + 1) % 3;
    const int lvl = k + 1;
    unsigned long long found = 0, edges = 0, m = 0;
    for (long long w = blockIdx.x * (long long)blockDim.x + threadIdx.x; w < a.cw;
         w += (long long)gridDim.x * blockDim.x) {
        const unsigned in = a.inbox[w];
        unsigned vis = a.vis[w];
        const unsigned nw = in & ~vis;
        if (in) a.inbox[w] = 0;
        for (unsigned b = nw; b; b &= b - 1) {
            const int bit = __ffs(b) - 1;
            const long long vl = w * 32 + bit;
            unsigned long long pr = 0;
            const int par = find_parent(a, cur, vl, pr);
            a.level[vl] = lvl;
            a.parent[vl] = par;   // >= 0: the vertex was discovered from F_k
        }
        vis |= nw;
        if (nw) a.vis[w] = vis;
        const unsigned fin = a.fb[slot][a.lo_w + w] | nw;
        for (unsigned b = fin; b; b &= b - 1) {
            const long long vl = w * 32 + __ffs(b) - 1;
            edges += __ldg(a.head + vl) >> 32;
            m += (unsigned long long)a.tcount[vl];
            ++found;
        }
        if (fin) publish_word(a, slot, w, fin);   // zero words are zero in every replica
    }
    for (int o = 16; o; o >>= 1) {
        found += __shfl_xor_sync(FULL, found, o);
        edges += __shfl_xor_sync(FULL, edges, o);
        m += __shfl_xor_sync(FULL, m, o);
    }
    if ((threadIdx.x & 31) == 0 && found) {
        atomicAdd(&a.acc->found, found);
        atomicAdd(&a.acc->edges, edges);
        atomicAdd(&a.acc->m, m);
    }
}

// ---------------------------------------------------------------- build
// Pass 1 over this rank's tuples: per destination rank, how many arc keys go
// there (both directions of every tuple; a self-loop only once, for its tuple
// count).  Pass 2 writes the keys (row_local << nb | neighbour, kFirst on the
// tuple's first endpoint: tcount) into the destination's segment of the send
// buffer.  Ids out of range set *bad.
template <typename IdT, bool WRITE>
__global__ __launch_bounds__(kB) void k_route(const IdT* __restrict__ src, const IdT* __restrict__ dst, long long m,
                                              long long n, long long blk, int nb,
                                              unsigned long long* __restrict__ cursor,
                                              unsigned long long* __restrict__ keys, int* __restrict__ bad) {
    __shared__ unsigned long long s_cnt[XBFS_DIST_MAX_RANKS];
    if (!WRITE) {
        if (threadIdx.x < XBFS_DIST_MAX_RANKS) s_cnt[threadIdx.x] = 0;
        __syncthreads();
    }
    for (long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x; e < m;
         e += (long long)gridDim.x * blockDim.x) {
        const long long u = (long long)src[e], v = (long long)dst[e];
        if (u < 0 || v < 0 || u >= n || v >= n) { *bad = 1; continue; }
        const int ou = (int)(u / blk), ov = (int)(v / blk);
        if (!WRITE) {
            atomicAdd(&s_cnt[ou], 1ull);
            if (u != v) atomicAdd(&s_cnt[ov], 1ull);
        } else {
            keys[atomicAdd(&cursor[ou], 1ull)] =
                kFirst | ((unsigned long long)(u - (long long)ou * blk) << nb) | (unsigned long long)v;
            if (u != v)
                keys[atomicAdd(&cursor[ov], 1ull)] = ((unsigned long long)(v - (long long)ov * blk) << nb) |
                                                     (unsigned long long)u;
        }
    }
    if (!WRITE) {
        __syncthreads();
        if (threadIdx.x < XBFS_DIST_MAX_RANKS && s_cnt[threadIdx.x]) atomicAdd(&cursor[threadIdx.x], s_cnt[threadIdx.x]);
    }
}

// Received keys: count the tuples of every owned first endpoint (Graph500 m,
// O-6: duplicates and self-loops included), clear the flag, drop self-loops.
__global__ __launch_bounds__(kB) void k_strip(unsigned long long* __restrict__ keys, long long nk, long long lo, int nb,
                                              int* __restrict__ tcount) {
    const unsigned long long lowmask = (1ull << nb) - 1ull;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < nk;
         i += (long long)gridDim.x * blockDim.x) {
        unsigned long long key = keys[i];
        const long long row = (long long)((key & ~kFirst) >> nb);
        if (key & kFirst) atomicAdd(&tcount[row], 1);
        key &= ~kFirst;
        keys[i] = ((long long)(key & lowmask) == lo + row) ? kDrop : key;
    }
}

__global__ __launch_bounds__(kB) void k_split(const unsigned long long* __restrict__ keys, long long a,
                                              long long count, int nb, int* __restrict__ col,
                                              long long* __restrict__ row_ptr) {
    const unsigned long long lowmask = (1ull << nb) - 1ull;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < a;
         i += (long long)gridDim.x * blockDim.x) {
        const unsigned long long key = keys[i];
        const long long r = (long long)(key >> nb);
        col[i] = (int)(key & lowmask);
        const long long prev = i == 0 ? -1 : (long long)(keys[i - 1] >> nb);
        for (long long q = prev + 1; q <= r; ++q) row_ptr[q] = i;
        if (i == a - 1)
            for (long long q = r + 1; q <= count; ++q) row_ptr[q] = a;
    }
}

__global__ __launch_bounds__(kB) void k_fill64(long long* p, long long n, long long v) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n;
         i += (long long)gridDim.x * blockDim.x)
        p[i] = v;
}

__global__ __launch_bounds__(kB) void k_degrees(const long long* __restrict__ row_ptr, long long count,
                                                int* __restrict__ deg, unsigned* __restrict__ maxdeg) {
    unsigned mx = 0;
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < count;
         v += (long long)gridDim.x * blockDim.x) {
        const int d = (int)(row_ptr[v + 1] - row_ptr[v]);
        deg[v] = d;
        mx = max(mx, (unsigned)d);
    }
    for (int o = 16; o; o >>= 1) mx = max(mx, __shfl_xor_sync(FULL, mx, o));
    if ((threadIdx.x & 31) == 0 && mx) atomicMax(maxdeg, mx);
}

// Re-arrangement keys: (row << db) | (maxdeg - deg[col]); stable, so ties stay
// id-ascending: exactly xbfs_reorder's order (C-12) with true degrees.
__global__ __launch_bounds__(kB) void k_rkeys(const long long* __restrict__ row_ptr, const int* __restrict__ col,
                                              const int* __restrict__ deg_all, long long count, long long a, int db,
                                              unsigned long long maxdeg, unsigned long long* __restrict__ keys) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < a;
         i += (long long)gridDim.x * blockDim.x) {
        long long lo = 0, hi = count - 1;
        while (lo < hi) {
            const long long mid = (lo + hi + 1) >> 1;
            if (row_ptr[mid] <= i) lo = mid; else hi = mid - 1;
        }
        keys[i] = ((unsigned long long)lo << db) | (maxdeg - (unsigned long long)deg_all[col[i]]);
    }
}

__global__ __launch_bounds__(kB) void k_facts(const long long* __restrict__ row_ptr, const int* __restrict__ col,
                                              long long count, long long cw, unsigned* __restrict__ noniso,
                                              unsigned long long* __restrict__ head,
                                              unsigned long long* __restrict__ nnon) {
    unsigned long long c = 0;
    for (long long w = blockIdx.x * (long long)blockDim.x + threadIdx.x; w < cw;
         w += (long long)gridDim.x * blockDim.x) {
        unsigned bits = 0;
        for (int b = 0; b < 32; ++b) {
            const long long v = w * 32 + b;
            if (v >= count) break;
            const long long rs = row_ptr[v], d = row_ptr[v + 1] - rs;
            head[v] = ((unsigned long long)d << 32) | (d > 0 ? (unsigned)col[rs] : 0xffffffffu);
            if (d > 0) bits |= 1u << b;
        }
        noniso[w] = bits;
        c += __popc(bits);
    }
    for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(FULL, c, o);
    if ((threadIdx.x & 31) == 0 && c) atomicAdd(nnon, c);
}

inline int grid_for(long long n, int cap = 148 * 16) {
    long long g = (n + kB - 1) / kB;
    return (int)std::max(1ll, std::min<long long>(g, cap));
}

inline int bitlen(unsigned long long x) { return x ? 64 - __builtin_clzll(x) : 0; }

// host mirror of choose_strategy (bfs.cu): identical inputs on every rank
int choose(const xbfs_run_opts& o, long long arcs, long long fsize, long long fprev, long long fedges,
           long long unvisited, int prev) {
    if (o.force_strategy >= 0) return o.force_strategy;
    const double e = (double)fedges, A = (double)arcs;
    if (arcs > 0 && e > o.alpha * A) return XBFS_BU;                                          // P:L87, C-8
    if (o.bu_stay > 0.0 && prev == XBFS_BU && (double)unvisited * o.bu_stay < e) return XBFS_BU;   // C-11
    if ((double)fsize > o.grow * (double)fprev && arcs > 0 && e > o.ratio_min * A) return XBFS_SS; // C-10
    return XBFS_SF;
}

}  // namespace dist
}  // namespace xbfs

using namespace xbfs;
using namespace xbfs::dist;

// The multi-GPU part of a graph handle (xbfs_graph::dist).
struct xbfs_dist_part {
    xbfs_comm* comm = nullptr;
    int rank = 0, nranks = 1;
    long long n = 0, lo = 0, count = 0, blk = 0, arcs_local = 0, arcs_global = 0, fwords = 0, fwords_pad = 0,
              cw = 0, blk_w = 0;
    long long nonisolated_local = 0, nonisolated_global = 0;
    long long* row_ptr = nullptr;
    int* col = nullptr;
    unsigned long long* head = nullptr;
    int* tcount = nullptr;
    unsigned* noniso = nullptr;
    unsigned* vis = nullptr;
    unsigned* shared = nullptr;            // fb[0..2] + inbox, one allocation (IPC-exported)
    unsigned* peer_base[XBFS_DIST_MAX_RANKS] = {};
    unsigned long long* items = nullptr;
    long long items_cap = 0;
    DAcc* acc = nullptr;
    DAcc* acc_host = nullptr;               // pinned
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;

    unsigned* fb_of(unsigned* base, int i) const { return base + (long long)i * fwords_pad; }
    unsigned* inbox_of(unsigned* base) const { return base + 3 * fwords_pad; }
    DArgs args(int* level, int* parent) const {
        DArgs a;
        a.row_ptr = row_ptr;
        a.col = col;
        a.head = head;
        a.tcount = tcount;
        a.noniso = noniso;
        a.vis = vis;
        for (int i = 0; i < 3; ++i) a.fb[i] = fb_of(shared, i);
        a.inbox = inbox_of(shared);
        for (int p = 0; p < XBFS_DIST_MAX_RANKS; ++p) {
            unsigned* b = p < nranks ? (p == rank ? shared : peer_base[p]) : nullptr;
            for (int i = 0; i < 3; ++i) a.peer_fb[p][i] = b ? fb_of(b, i) : nullptr;
            a.peer_inbox[p] = b ? inbox_of(b) : nullptr;
        }
        a.items = items;
        a.acc = acc;
        a.level = level;
        a.parent = parent;
        a.n = n;
        a.lo = lo;
        a.count = count;
        a.lo_w = lo / 32;
        a.cw = cw;
        a.fwords = fwords;
        a.blk = blk;
        a.blk_w = blk_w;
        a.rank = rank;
        a.nranks = nranks;
        return a;
    }
};

namespace xbfs {
void dist_destroy(xbfs_dist_part* d) {
    if (!d) return;
    for (int p = 0; p < XBFS_DIST_MAX_RANKS; ++p)
        if (d->peer_base[p]) cudaIpcCloseMemHandle(d->peer_base[p]);
    void* ptrs[] = {d->row_ptr, d->col, d->head, d->tcount, d->noniso, d->vis, d->shared, d->items, d->acc};
    for (void* p : ptrs)
        if (p) cudaFree(p);
    if (d->acc_host) cudaFreeHost(d->acc_host);
    if (d->ev0) cudaEventDestroy(d->ev0);
    if (d->ev1) cudaEventDestroy(d->ev1);
    delete d;
}
}  // namespace xbfs

namespace {

#define DCUDA(g, call) XBFS_CUDA(g, call)
#define DTRY(expr) XBFS_TRY_D(expr)

// A device buffer every rank can see: allocate locally, all-gather the IPC
// handles, open the peers' (peer memory; the same device in the tests).
xbfs_status exchange_handles(xbfs_graph* g, xbfs_comm* c, void* mine, void** peers) {
    const int nr = comm_size(c), r = comm_rank(c);
    if (nr == 1) {
        peers[0] = mine;
        return XBFS_OK;
    }
    cudaIpcMemHandle_t h;
    memset(&h, 0, sizeof(h));
    if (mine) DCUDA(g, cudaIpcGetMemHandle(&h, mine));
    std::vector<cudaIpcMemHandle_t> all(nr);
    DTRY(comm_allgather(c, &h, sizeof(h), all.data()));
    for (int p = 0; p < nr; ++p) {
        peers[p] = nullptr;
        if (p == r) { peers[p] = mine; continue; }
        cudaIpcMemHandle_t z;
        memset(&z, 0, sizeof(z));
        if (!memcmp(&all[p], &z, sizeof(z))) continue;   // that rank had nothing to share
        DCUDA(g, cudaIpcOpenMemHandle(&peers[p], all[p], cudaIpcMemLazyEnablePeerAccess));
    }
    return XBFS_OK;
}

void close_handles(xbfs_comm* c, void** peers) {
    for (int p = 0; p < comm_size(c); ++p)
        if (p != comm_rank(c) && peers[p]) cudaIpcCloseMemHandle(peers[p]);
}

template <typename IdT>
xbfs_status route(xbfs_graph* g, xbfs_dist_part* d, const void* src, const void* dst, long long m, bool on_dev, int nb,
                  unsigned long long* cursor, unsigned long long* keys, int* bad, bool write) {
    const IdT* s = (const IdT*)src;
    const IdT* t = (const IdT*)dst;
    IdT *ds = nullptr, *dd = nullptr;
    const long long chunk = on_dev ? std::max(m, 1ll) : std::min<long long>(std::max(m, 1ll), 1ll << 27);
    if (!on_dev && m > 0) {
        DCUDA(g, cudaMalloc(&ds, chunk * sizeof(IdT)));
        DCUDA(g, cudaMalloc(&dd, chunk * sizeof(IdT)));
    }
    xbfs_status st = XBFS_OK;
    for (long long e0 = 0; e0 < m && st == XBFS_OK; e0 += chunk) {
        const long long cn = std::min(chunk, m - e0);
        const IdT* ps = s + e0;
        const IdT* pt = t + e0;
        if (!on_dev) {
            cudaMemcpyAsync(ds, ps, cn * sizeof(IdT), cudaMemcpyHostToDevice, g->stream);
            cudaMemcpyAsync(dd, pt, cn * sizeof(IdT), cudaMemcpyHostToDevice, g->stream);
            ps = ds;
            pt = dd;
        }
        if (write)
            k_route<IdT, true><<<grid_for(cn), kB, 0, g->stream>>>(ps, pt, cn, d->n, d->blk, nb, cursor, keys, bad);
        else
            k_route<IdT, false><<<grid_for(cn), kB, 0, g->stream>>>(ps, pt, cn, d->n, d->blk, nb, cursor, keys, bad);
        const cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) st = cuda_fail(g, e, "k_route");
    }
    if (st == XBFS_OK) {
        const cudaError_t e = cudaStreamSynchronize(g->stream);
        if (e != cudaSuccess) st = cuda_fail(g, e, "k_route sync");
    }
    if (ds) { cudaFree(ds); cudaFree(dd); }
    return st;
}

xbfs_status build_dist(xbfs_graph* g, xbfs_dist_part* d, const void* src, const void* dst, long long m,
                       const xbfs_build_opts& o) {
    xbfs_comm* c = d->comm;
    const int nr = d->nranks, me = d->rank;
    const long long n = d->n, count = d->count;
    const int nb_row = std::max(1, bitlen((unsigned long long)std::max(d->blk - 1, 1ll)));
    const int nb = std::max(1, bitlen((unsigned long long)(n - 1)));
    if (nb_row + nb > 63) return set_error(XBFS_ERR_UNSUPPORTED, "dist key does not fit in 63 bits");
    const bool on_dev = o.edges_on_device != 0;
    // 1. how many keys go to every rank (pass 1), all-gathered: row r = what rank r sends
    unsigned long long *cursor = nullptr, *sendk = nullptr;
    int* bad = nullptr;
    DCUDA(g, cudaMalloc(&cursor, XBFS_DIST_MAX_RANKS * sizeof(unsigned long long)));
    DCUDA(g, cudaMemsetAsync(cursor, 0, XBFS_DIST_MAX_RANKS * sizeof(unsigned long long), g->stream));
    DCUDA(g, cudaMalloc(&bad, sizeof(int)));
    DCUDA(g, cudaMemsetAsync(bad, 0, sizeof(int), g->stream));
    DTRY(o.id_bytes == 8 ? route<long long>(g, d, src, dst, m, on_dev, nb, cursor, nullptr, bad, false)
                         : route<unsigned>(g, d, src, dst, m, on_dev, nb, cursor, nullptr, bad, false));
    long long mine[XBFS_DIST_MAX_RANKS + 1] = {0};
    {
        unsigned long long hc[XBFS_DIST_MAX_RANKS];
        int hbad = 0;
        DCUDA(g, cudaMemcpy(hc, cursor, sizeof(hc), cudaMemcpyDeviceToHost));
        DCUDA(g, cudaMemcpy(&hbad, bad, sizeof(int), cudaMemcpyDeviceToHost));
        for (int p = 0; p < nr; ++p) mine[p] = (long long)hc[p];
        mine[XBFS_DIST_MAX_RANKS] = hbad;
    }
    std::vector<long long> cnt((size_t)nr * (XBFS_DIST_MAX_RANKS + 1));
    DTRY(comm_allgather(c, mine, sizeof(mine), cnt.data()));
    auto C = [&](int from, int to) { return cnt[(size_t)from * (XBFS_DIST_MAX_RANKS + 1) + to]; };
    for (int p = 0; p < nr; ++p)
        if (C(p, XBFS_DIST_MAX_RANKS)) {
            cudaFree(cursor); cudaFree(bad);
            return set_error(XBFS_ERR_INVALID_ARG, "edge id out of range [0, %lld) on rank %d", n, p);
        }
    long long send_total = 0, recv_total = 0;
    for (int p = 0; p < nr; ++p) { send_total += C(me, p); recv_total += C(p, me); }
    // 2. keys into per-destination segments of the send buffer (pass 2)
    std::vector<unsigned long long> start(XBFS_DIST_MAX_RANKS, 0);
    for (int p = 1; p < nr; ++p) start[p] = start[p - 1] + (unsigned long long)C(me, p - 1);
    DCUDA(g, cudaMemcpy(cursor, start.data(), XBFS_DIST_MAX_RANKS * sizeof(unsigned long long), cudaMemcpyHostToDevice));
    DCUDA(g, cudaMalloc(&sendk, std::max(send_total, 1ll) * sizeof(unsigned long long)));
    DTRY(o.id_bytes == 8 ? route<long long>(g, d, src, dst, m, on_dev, nb, cursor, sendk, bad, true)
                         : route<unsigned>(g, d, src, dst, m, on_dev, nb, cursor, sendk, bad, true));
    cudaFree(cursor);
    cudaFree(bad);
    // 3. ship every segment to its owner over peer memory: rank p's keys for me land at
    //    offset sum_{q<p} C(q, me) of my receive buffer (one rank: the send buffer is it)
    unsigned long long* recvk = nullptr;
    long long nk = recv_total;
    if (nr == 1) {
        recvk = sendk;
        sendk = nullptr;
    } else {
        DCUDA(g, cudaMalloc(&recvk, std::max(recv_total, 1ll) * sizeof(unsigned long long)));
        void* peers[XBFS_DIST_MAX_RANKS];
        DTRY(exchange_handles(g, c, recvk, peers));
        for (int p = 0; p < nr; ++p) {
            long long off = 0;
            for (int q = 0; q < me; ++q) off += C(q, p);
            if (C(me, p) == 0) continue;
            DCUDA(g, cudaMemcpyAsync((unsigned long long*)peers[p] + off, sendk + start[p],
                                     C(me, p) * sizeof(unsigned long long), cudaMemcpyDefault, g->stream));
        }
        DCUDA(g, cudaStreamSynchronize(g->stream));
        DTRY(comm_barrier(c));                  // every segment has landed everywhere
        close_handles(c, peers);
        cudaFree(sendk);
        sendk = nullptr;
        DTRY(comm_barrier(c));                  // nobody frees a buffer a peer still maps
    }
    // 4. tuple counts, self-loops dropped, sort, dedup (C-3), rows
    DCUDA(g, cudaMalloc(&d->tcount, std::max(count, 1ll) * sizeof(int)));
    DCUDA(g, cudaMemsetAsync(d->tcount, 0, std::max(count, 1ll) * sizeof(int), g->stream));
    DCUDA(g, cudaMalloc(&d->row_ptr, (count + 1) * sizeof(long long)));
    long long arcs = 0;
    if (nk > 0) {
        k_strip<<<grid_for(nk), kB, 0, g->stream>>>(recvk, nk, d->lo, nb, d->tcount);
        DCUDA(g, cudaGetLastError());
        unsigned long long* k1 = nullptr;
        DCUDA(g, cudaMalloc(&k1, nk * sizeof(unsigned long long)));
        cub::DoubleBuffer<unsigned long long> db(recvk, k1);
        size_t tb = 0;
        DCUDA(g, cub::DeviceRadixSort::SortKeys(nullptr, tb, db, nk, 0, 64, g->stream));
        void* tmp = nullptr;
        DCUDA(g, cudaMalloc(&tmp, tb));
        DCUDA(g, cub::DeviceRadixSort::SortKeys(tmp, tb, db, nk, 0, 64, g->stream));
        cudaFree(tmp);
        unsigned long long* sorted = db.Current();
        unsigned long long* other = db.Alternate();
        long long* nsel = nullptr;
        DCUDA(g, cudaMalloc(&nsel, sizeof(long long)));
        size_t ub = 0;
        DCUDA(g, cub::DeviceSelect::Unique(nullptr, ub, sorted, other, nsel, nk, g->stream));
        DCUDA(g, cudaMalloc(&tmp, ub));
        DCUDA(g, cub::DeviceSelect::Unique(tmp, ub, sorted, other, nsel, nk, g->stream));
        DCUDA(g, cudaMemcpyAsync(&arcs, nsel, sizeof(long long), cudaMemcpyDeviceToHost, g->stream));
        DCUDA(g, cudaStreamSynchronize(g->stream));
        cudaFree(tmp);
        cudaFree(nsel);
        if (arcs > 0) {                          // the self-loop sentinel sorts last
            unsigned long long last = 0;
            DCUDA(g, cudaMemcpy(&last, other + arcs - 1, sizeof(last), cudaMemcpyDeviceToHost));
            if (last == kDrop) --arcs;
        }
        DCUDA(g, cudaMalloc(&d->col, std::max(arcs, 1ll) * sizeof(int)));
        if (arcs > 0) {
            k_split<<<grid_for(arcs), kB, 0, g->stream>>>(other, arcs, count, nb, d->col, d->row_ptr);
        } else {
            k_fill64<<<grid_for(count + 1), kB, 0, g->stream>>>(d->row_ptr, count + 1, 0);
        }
        DCUDA(g, cudaGetLastError());
        DCUDA(g, cudaStreamSynchronize(g->stream));
        cudaFree(recvk);                         // both key buffers (sorted / other are these two)
        cudaFree(k1);
        recvk = nullptr;
    } else {
        DCUDA(g, cudaMalloc(&d->col, sizeof(int)));
        k_fill64<<<grid_for(count + 1), kB, 0, g->stream>>>(d->row_ptr, count + 1, 0);
        DCUDA(g, cudaGetLastError());
        if (recvk) cudaFree(recvk);
    }
    d->arcs_local = arcs;
    // 5. true degrees of every vertex (owned slices all-gathered over peer memory),
    //    then the re-arrangement of every owned row as xbfs_reorder does
    int* deg_all = nullptr;
    unsigned* mx = nullptr;
    DCUDA(g, cudaMalloc(&deg_all, ((long long)nr * d->blk) * sizeof(int)));
    DCUDA(g, cudaMalloc(&mx, sizeof(unsigned)));
    DCUDA(g, cudaMemsetAsync(mx, 0, sizeof(unsigned), g->stream));
    int* my_deg = deg_all + (long long)me * d->blk;
    if (count > 0) k_degrees<<<grid_for(count), kB, 0, g->stream>>>(d->row_ptr, count, my_deg, mx);
    DCUDA(g, cudaGetLastError());
    unsigned hmx = 0;
    DCUDA(g, cudaMemcpyAsync(&hmx, mx, sizeof(unsigned), cudaMemcpyDeviceToHost, g->stream));
    DCUDA(g, cudaStreamSynchronize(g->stream));
    cudaFree(mx);
    {
        void* peers[XBFS_DIST_MAX_RANKS];
        DTRY(exchange_handles(g, c, deg_all, peers));
        for (int p = 0; p < nr; ++p) {
            if (p == me || !peers[p]) continue;
            const long long plo = std::min<long long>(n, (long long)p * d->blk);
            const long long pc = std::max(0ll, std::min<long long>(d->blk, n - plo));
            if (pc > 0)
                DCUDA(g, cudaMemcpyAsync(deg_all + (long long)p * d->blk, (int*)peers[p] + (long long)p * d->blk,
                                         pc * sizeof(int), cudaMemcpyDefault, g->stream));
        }
        DCUDA(g, cudaStreamSynchronize(g->stream));
        DTRY(comm_barrier(c));
        close_handles(c, peers);
    }
    int64_t gl[4] = {arcs, (int64_t)hmx, 0, 0}, gsum[4];
    {
        std::vector<int64_t> allmx(nr * 4);
        DTRY(comm_allgather(c, gl, sizeof(gl), allmx.data()));
        gsum[0] = 0;
        gsum[1] = 0;
        for (int p = 0; p < nr; ++p) {
            gsum[0] += allmx[p * 4];
            gsum[1] = std::max<int64_t>(gsum[1], allmx[p * 4 + 1]);
        }
    }
    d->arcs_global = gsum[0];
    const unsigned long long maxdeg = (unsigned long long)gsum[1];
    g->max_deg = (int)maxdeg;
    if (arcs > 0) {
        const int dbits = std::max(1, bitlen(maxdeg));
        unsigned long long *r0 = nullptr, *r1 = nullptr;
        int* c1 = nullptr;
        DCUDA(g, cudaMalloc(&r0, arcs * sizeof(unsigned long long)));
        DCUDA(g, cudaMalloc(&r1, arcs * sizeof(unsigned long long)));
        DCUDA(g, cudaMalloc(&c1, arcs * sizeof(int)));
        k_rkeys<<<grid_for(arcs), kB, 0, g->stream>>>(d->row_ptr, d->col, deg_all, count, arcs, dbits, maxdeg, r0);
        DCUDA(g, cudaGetLastError());
        cub::DoubleBuffer<unsigned long long> dk(r0, r1);
        cub::DoubleBuffer<int> dv(d->col, c1);
        size_t tb = 0;
        DCUDA(g, cub::DeviceRadixSort::SortPairs(nullptr, tb, dk, dv, arcs, 0, nb_row + dbits, g->stream));
        void* tmp = nullptr;
        DCUDA(g, cudaMalloc(&tmp, tb));
        DCUDA(g, cub::DeviceRadixSort::SortPairs(tmp, tb, dk, dv, arcs, 0, nb_row + dbits, g->stream));
        DCUDA(g, cudaStreamSynchronize(g->stream));
        cudaFree(tmp);
        if (dv.Current() != d->col) { cudaFree(d->col); d->col = dv.Current(); } else { cudaFree(c1); }
        cudaFree(r0);
        cudaFree(r1);
    }
    DTRY(comm_barrier(c));                  // every peer has copied my degree slice
    cudaFree(deg_all);
    // 6. per-vertex facts, BFS state, the shared region every peer maps
    DCUDA(g, cudaMalloc(&d->head, std::max(count, 1ll) * sizeof(unsigned long long)));
    DCUDA(g, cudaMalloc(&d->noniso, std::max(d->cw, 1ll) * sizeof(unsigned)));
    DCUDA(g, cudaMalloc(&d->vis, std::max(d->cw, 1ll) * sizeof(unsigned)));
    DCUDA(g, cudaMalloc(&d->acc, sizeof(DAcc)));
    DCUDA(g, cudaMemsetAsync(d->acc, 0, sizeof(DAcc), g->stream));
    DCUDA(g, cudaHostAlloc(&d->acc_host, sizeof(DAcc), cudaHostAllocDefault));
    k_facts<<<grid_for(d->cw), kB, 0, g->stream>>>(d->row_ptr, d->col, count, d->cw, d->noniso, d->head,
                                                   &d->acc->found);
    DCUDA(g, cudaGetLastError());
    DCUDA(g, cudaMemcpyAsync(d->acc_host, d->acc, sizeof(DAcc), cudaMemcpyDeviceToHost, g->stream));
    DCUDA(g, cudaStreamSynchronize(g->stream));
    d->nonisolated_local = (long long)d->acc_host->found;
    DCUDA(g, cudaMemsetAsync(d->acc, 0, sizeof(DAcc), g->stream));
    {
        int64_t in[2] = {d->nonisolated_local, 0}, out[2];
        DTRY(comm_allreduce_sum(c, in, out, 2));
        d->nonisolated_global = out[0];
    }
    d->items_cap = arcs / kChunkArcs + count + 1;
    DCUDA(g, cudaMalloc(&d->items, d->items_cap * sizeof(unsigned long long)));
    const size_t sh = (3 * d->fwords_pad + d->blk_w) * sizeof(unsigned);
    DCUDA(g, cudaMalloc(&d->shared, sh));
    DCUDA(g, cudaMemsetAsync(d->shared, 0, sh, g->stream));
    DCUDA(g, cudaStreamSynchronize(g->stream));
    {
        void* peers[XBFS_DIST_MAX_RANKS];
        DTRY(exchange_handles(g, c, d->shared, peers));
        for (int p = 0; p < nr; ++p) d->peer_base[p] = p == me ? nullptr : (unsigned*)peers[p];
    }
    DCUDA(g, cudaEventCreate(&d->ev0));
    DCUDA(g, cudaEventCreate(&d->ev1));
    DTRY(comm_barrier(c));
    return XBFS_OK;
}

}  // namespace

extern "C" {

xbfs_status xbfs_build_csr_dist(xbfs_comm* c, const void* src, const void* dst, int64_t m, int64_t n,
                                const xbfs_build_opts* opts, xbfs_graph** out) {
    if (!out) return set_error(XBFS_ERR_INVALID_ARG, "xbfs_build_csr_dist: out is NULL");
    *out = nullptr;
    if (!c) return set_error(XBFS_ERR_INVALID_ARG, "xbfs_build_csr_dist: NULL comm");
    if (n <= 0 || n >= (1ll << 31)) return set_error(XBFS_ERR_INVALID_ARG, "num_vertices %lld out of (0, 2^31)", (long long)n);
    if (m < 0 || (m > 0 && (!src || !dst))) return set_error(XBFS_ERR_INVALID_ARG, "bad edge arrays");
    xbfs_build_opts o{};
    if (opts) o = *opts;
    if (o.id_bytes == 0) o.id_bytes = 4;
    if (o.id_bytes != 4 && o.id_bytes != 8) return set_error(XBFS_ERR_INVALID_ARG, "id_bytes must be 4 or 8");
    if (o.directed) return set_error(XBFS_ERR_UNSUPPORTED, "directed graphs are single-GPU only (xbfs_build_csr)");
    xbfs_graph* g = new (std::nothrow) xbfs_graph();
    xbfs_dist_part* d = new (std::nothrow) xbfs_dist_part();
    if (!g || !d) { delete g; delete d; return set_error(XBFS_ERR_OUT_OF_MEMORY, "host allocation failed"); }
    g->dist = d;
    struct Guard {
        xbfs_graph*& g;
        bool keep = false;
        ~Guard() { if (!keep) xbfs_destroy(g); }
    } guard{g};
    if (o.device >= 0) {
        XBFS_CUDA(g, cudaSetDevice(o.device));
        g->device = o.device;
    } else {
        XBFS_CUDA(g, cudaGetDevice(&g->device));
    }
    g->stream = (cudaStream_t)o.stream;
    XBFS_CUDA(g, cudaDeviceGetAttribute(&g->num_sms, cudaDevAttrMultiProcessorCount, g->device));
    d->comm = c;
    d->rank = comm_rank(c);
    d->nranks = comm_size(c);
    d->n = n;
    d->blk = ((n + 32LL * d->nranks - 1) / (32LL * d->nranks)) * 32;
    d->blk_w = d->blk / 32;
    d->lo = std::min<long long>(n, (long long)d->rank * d->blk);
    d->count = std::max(0ll, std::min<long long>(d->blk, n - d->lo));
    d->cw = (d->count + 31) / 32;
    d->fwords = (n + 31) / 32;
    d->fwords_pad = (d->fwords + 31) / 32 * 32;
    g->n = n;
    XBFS_TRY_D(build_dist(g, d, src, dst, m, o));
    {
        int64_t in[2] = {m, 0}, outv[2];
        XBFS_TRY_D(comm_allreduce_sum(c, in, outv, 2));
        g->m_input = outv[0];
    }
    g->arcs = d->arcs_global;
    guard.keep = true;
    *out = g;
    return XBFS_OK;
}

xbfs_status xbfs_partition_range(const xbfs_graph* g, int64_t* first, int64_t* count) {
    if (!g) return set_error(XBFS_ERR_INVALID_ARG, "xbfs_partition_range: NULL handle");
    if (!g->dist) {   // a single-GPU handle owns everything
        if (first) *first = 0;
        if (count) *count = g->n;
        return XBFS_OK;
    }
    if (first) *first = g->dist->lo;
    if (count) *count = g->dist->count;
    return XBFS_OK;
}

xbfs_status xbfs_run_dist(xbfs_graph* g, int64_t source, int32_t* level, int32_t* parent, const xbfs_run_opts* opts,
                          xbfs_run_stats* stats) {
    if (!g) return set_error(XBFS_ERR_INVALID_ARG, "xbfs_run_dist: NULL handle");
    xbfs_dist_part* d = g->dist;
    if (!d) return set_error(XBFS_ERR_STATE, "xbfs_run_dist: not a distributed handle (xbfs_build_csr_dist)");
    if (g->poisoned) return set_error(XBFS_ERR_STATE, "handle poisoned by an earlier failure");
    if ((!level || !parent) && d->count > 0) return set_error(XBFS_ERR_INVALID_ARG, "NULL level/parent");
    if (source < 0 || source >= d->n) return set_error(XBFS_ERR_INVALID_ARG, "source %lld outside [0, %lld)",
                                                       (long long)source, d->n);
    xbfs_run_opts o;
    xbfs_run_opts_default(&o);
    if (opts) o = *opts;
    if (o.force_strategy < -1 || o.force_strategy > 2)
        return set_error(XBFS_ERR_INVALID_ARG, "force_strategy must be -1..2");
    XBFS_CUDA(g, cudaSetDevice(g->device));
    xbfs_comm* c = d->comm;
    const DArgs a = d->args(level, parent);
    cudaStream_t s = g->stream;
    XBFS_CUDA(g, cudaEventRecord(d->ev0, s));
    k_init<<<grid_for(std::max(d->fwords, d->count)), kB, 0, s>>>(a);
    k_seed<<<1, 1, 0, s>>>(a, source);
    XBFS_CUDA(g, cudaGetLastError());
    // the source's facts from its owner: {owns, deg, tuples}; all ranks' sum
    int64_t cnt[4] = {0, 0, 0, 0}, gc[4];
    if (source >= d->lo && source < d->lo + d->count) {
        unsigned long long hd = 0;
        int t = 0;
        XBFS_CUDA(g, cudaMemcpyAsync(&hd, d->head + (source - d->lo), sizeof(hd), cudaMemcpyDeviceToHost, s));
        XBFS_CUDA(g, cudaMemcpyAsync(&t, d->tcount + (source - d->lo), sizeof(t), cudaMemcpyDeviceToHost, s));
        cnt[0] = 1;
        cnt[1] = (int64_t)(hd >> 32);
        cnt[2] = t;
    }
    XBFS_CUDA(g, cudaStreamSynchronize(s));
    XBFS_TRY_D(comm_allreduce_sum(c, cnt, gc, 4));      // also: every rank has seeded its replica
    long long fsize = gc[0], fedges = gc[1], m_total = gc[2], fprev = 0;
    long long unvisited = d->nonisolated_global - (gc[1] > 0 ? 1 : 0);
    long long reached = 0, arcs_tr = 0;
    int strategy = choose(o, d->arcs_global, fsize, 0, fedges, unvisited, -1);
    int k = 0;
    unsigned launches = 2;            // k_init, k_seed; then per level k_bu or k_items + k_td + k_merge
    const int grid = grid_for(std::max(d->fwords, d->cw) * 4, 148 * 8);
    const int cap = stats ? stats->level_capacity : 0;
    while (fsize > 0) {
        if (stats && k < cap) {
            if (stats->strategy) stats->strategy[k] = (int8_t)strategy;
            if (stats->frontier_vertices) stats->frontier_vertices[k] = fsize;
            if (stats->frontier_edges) stats->frontier_edges[k] = fedges;
            if (stats->unvisited) stats->unvisited[k] = unvisited;
        }
        XBFS_CUDA(g, cudaMemsetAsync(d->acc, 0, sizeof(DAcc), s));
        launches += strategy == XBFS_BU ? 1 : 3;
        if (strategy == XBFS_BU) {
            k_bu<<<g->num_sms * 5, kBuThreads, 0, s>>>(a, k);
        } else {
            k_items<<<grid, kB, 0, s>>>(a, k);
            k_td<<<grid, kB, 0, s>>>(a, k);
            XBFS_CUDA(g, cudaGetLastError());
            XBFS_CUDA(g, cudaStreamSynchronize(s));
            XBFS_TRY_D(comm_barrier(c));               // every remote discovery is in its owner's inbox
            k_merge<<<grid, kB, 0, s>>>(a, k);
        }
        XBFS_CUDA(g, cudaGetLastError());
        XBFS_CUDA(g, cudaMemcpyAsync(d->acc_host, d->acc, sizeof(DAcc), cudaMemcpyDeviceToHost, s));
        XBFS_CUDA(g, cudaStreamSynchronize(s));
        int64_t lc[4] = {(int64_t)d->acc_host->found, (int64_t)d->acc_host->edges, (int64_t)d->acc_host->m,
                         (int64_t)d->acc_host->probes};
        XBFS_TRY_D(comm_allreduce_sum(c, lc, gc, 4));  // also orders this level's peer stores before the next
        if (stats && k < cap && stats->bu_probes) stats->bu_probes[k] = strategy == XBFS_BU ? gc[3] : 0;
        reached += fsize;
        arcs_tr += fedges;
        fprev = fsize;
        fsize = gc[0];
        fedges = gc[1];
        m_total += gc[2];
        unvisited -= gc[0];
        ++k;
        if (fsize > 0) strategy = choose(o, d->arcs_global, fsize, fprev, fedges, unvisited, strategy);
    }
    XBFS_CUDA(g, cudaEventRecord(d->ev1, s));
    XBFS_CUDA(g, cudaEventSynchronize(d->ev1));
    if (stats) {
        float ms = 0.f;
        XBFS_CUDA(g, cudaEventElapsedTime(&ms, d->ev0, d->ev1));
        stats->elapsed_ms = ms;
        stats->num_levels = k;
        stats->vertices_reached = reached;
        stats->arcs_traversed = arcs_tr;
        stats->input_edges_traversed = m_total;
        stats->kernel_launches = launches;
        stats->num_kernels = 0;
        stats->init_ms = 0.f;
    }
    return XBFS_OK;
}

}  // extern "C"
