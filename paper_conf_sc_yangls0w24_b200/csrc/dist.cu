// dist.cu — multi-GPU XBFS (include/xbfs_dist.h): 1D vertex partition, one
// process per GPU, frontier exchange fused into the producing kernels as stores
// to peer memory (CUDA IPC; NVLink/NVSwitch between GPUs).
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

namespace xbfs {
namespace dist {

constexpr unsigned FULL = 0xffffffffu;
constexpr int kB = 256;
constexpr int kChunkArcs = 1024;     // TD work item: one vertex, up to 1024 arcs

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

__global__ __launch_bounds__(kB) void k_clear(unsigned* bm, long long words) {
    for (long long w = blockIdx.x * (long long)blockDim.x + threadIdx.x; w < words;
         w += (long long)gridDim.x * blockDim.x)
        bm[w] = 0;
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
// parent with a bottom-up probe against F_k, then the owned F_{k+1} words go to
// every replica and are counted.
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
template <typename IdT>
__global__ __launch_bounds__(kB) void k_pack_owned(const IdT* __restrict__ src, const IdT* __restrict__ dst,
                                                   long long m, long long n, long long lo, long long count, int nb,
                                                   unsigned long long* __restrict__ keys,
                                                   unsigned long long* __restrict__ nkeys, int* __restrict__ inc,
                                                   int* __restrict__ tcount, int* __restrict__ bad) {
    for (long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x; e < m;
         e += (long long)gridDim.x * blockDim.x) {
        const long long u = (long long)src[e], v = (long long)dst[e];
        if (u < 0 || v < 0 || u >= n || v >= n) { *bad = 1; continue; }
        const bool ou = u >= lo && u < lo + count, ov = v >= lo && v < lo + count;
        if (ou) atomicAdd(&tcount[u - lo], 1);
        if (u == v) continue;
        atomicAdd(&inc[u], 1);
        atomicAdd(&inc[v], 1);
        if (ou) keys[atomicAdd(nkeys, 1ull)] = ((unsigned long long)(u - lo) << nb) | (unsigned long long)v;
        if (ov) keys[atomicAdd(nkeys, 1ull)] = ((unsigned long long)(v - lo) << nb) | (unsigned long long)u;
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

// Reorder keys: (row << db) | (maxinc - inc[col]); stable, so ties stay id-ascending.
__global__ __launch_bounds__(kB) void k_rkeys(const long long* __restrict__ row_ptr, const int* __restrict__ col,
                                              const int* __restrict__ inc, long long count, long long a, int db,
                                              unsigned long long maxinc, unsigned long long* __restrict__ keys) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < a;
         i += (long long)gridDim.x * blockDim.x) {
        long long lo = 0, hi = count - 1;
        while (lo < hi) {
            const long long mid = (lo + hi + 1) >> 1;
            if (row_ptr[mid] <= i) lo = mid; else hi = mid - 1;
        }
        keys[i] = ((unsigned long long)lo << db) | (maxinc - (unsigned long long)inc[col[i]]);
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

__global__ __launch_bounds__(kB) void k_maxinc(const int* __restrict__ inc, long long n, unsigned* out) {
    unsigned mx = 0;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n;
         i += (long long)gridDim.x * blockDim.x)
        mx = max(mx, (unsigned)inc[i]);
    for (int o = 16; o; o >>= 1) mx = max(mx, __shfl_xor_sync(FULL, mx, o));
    if ((threadIdx.x & 31) == 0) atomicMax(out, mx);
}

inline int grid_for(long long n, int cap = 148 * 16) {
    long long g = (n + kB - 1) / kB;
    return (int)std::max(1ll, std::min<long long>(g, cap));
}

inline int bitlen(unsigned long long x) { return x ? 64 - __builtin_clzll(x) : 0; }

}  // namespace dist
}  // namespace xbfs

using namespace xbfs;
using namespace xbfs::dist;

struct xbfs_dist {
    int device = 0;
    cudaStream_t stream = nullptr;
    bool poisoned = false;
    int rank = 0, nranks = 1;
    long long n = 0, lo = 0, count = 0, blk = 0, arcs = 0, fwords = 0, fwords_pad = 0, cw = 0, blk_w = 0;
    long long nonisolated_local = 0;
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
    DAcc* acc_host = nullptr;
    bool attached = false;
    // current BFS
    int* level = nullptr;
    int* parent = nullptr;
    int k = 0, strategy = 0, started = 0;
    long long fsize = 0, fedges = 0, fprev = 0, unvisited = 0, m_total = 0, arcs_global = 0;
    xbfs_run_opts opts;
    std::vector<int8_t> log_s;
    std::vector<long long> log_f, log_e;

    unsigned* fb_of(unsigned* base, int i) const { return base + (long long)i * fwords_pad; }
    unsigned* inbox_of(unsigned* base) const { return base + 3 * fwords_pad; }
    DArgs args() const {
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

namespace {

xbfs_status dfail(xbfs_dist* d, cudaError_t e, const char* what) {
    if (d) d->poisoned = true;
    return cuda_fail(nullptr, e, what);
}

#define DCUDA(d, call)                                              \
    do {                                                            \
        cudaError_t _e = (call);                                    \
        if (_e != cudaSuccess) return dfail((d), _e, #call);        \
    } while (0)

// host mirror of choose_strategy (bfs.cu): identical inputs on every rank
int choose(const xbfs_run_opts& o, long long arcs, long long fsize, long long fprev, long long fedges,
           long long unvisited, int prev) {
    if (o.force_strategy >= 0) return o.force_strategy;
    const double ratio = arcs > 0 ? (double)fedges / (double)arcs : 0.0;
    if (ratio > o.alpha) return XBFS_BU;
    if (o.bu_stay > 0.0 && prev == XBFS_BU && (double)unvisited * o.bu_stay < (double)fedges) return XBFS_BU;
    if ((double)fsize > o.grow * (double)fprev && ratio > o.ratio_min) return XBFS_SS;
    return XBFS_SF;
}

template <typename IdT>
xbfs_status pack(xbfs_dist* d, const void* src, const void* dst, long long m, bool on_dev, int nb,
                 unsigned long long* keys, unsigned long long* nkeys, int* inc, int* bad) {
    const IdT* s = (const IdT*)src;
    const IdT* t = (const IdT*)dst;
    IdT *ds = nullptr, *dd = nullptr;
    const long long chunk = on_dev ? std::max(m, 1ll) : std::min<long long>(std::max(m, 1ll), 1ll << 27);
    if (!on_dev && m > 0) {
        DCUDA(d, cudaMalloc(&ds, chunk * sizeof(IdT)));
        DCUDA(d, cudaMalloc(&dd, chunk * sizeof(IdT)));
    }
    for (long long e0 = 0; e0 < m; e0 += chunk) {
        const long long c = std::min(chunk, m - e0);
        const IdT* ps = s + e0;
        const IdT* pt = t + e0;
        if (!on_dev) {
            DCUDA(d, cudaMemcpyAsync(ds, ps, c * sizeof(IdT), cudaMemcpyHostToDevice, d->stream));
            DCUDA(d, cudaMemcpyAsync(dd, pt, c * sizeof(IdT), cudaMemcpyHostToDevice, d->stream));
            ps = ds;
            pt = dd;
        }
        k_pack_owned<IdT><<<grid_for(c), kB, 0, d->stream>>>(ps, pt, c, d->n, d->lo, d->count, nb, keys, nkeys,
                                                            inc, d->tcount, bad);
        DCUDA(d, cudaGetLastError());
    }
    DCUDA(d, cudaStreamSynchronize(d->stream));
    if (ds) { cudaFree(ds); cudaFree(dd); }
    return XBFS_OK;
}

xbfs_status build_impl(xbfs_dist* d, const void* src, const void* dst, long long m, const xbfs_build_opts& o) {
    const long long n = d->n, count = d->count;
    const int nb_row = std::max(1, bitlen((unsigned long long)std::max(count - 1, 1ll)));
    const int nb = std::max(1, bitlen((unsigned long long)(n - 1)));
    if (nb_row + nb > 64) return set_error(XBFS_ERR_UNSUPPORTED, "dist key does not fit in 64 bits");
    int* inc = nullptr;
    int* bad = nullptr;
    unsigned long long *k0 = nullptr, *k1 = nullptr, *nkeys = nullptr;
    DCUDA(d, cudaMalloc(&inc, n * sizeof(int)));
    DCUDA(d, cudaMemsetAsync(inc, 0, n * sizeof(int), d->stream));
    DCUDA(d, cudaMalloc(&d->tcount, std::max(count, 1ll) * sizeof(int)));
    DCUDA(d, cudaMemsetAsync(d->tcount, 0, std::max(count, 1ll) * sizeof(int), d->stream));
    DCUDA(d, cudaMalloc(&bad, sizeof(int)));
    DCUDA(d, cudaMemsetAsync(bad, 0, sizeof(int), d->stream));
    DCUDA(d, cudaMalloc(&nkeys, sizeof(unsigned long long)));
    DCUDA(d, cudaMemsetAsync(nkeys, 0, sizeof(unsigned long long), d->stream));
    // upper bound on owned arcs: 2 per tuple
    const long long cap = std::max(2 * m, 1ll);
    DCUDA(d, cudaMalloc(&k0, cap * sizeof(unsigned long long)));
    const bool on_dev = o.edges_on_device != 0;
    xbfs_status st = o.id_bytes == 8 ? pack<long long>(d, src, dst, m, on_dev, nb, k0, nkeys, inc, bad)
                                     : pack<unsigned int>(d, src, dst, m, on_dev, nb, k0, nkeys, inc, bad);
    if (st != XBFS_OK) return st;
    int hbad = 0;
    unsigned long long hk = 0;
    DCUDA(d, cudaMemcpy(&hbad, bad, sizeof(int), cudaMemcpyDeviceToHost));
    DCUDA(d, cudaMemcpy(&hk, nkeys, sizeof(hk), cudaMemcpyDeviceToHost));
    if (hbad) {
        cudaFree(inc); cudaFree(bad); cudaFree(k0); cudaFree(nkeys);
        return set_error(XBFS_ERR_INVALID_ARG, "edge id out of range [0, %lld)", n);
    }
    long long nk = (long long)hk;
    DCUDA(d, cudaMalloc(&k1, std::max(nk, 1ll) * sizeof(unsigned long long)));
    long long arcs = 0;
    d->row_ptr = nullptr;
    DCUDA(d, cudaMalloc(&d->row_ptr, (count + 1) * sizeof(long long)));
    if (nk > 0) {
        cub::DoubleBuffer<unsigned long long> db(k0, k1);
        size_t tb = 0;
        DCUDA(d, cub::DeviceRadixSort::SortKeys(nullptr, tb, db, nk, 0, nb_row + nb, d->stream));
        void* tmp = nullptr;
        DCUDA(d, cudaMalloc(&tmp, tb));
        DCUDA(d, cub::DeviceRadixSort::SortKeys(tmp, tb, db, nk, 0, nb_row + nb, d->stream));
        cudaFree(tmp);
        unsigned long long* sorted = db.Current();
        unsigned long long* other = db.Alternate();
        long long* nsel = nullptr;
        DCUDA(d, cudaMalloc(&nsel, sizeof(long long)));
        size_t ub = 0;
        DCUDA(d, cub::DeviceSelect::Unique(nullptr, ub, sorted, other, nsel, nk, d->stream));
        DCUDA(d, cudaMalloc(&tmp, ub));
        DCUDA(d, cub::DeviceSelect::Unique(tmp, ub, sorted, other, nsel, nk, d->stream));
        DCUDA(d, cudaMemcpyAsync(&arcs, nsel, sizeof(long long), cudaMemcpyDeviceToHost, d->stream));
        DCUDA(d, cudaStreamSynchronize(d->stream));
        cudaFree(tmp);
        cudaFree(nsel);
        DCUDA(d, cudaMalloc(&d->col, std::max(arcs, 1ll) * sizeof(int)));
        k_split<<<grid_for(arcs), kB, 0, d->stream>>>(other, arcs, count, nb, d->col, d->row_ptr);
        DCUDA(d, cudaGetLastError());
    } else {
        DCUDA(d, cudaMalloc(&d->col, sizeof(int)));
        k_fill64<<<grid_for(count + 1), kB, 0, d->stream>>>(d->row_ptr, count + 1, 0);
        DCUDA(d, cudaGetLastError());
    }
    DCUDA(d, cudaStreamSynchronize(d->stream));
    cudaFree(k0);
    cudaFree(k1);
    cudaFree(nkeys);
    cudaFree(bad);
    d->arcs = arcs;
    // degree-aware re-arrangement by global tuple-incidence count (R-6)
    if (arcs > 0) {
        unsigned* mx = nullptr;
        DCUDA(d, cudaMalloc(&mx, sizeof(unsigned)));
        DCUDA(d, cudaMemsetAsync(mx, 0, sizeof(unsigned), d->stream));
        k_maxinc<<<grid_for(n), kB, 0, d->stream>>>(inc, n, mx);
        unsigned hmx = 0;
        DCUDA(d, cudaMemcpyAsync(&hmx, mx, sizeof(unsigned), cudaMemcpyDeviceToHost, d->stream));
        DCUDA(d, cudaStreamSynchronize(d->stream));
        cudaFree(mx);
        const int db = std::max(1, bitlen(hmx));
        unsigned long long *r0 = nullptr, *r1 = nullptr;
        int* c1 = nullptr;
        DCUDA(d, cudaMalloc(&r0, arcs * sizeof(unsigned long long)));
        DCUDA(d, cudaMalloc(&r1, arcs * sizeof(unsigned long long)));
        DCUDA(d, cudaMalloc(&c1, arcs * sizeof(int)));
        k_rkeys<<<grid_for(arcs), kB, 0, d->stream>>>(d->row_ptr, d->col, inc, count, arcs, db,
                                                       (unsigned long long)hmx, r0);
        DCUDA(d, cudaGetLastError());
        cub::DoubleBuffer<unsigned long long> dk(r0, r1);
        cub::DoubleBuffer<int> dv(d->col, c1);
        size_t tb = 0;
        DCUDA(d, cub::DeviceRadixSort::SortPairs(nullptr, tb, dk, dv, arcs, 0, nb_row + db, d->stream));
        void* tmp = nullptr;
        DCUDA(d, cudaMalloc(&tmp, tb));
        DCUDA(d, cub::DeviceRadixSort::SortPairs(tmp, tb, dk, dv, arcs, 0, nb_row + db, d->stream));
        DCUDA(d, cudaStreamSynchronize(d->stream));
        cudaFree(tmp);
        if (dv.Current() != d->col) { cudaFree(d->col); d->col = dv.Current(); } else { cudaFree(c1); }
        cudaFree(r0);
        cudaFree(r1);
    }
    cudaFree(inc);
    // per-vertex facts and BFS state
    DCUDA(d, cudaMalloc(&d->head, std::max(count, 1ll) * sizeof(unsigned long long)));
    DCUDA(d, cudaMalloc(&d->noniso, std::max(d->cw, 1ll) * sizeof(unsigned)));
    DCUDA(d, cudaMalloc(&d->vis, std::max(d->cw, 1ll) * sizeof(unsigned)));
    DCUDA(d, cudaMalloc(&d->acc, sizeof(DAcc)));
    DCUDA(d, cudaMemsetAsync(d->acc, 0, sizeof(DAcc), d->stream));
    DCUDA(d, cudaHostAlloc(&d->acc_host, sizeof(DAcc), cudaHostAllocDefault));
    k_facts<<<grid_for(d->cw), kB, 0, d->stream>>>(d->row_ptr, d->col, count, d->cw, d->noniso, d->head,
                                                   &d->acc->found);
    DCUDA(d, cudaGetLastError());
    DCUDA(d, cudaMemcpyAsync(d->acc_host, d->acc, sizeof(DAcc), cudaMemcpyDeviceToHost, d->stream));
    DCUDA(d, cudaStreamSynchronize(d->stream));
    d->nonisolated_local = (long long)d->acc_host->found;
    DCUDA(d, cudaMemsetAsync(d->acc, 0, sizeof(DAcc), d->stream));
    // TD work items: one per 1024-arc chunk, at most arcs/1024 + count
    d->items_cap = arcs / kChunkArcs + count + 1;
    DCUDA(d, cudaMalloc(&d->items, d->items_cap * sizeof(unsigned long long)));
    // shared region: 3 replicated frontier bitmaps + inbox
    const size_t sh = (3 * d->fwords_pad + d->blk_w) * sizeof(unsigned);
    DCUDA(d, cudaMalloc(&d->shared, sh));
    DCUDA(d, cudaMemsetAsync(d->shared, 0, sh, d->stream));
    DCUDA(d, cudaStreamSynchronize(d->stream));
    return XBFS_OK;
}

xbfs_status check(xbfs_dist* d) {
    if (!d) return set_error(XBFS_ERR_INVALID_ARG, "NULL dist handle");
    if (d->poisoned) return set_error(XBFS_ERR_STATE, "dist handle poisoned by an earlier failure");
    return XBFS_OK;
}

}  // namespace

extern "C" {

xbfs_status xbfs_dist_build(const void* src, const void* dst, int64_t m, int64_t n, int32_t nranks, int32_t rank,
                            const xbfs_build_opts* opts, xbfs_dist** out) {
    if (!out) return set_error(XBFS_ERR_INVALID_ARG, "xbfs_dist_build: out is NULL");
    *out = nullptr;
    if (n <= 0 || n >= (1ll << 31)) return set_error(XBFS_ERR_INVALID_ARG, "num_vertices %lld out of (0, 2^31)", (long long)n);
    if (m < 0 || (m > 0 && (!src || !dst))) return set_error(XBFS_ERR_INVALID_ARG, "bad edge arrays");
    if (nranks < 1 || nranks > XBFS_DIST_MAX_RANKS || rank < 0 || rank >= nranks)
        return set_error(XBFS_ERR_INVALID_ARG, "rank %d / nranks %d invalid", rank, nranks);
    xbfs_build_opts o{};
    if (opts) o = *opts;
    if (o.id_bytes == 0) o.id_bytes = 4;
    if (o.id_bytes != 4 && o.id_bytes != 8) return set_error(XBFS_ERR_INVALID_ARG, "id_bytes must be 4 or 8");
    if (o.directed) return set_error(XBFS_ERR_UNSUPPORTED, "directed graphs are single-GPU only (xbfs_build_csr)");
    xbfs_dist* d = new (std::nothrow) xbfs_dist();
    if (!d) return set_error(XBFS_ERR_OUT_OF_MEMORY, "host allocation failed");
    if (o.device >= 0) {
        if (cudaSetDevice(o.device) != cudaSuccess) { delete d; return set_error(XBFS_ERR_CUDA, "cudaSetDevice"); }
        d->device = o.device;
    } else {
        cudaGetDevice(&d->device);
    }
    d->stream = (cudaStream_t)o.stream;
    d->rank = rank;
    d->nranks = nranks;
    d->n = n;
    d->blk = ((n + 32LL * nranks - 1) / (32LL * nranks)) * 32;
    d->blk_w = d->blk / 32;
    d->lo = std::min<long long>(n, (long long)rank * d->blk);
    d->count = std::max(0ll, std::min<long long>(d->blk, n - d->lo));
    d->cw = (d->count + 31) / 32;
    d->fwords = (n + 31) / 32;
    d->fwords_pad = (d->fwords + 31) / 32 * 32;
    xbfs_run_opts_default(&d->opts);
    xbfs_status s = build_impl(d, src, dst, m, o);
    if (s != XBFS_OK) { xbfs_dist_destroy(d); return s; }
    *out = d;
    return XBFS_OK;
}

xbfs_status xbfs_dist_info(const xbfs_dist* d, int64_t* first, int64_t* count, int64_t* local_arcs, int64_t* nv) {
    if (!d) return set_error(XBFS_ERR_INVALID_ARG, "NULL dist handle");
    if (first) *first = d->lo;
    if (count) *count = d->count;
    if (local_arcs) *local_arcs = d->arcs;
    if (nv) *nv = d->n;
    return XBFS_OK;
}

xbfs_status xbfs_dist_export(xbfs_dist* d, void* handle_out) {
    xbfs_status s = check(d);
    if (s != XBFS_OK) return s;
    if (!handle_out) return set_error(XBFS_ERR_INVALID_ARG, "NULL handle_out");
    static_assert(sizeof(cudaIpcMemHandle_t) == XBFS_IPC_HANDLE_BYTES, "IPC handle size");
    cudaIpcMemHandle_t h;
    DCUDA(d, cudaSetDevice(d->device));
    DCUDA(d, cudaIpcGetMemHandle(&h, d->shared));
    memcpy(handle_out, &h, sizeof(h));
    return XBFS_OK;
}

xbfs_status xbfs_dist_attach(xbfs_dist* d, const void* handles) {
    xbfs_status s = check(d);
    if (s != XBFS_OK) return s;
    if (!handles) return set_error(XBFS_ERR_INVALID_ARG, "NULL handles");
    if (d->attached) return set_error(XBFS_ERR_STATE, "already attached");
    DCUDA(d, cudaSetDevice(d->device));
    for (int p = 0; p < d->nranks; ++p) {
        if (p == d->rank) continue;
        cudaIpcMemHandle_t h;
        memcpy(&h, (const char*)handles + (size_t)p * XBFS_IPC_HANDLE_BYTES, sizeof(h));
        void* ptr = nullptr;
        DCUDA(d, cudaIpcOpenMemHandle(&ptr, h, cudaIpcMemLazyEnablePeerAccess));
        d->peer_base[p] = (unsigned*)ptr;
    }
    d->attached = true;
    return XBFS_OK;
}

xbfs_status xbfs_dist_begin(xbfs_dist* d, int64_t source, int32_t* level, int32_t* parent,
                            const xbfs_run_opts* opts, int64_t counts[XBFS_DIST_NCOUNTS]) {
    xbfs_status s = check(d);
    if (s != XBFS_OK) return s;
    if (!d->attached && d->nranks > 1) return set_error(XBFS_ERR_STATE, "xbfs_dist_attach first");
    if ((!level || !parent) && d->count > 0) return set_error(XBFS_ERR_INVALID_ARG, "NULL level/parent");
    if (source < 0 || source >= d->n) return set_error(XBFS_ERR_INVALID_ARG, "source out of range");
    if (!counts) return set_error(XBFS_ERR_INVALID_ARG, "NULL counts");
    xbfs_run_opts_default(&d->opts);
    if (opts) d->opts = *opts;
    if (d->opts.force_strategy < -1 || d->opts.force_strategy > 2)
        return set_error(XBFS_ERR_INVALID_ARG, "force_strategy must be -1..2");
    DCUDA(d, cudaSetDevice(d->device));
    d->level = level;
    d->parent = parent;
    DArgs a = d->args();
    k_init<<<grid_for(std::max(d->fwords, d->count)), kB, 0, d->stream>>>(a);
    k_seed<<<1, 1, 0, d->stream>>>(a, source);
    DCUDA(d, cudaGetLastError());
    long long deg = 0, tc = 0;
    const bool owner = source >= d->lo && source < d->lo + d->count;
    if (owner) {
        unsigned long long hd = 0;
        int t = 0;
        DCUDA(d, cudaMemcpyAsync(&hd, d->head + (source - d->lo), sizeof(hd), cudaMemcpyDeviceToHost, d->stream));
        DCUDA(d, cudaMemcpyAsync(&t, d->tcount + (source - d->lo), sizeof(t), cudaMemcpyDeviceToHost, d->stream));
        DCUDA(d, cudaStreamSynchronize(d->stream));
        deg = (long long)(hd >> 32);
        tc = t;
    }
    DCUDA(d, cudaStreamSynchronize(d->stream));
    for (int i = 0; i < XBFS_DIST_NCOUNTS; ++i) counts[i] = 0;
    counts[0] = owner ? 1 : 0;
    counts[1] = deg;
    counts[2] = tc;
    counts[3] = d->nonisolated_local;
    counts[4] = d->arcs;
    d->k = 0;
    d->started = 0;
    d->log_s.clear();
    d->log_f.clear();
    d->log_e.clear();
    return XBFS_OK;
}

xbfs_status xbfs_dist_level(xbfs_dist* d, int32_t phase, int64_t counts[XBFS_DIST_NCOUNTS]) {
    xbfs_status s = check(d);
    if (s != XBFS_OK) return s;
    if (!d->started) return set_error(XBFS_ERR_STATE, "xbfs_dist_advance must follow xbfs_dist_begin");
    if (!counts || (phase != 0 && phase != 1)) return set_error(XBFS_ERR_INVALID_ARG, "bad phase/counts");
    DCUDA(d, cudaSetDevice(d->device));
    DArgs a = d->args();
    const int k = d->k;
    const int grid = grid_for(std::max(d->fwords, d->cw) * 4, 148 * 8);
    for (int i = 0; i < XBFS_DIST_NCOUNTS; ++i) counts[i] = 0;
    if (d->strategy == XBFS_BU) {
        if (phase == 0) {
            DCUDA(d, cudaMemsetAsync(d->acc, 0, sizeof(DAcc), d->stream));
            int nsm = 148;
            cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, d->device);
            k_bu<<<nsm * 5, kBuThreads, 0, d->stream>>>(a, k);
            DCUDA(d, cudaGetLastError());
        }
    } else if (phase == 0) {
        DCUDA(d, cudaMemsetAsync(d->acc, 0, sizeof(DAcc), d->stream));
        k_items<<<grid, kB, 0, d->stream>>>(a, k);
        k_td<<<grid, kB, 0, d->stream>>>(a, k);
        DCUDA(d, cudaGetLastError());
    } else {
        k_merge<<<grid, kB, 0, d->stream>>>(a, k);
        DCUDA(d, cudaGetLastError());
    }
    DCUDA(d, cudaMemcpyAsync(d->acc_host, d->acc, sizeof(DAcc), cudaMemcpyDeviceToHost, d->stream));
    DCUDA(d, cudaStreamSynchronize(d->stream));
    const bool last = d->strategy == XBFS_BU ? phase == 0 : phase == 1;
    if (last) {
        counts[0] = (int64_t)d->acc_host->found;
        counts[1] = (int64_t)d->acc_host->edges;
        counts[2] = (int64_t)d->acc_host->m;
        counts[3] = (int64_t)d->acc_host->probes;
    }
    return XBFS_OK;
}

xbfs_status xbfs_dist_advance(xbfs_dist* d, const int64_t g[XBFS_DIST_NCOUNTS], int32_t* strategy_out,
                              int32_t* done) {
    xbfs_status s = check(d);
    if (s != XBFS_OK) return s;
    if (!g) return set_error(XBFS_ERR_INVALID_ARG, "NULL counts");
    if (!d->started) {
        // first call: g = {1, deg(s), tcount(s), non-isolated vertices, arcs A}
        d->fsize = g[0];
        d->fedges = g[1];
        d->m_total = g[2];
        d->unvisited = g[3] - (g[1] > 0 ? 1 : 0);
        d->arcs_global = g[4];
        d->fprev = 0;
        d->started = 1;
        d->strategy = choose(d->opts, d->arcs_global, d->fsize, 0, d->fedges, d->unvisited, -1);
    } else {
        d->log_s.push_back((int8_t)d->strategy);
        d->log_f.push_back(d->fsize);
        d->log_e.push_back(d->fedges);
        const int prev = d->strategy;
        d->fprev = d->fsize;
        d->fsize = g[0];
        d->fedges = g[1];
        d->m_total += g[2];
        d->unvisited -= g[0];
        d->k += 1;
        d->strategy = choose(d->opts, d->arcs_global, d->fsize, d->fprev, d->fedges, d->unvisited, prev);
    }
    if (strategy_out) *strategy_out = d->strategy;
    if (done) *done = d->fsize == 0 ? 1 : 0;
    return XBFS_OK;
}

xbfs_status xbfs_dist_levels(const xbfs_dist* d, int32_t cap, int8_t* strategy, int64_t* fv, int64_t* fe,
                             int32_t* num_levels, int64_t* input_edges) {
    if (!d) return set_error(XBFS_ERR_INVALID_ARG, "NULL dist handle");
    const int nl = (int)d->log_s.size();
    for (int i = 0; i < std::min(nl, cap); ++i) {
        if (strategy) strategy[i] = d->log_s[i];
        if (fv) fv[i] = d->log_f[i];
        if (fe) fe[i] = d->log_e[i];
    }
    if (num_levels) *num_levels = nl;
    if (input_edges) *input_edges = d->m_total;
    return XBFS_OK;
}

void xbfs_dist_destroy(xbfs_dist* d) {
    if (!d) return;
    cudaSetDevice(d->device);
    if (d->stream) cudaStreamSynchronize(d->stream);
    for (int p = 0; p < XBFS_DIST_MAX_RANKS; ++p)
        if (d->peer_base[p]) cudaIpcCloseMemHandle(d->peer_base[p]);
    void* ptrs[] = {d->row_ptr, d->col, d->head, d->tcount, d->noniso, d->vis, d->shared, d->items, d->acc};
    for (void* p : ptrs)
        if (p) cudaFree(p);
    if (d->acc_host) cudaFreeHost(d->acc_host);
    cudaGetLastError();
    delete d;
}

}  // extern "C"
