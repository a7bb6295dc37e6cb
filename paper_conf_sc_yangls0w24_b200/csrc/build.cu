// build.cu — CSR construction (Graph500 "kernel 1") and
// the degree-aware neighbour re-arrangement (row a2, §IV-B).
//
// Both are untimed preprocessing.  The sort / unique / scan steps use CUB
// (library primitives, like a cuBLAS GEMM); the packing, range check, row
// boundaries, degree/bitmap and tuple-count kernels are ours.
#include <cub/cub.cuh>

#include <algorithm>
#include <new>

#include "common.cuh"

namespace xbfs {
namespace {

constexpr int kB = 256;

inline int grid_for(long long n, int per_block = kB, int cap = 148 * 32) {
    long long g = (n + per_block - 1) / per_block;
    if (g < 1) g = 1;
    return (int)std::min<long long>(g, cap);
}

inline int bitlen(unsigned long long x) { return x ? 64 - __builtin_clzll(x) : 0; }

template <typename IdT>
__global__ __launch_bounds__(kB) void k_check_and_pack(const IdT* __restrict__ src, const IdT* __restrict__ dst,
                                                       long long m, long long n, int nb,
                                                       unsigned long long* __restrict__ keys,
                                                       int* __restrict__ tcount, int* __restrict__ bad,
                                                       int directed) {
    const unsigned long long sentinel = (nb >= 32) ? ~0ull : ((1ull << (2 * nb)) - 1ull);
    for (long long e = blockIdx.x * (long long)blockDim.x + threadIdx.x; e < m;
         e += (long long)gridDim.x * blockDim.x) {
        long long u = (long long)src[e], v = (long long)dst[e];
        if (u < 0 || v < 0 || u >= n || v >= n) {
            *bad = 1;
            keys[2 * e] = keys[2 * e + 1] = sentinel;
            continue;
        }
        atomicAdd(&tcount[u], 1);  // Graph500 m counts every tuple by its first endpoint (O-6)
        if (u == v) {              // self-loop dropped (reading C-3)
            keys[2 * e] = keys[2 * e + 1] = sentinel;
        } else {                   // both arcs of the undirected edge (reading C-2)
            keys[2 * e] = ((unsigned long long)u << nb) | (unsigned long long)v;
            keys[2 * e + 1] = directed ? sentinel   // arc u -> v only (f4, reading R-9)
                                       : ((unsigned long long)v << nb) | (unsigned long long)u;
        }
    }
}

// col[i] = low nb bits; row_ptr[r] = first i with row(key[i]) >= r.
__global__ __launch_bounds__(kB) void k_split_keys(const unsigned long long* __restrict__ keys, long long a,
                                                   long long n, int nb, int* __restrict__ col,
                                                   long long* __restrict__ row_ptr) {
    const unsigned long long lowmask = (1ull << nb) - 1ull;
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < a;
         i += (long long)gridDim.x * blockDim.x) {
        unsigned long long k = keys[i];
        long long r = (long long)(k >> nb);
        col[i] = (int)(k & lowmask);
        long long prev = (i == 0) ? -1 : (long long)(keys[i - 1] >> nb);
        for (long long q = prev + 1; q <= r; ++q) row_ptr[q] = i;
        if (i == a - 1)
            for (long long q = r + 1; q <= n; ++q) row_ptr[q] = a;
    }
}

__global__ __launch_bounds__(kB) void k_fill_rowptr(long long* row_ptr, long long n, long long val) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i <= n;
         i += (long long)gridDim.x * blockDim.x)
        row_ptr[i] = val;
}

// non-isolated bitmap words, count and max degree.
__global__ __launch_bounds__(kB) void k_degree_facts(const long long* __restrict__ row_ptr, long long n,
                                                     long long words, unsigned int* __restrict__ nonisolated,
                                                     unsigned long long* __restrict__ red) {
    unsigned long long cnt = 0, mx = 0;
    for (long long w = blockIdx.x * (long long)blockDim.x + threadIdx.x; w < words;
         w += (long long)gridDim.x * blockDim.x) {
        unsigned int bits = 0;
        for (int b = 0; b < 32; ++b) {
            long long v = w * 32 + b;
            if (v >= n) break;
            long long d = row_ptr[v + 1] - row_ptr[v];
            if (d > 0) bits |= 1u << b;
            if ((unsigned long long)d > mx) mx = (unsigned long long)d;
        }
        nonisolated[w] = bits;
        cnt += __popc(bits);
    }
    for (int o = 16; o; o >>= 1) {
        cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
        mx = max(mx, __shfl_xor_sync(0xffffffffu, mx, o));
    }
    if ((threadIdx.x & 31) == 0) {
        atomicAdd(&red[0], cnt);
        atomicMax(&red[1], mx);
    }
}

// head[v] = deg(v) << 32 | first stored neighbour: the bottom-up first probe reads
// this dense array in candidate order instead of a random sector of col.
// head32[v] = min(deg(v), dmax) << idbits | first stored neighbour, dmax =
// 2^(32 - idbits) - 1 meaning "deg >= dmax, read row_ptr": the single-GPU BU
// first probe reads 4 bytes per candidate instead of 8 (idbits = bitlen(N-1)).
__global__ __launch_bounds__(kB) void k_head(const long long* __restrict__ row_ptr, const int* __restrict__ col,
                                             long long n, unsigned long long* __restrict__ head,
                                             unsigned* __restrict__ head32, int idbits) {
    const unsigned dmax = idbits >= 32 ? 0u : (0xffffffffu >> idbits);
    for (long long v = blockIdx.x * (long long)blockDim.x + threadIdx.x; v < n;
         v += (long long)gridDim.x * blockDim.x) {
        const long long rs = row_ptr[v], d = row_ptr[v + 1] - rs;
        if (head) head[v] = ((unsigned long long)d << 32) | (d > 0 ? (unsigned)col[rs] : 0xffffffffu);
        const unsigned dc = d < (long long)dmax ? (unsigned)d : dmax;
        head32[v] = (idbits >= 32 ? 0u : (dc << idbits)) | (d > 0 ? (unsigned)col[rs] : 0u);
    }
}

// Reorder keys: (row << db) | (maxdeg - deg(col))  -> degree descending within the
// row; the radix sort is stable so ties keep ascending id order (reading C-12).
// mode 0 keys: (row << nb) | col  -> id order.
// deg_rp: the row_ptr degrees are read from (the out-arc CSR also for the in-arc one).
__global__ __launch_bounds__(kB) void k_reorder_keys(const long long* __restrict__ row_ptr,
                                                     const int* __restrict__ col, long long n, long long a,
                                                     int mode, int shift, unsigned long long maxdeg,
                                                     unsigned long long* __restrict__ keys,
                                                     const long long* __restrict__ deg_rp) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < a;
         i += (long long)gridDim.x * blockDim.x) {
        // row of arc i: last r with row_ptr[r] <= i
        long long lo = 0, hi = n - 1;
        while (lo < hi) {
            long long mid = (lo + hi + 1) >> 1;
            if (row_ptr[mid] <= i) lo = mid; else hi = mid - 1;
        }
        int c = col[i];
        unsigned long long low = mode == 1 ? maxdeg - (unsigned long long)(deg_rp[c + 1] - deg_rp[c])
                                           : (unsigned long long)c;
        keys[i] = ((unsigned long long)lo << shift) | low;
    }
}

// Directed graphs (f4): key (col << nb) | row of every out-arc, i.e. the arc as a row of
// the transposed (in-arc) CSR; sorted and split like the input tuples.
__global__ __launch_bounds__(kB) void k_transpose_keys(const long long* __restrict__ row_ptr,
                                                       const int* __restrict__ col, long long n, long long a,
                                                       int nb, unsigned long long* __restrict__ keys) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < a;
         i += (long long)gridDim.x * blockDim.x) {
        long long lo = 0, hi = n - 1;
        while (lo < hi) {
            long long mid = (lo + hi + 1) >> 1;
            if (row_ptr[mid] <= i) lo = mid; else hi = mid - 1;
        }
        keys[i] = ((unsigned long long)col[i] << nb) | (unsigned long long)lo;
    }
}

template <typename IdT>
xbfs_status pack_edges(xbfs_graph* g, const void* src, const void* dst, long long m, int nb,
                       bool on_device, unsigned long long* keys, int* bad) {
    const IdT* s = (const IdT*)src;
    const IdT* d = (const IdT*)dst;
    IdT *ds = nullptr, *dd = nullptr;
    // host edges are staged through the device in chunks to bound memory
    const long long chunk = on_device ? m : std::min<long long>(m, 1ll << 27);
    if (!on_device && m > 0) {
        XBFS_CUDA(g, cudaMalloc(&ds, chunk * sizeof(IdT)));
        XBFS_CUDA(g, cudaMalloc(&dd, chunk * sizeof(IdT)));
    }
    for (long long e0 = 0; e0 < m; e0 += chunk) {
        long long c = std::min(chunk, m - e0);
        const IdT* ps = s + e0;
        const IdT* pd = d + e0;
        if (!on_device) {
            XBFS_CUDA(g, cudaMemcpyAsync(ds, ps, c * sizeof(IdT), cudaMemcpyHostToDevice, g->stream));
            XBFS_CUDA(g, cudaMemcpyAsync(dd, pd, c * sizeof(IdT), cudaMemcpyHostToDevice, g->stream));
            ps = ds;
            pd = dd;
        }
        k_check_and_pack<IdT><<<grid_for(c), kB, 0, g->stream>>>(ps, pd, c, g->n, nb, keys + 2 * e0,
                                                                 g->tcount, bad, g->directed);
        XBFS_CUDA(g, cudaGetLastError());
    }
    if (ds) {
        XBFS_CUDA(g, cudaStreamSynchronize(g->stream));
        cudaFree(ds);
        cudaFree(dd);
    }
    return XBFS_OK;
}

// Directed graphs (f4): the in-arc CSR (in_row_ptr, in_col) of the out-arc CSR just
// built, rows id-sorted; the bottom-up steps search it.
xbfs_status build_transpose(xbfs_graph* g, int nb) {
    const long long n = g->n, a = g->arcs;
    XBFS_CUDA(g, cudaMalloc(&g->in_row_ptr, (n + 1) * sizeof(long long)));
    XBFS_CUDA(g, cudaMalloc(&g->in_col, std::max<long long>(a, 1) * sizeof(int)));
    if (a == 0) {
        k_fill_rowptr<<<grid_for(n + 1), kB, 0, g->stream>>>(g->in_row_ptr, n, 0);
        XBFS_CUDA(g, cudaGetLastError());
        return XBFS_OK;
    }
    unsigned long long *k0 = nullptr, *k1 = nullptr;
    XBFS_CUDA(g, cudaMalloc(&k0, a * sizeof(unsigned long long)));
    XBFS_CUDA(g, cudaMalloc(&k1, a * sizeof(unsigned long long)));
    k_transpose_keys<<<grid_for(a), kB, 0, g->stream>>>(g->row_ptr, g->col, n, a, nb, k0);
    XBFS_CUDA(g, cudaGetLastError());
    cub::DoubleBuffer<unsigned long long> db(k0, k1);
    size_t tb = 0;
    XBFS_CUDA(g, cub::DeviceRadixSort::SortKeys(nullptr, tb, db, a, 0, 2 * nb, g->stream));
    void* tmp = nullptr;
    XBFS_CUDA(g, cudaMalloc(&tmp, tb));
    XBFS_CUDA(g, cub::DeviceRadixSort::SortKeys(tmp, tb, db, a, 0, 2 * nb, g->stream));
    k_split_keys<<<grid_for(a), kB, 0, g->stream>>>(db.Current(), a, n, nb, g->in_col, g->in_row_ptr);
    XBFS_CUDA(g, cudaGetLastError());
    XBFS_CUDA(g, cudaStreamSynchronize(g->stream));
    cudaFree(tmp);
    cudaFree(k0);
    cudaFree(k1);
    return XBFS_OK;
}

// Re-arrange the rows of (rp, *colp) by mode (1: neighbour out-degree descending,
// ties id ascending; 0: id order).  *colp may be replaced by the sort's buffer.
xbfs_status reorder_rows(xbfs_graph* g, const long long* rp, int** colp, int mode) {
    const long long a = g->arcs, n = g->n;
    const int nb = std::max(1, bitlen((unsigned long long)(n - 1)));
    const int db = std::max(1, bitlen((unsigned long long)g->max_deg));
    const int low = mode == 1 ? db : nb;
    const int shift = low;
    const int total_bits = nb + low;
    if (total_bits > 64) return set_error(XBFS_ERR_UNSUPPORTED, "reorder key does not fit in 64 bits");
    unsigned long long *k0 = nullptr, *k1 = nullptr;
    int* c1 = nullptr;
    XBFS_CUDA(g, cudaMalloc(&k0, a * sizeof(unsigned long long)));
    XBFS_CUDA(g, cudaMalloc(&k1, a * sizeof(unsigned long long)));
    XBFS_CUDA(g, cudaMalloc(&c1, a * sizeof(int)));
    k_reorder_keys<<<grid_for(a), kB, 0, g->stream>>>(rp, *colp, n, a, mode, shift,
                                                      (unsigned long long)g->max_deg, k0, g->row_ptr);
    XBFS_CUDA(g, cudaGetLastError());
    cub::DoubleBuffer<unsigned long long> dk(k0, k1);
    cub::DoubleBuffer<int> dv(*colp, c1);
    size_t tb = 0;
    XBFS_CUDA(g, cub::DeviceRadixSort::SortPairs(nullptr, tb, dk, dv, a, 0, total_bits, g->stream));
    void* tmp = nullptr;
    XBFS_CUDA(g, cudaMalloc(&tmp, tb));
    XBFS_CUDA(g, cub::DeviceRadixSort::SortPairs(tmp, tb, dk, dv, a, 0, total_bits, g->stream));
    XBFS_CUDA(g, cudaStreamSynchronize(g->stream));
    cudaFree(tmp);
    if (dv.Current() != *colp) {
        cudaFree(*colp);
        *colp = dv.Current();
    } else {
        cudaFree(c1);
    }
    cudaFree(k0);
    cudaFree(k1);
    return XBFS_OK;
}

xbfs_status alloc_work(xbfs_graph* g) {
    const long long n = g->n, words = (n + 31) / 32;
    g->tiles_cap = g->arcs / kTile + 4;
    XBFS_CUDA(g, cudaMalloc(&g->visited, words * sizeof(unsigned int)));
    XBFS_CUDA(g, cudaMalloc(&g->fb, 4 * ((words + 31) / 32 * 32) * sizeof(unsigned int)));
    XBFS_CUDA(g, cudaMalloc(&g->qv, 3 * n * sizeof(int)));
    XBFS_CUDA(g, cudaMalloc(&g->qoff, 3 * n * sizeof(long long)));
    XBFS_CUDA(g, cudaMalloc(&g->qdelta, 3 * n * sizeof(long long)));
    XBFS_CUDA(g, cudaMalloc(&g->tile_first, 3 * g->tiles_cap * sizeof(int)));
    XBFS_CUDA(g, cudaMalloc(&g->st, sizeof(DevState)));
    XBFS_CUDA(g, cudaMemset(g->st, 0, sizeof(DevState)));
    XBFS_CUDA(g, cudaMalloc(&g->log, kLogCap * sizeof(LevelRec)));
    XBFS_CUDA(g, cudaMalloc(&g->red_scratch, 8 * sizeof(unsigned long long)));
    XBFS_CUDA(g, cudaHostAlloc(&g->hctl, sizeof(HostCtl), cudaHostAllocMapped));
    XBFS_CUDA(g, cudaHostGetDevicePointer(&g->hctl_dev, g->hctl, 0));
    XBFS_CUDA(g, cudaHostAlloc(&g->hstage, xbfs_graph::kStageSlots * sizeof(DevState), cudaHostAllocDefault));
    for (int i = 0; i < xbfs_graph::kStageSlots; ++i)
        XBFS_CUDA(g, cudaEventCreateWithFlags(&g->ev_stage[i], cudaEventDisableTiming));
    XBFS_CUDA(g, cudaEventCreate(&g->ev0));
    XBFS_CUDA(g, cudaEventCreate(&g->ev1));
    // The packed queue counter keeps |F| in the high bits and the degree sum in
    // the low dbits: |F| <= N needs bitlen(N) bits.
    g->dbits = 64 - bitlen((unsigned long long)n);
    return XBFS_OK;
}

}  // namespace

}  // namespace xbfs

using namespace xbfs;

#define XBFS_TRY_B(expr)                        \
    do {                                        \
        xbfs_status _s = (expr);                \
        if (_s != XBFS_OK) return _s;           \
    } while (0)

extern "C" xbfs_status xbfs_build_csr(const void* src, const void* dst, int64_t m, int64_t n,
                                      const xbfs_build_opts* opts, xbfs_graph** out) {
    if (!out) return set_error(XBFS_ERR_INVALID_ARG, "xbfs_build_csr: out is NULL");
    *out = nullptr;
    if (n <= 0 || n >= (1ll << 31)) return set_error(XBFS_ERR_INVALID_ARG, "num_vertices %lld out of (0, 2^31)", (long long)n);
    if (m < 0) return set_error(XBFS_ERR_INVALID_ARG, "num_edges < 0");
    if (m > 0 && (!src || !dst)) return set_error(XBFS_ERR_INVALID_ARG, "src/dst NULL");
    xbfs_build_opts o{};
    if (opts) o = *opts;
    if (o.id_bytes == 0) o.id_bytes = 4;
    if (o.id_bytes != 4 && o.id_bytes != 8) return set_error(XBFS_ERR_INVALID_ARG, "id_bytes must be 4 or 8");

    xbfs_graph* g = new (std::nothrow) xbfs_graph();
    if (!g) return set_error(XBFS_ERR_OUT_OF_MEMORY, "host allocation failed");
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
    g->n = n;
    g->m_input = m;
    g->directed = o.directed ? 1 : 0;
    const int nb = std::max(1, bitlen((unsigned long long)(n - 1)));
    const long long nkeys = 2 * m;

    XBFS_CUDA(g, cudaMalloc(&g->tcount, n * sizeof(int)));
    XBFS_CUDA(g, cudaMemsetAsync(g->tcount, 0, n * sizeof(int), g->stream));
    XBFS_CUDA(g, cudaMalloc(&g->row_ptr, (n + 1) * sizeof(long long)));
    int* bad = nullptr;
    XBFS_CUDA(g, cudaMalloc(&bad, 2 * sizeof(int)));
    XBFS_CUDA(g, cudaMemsetAsync(bad, 0, 2 * sizeof(int), g->stream));

    long long arcs = 0;
    if (nkeys > 0) {
        unsigned long long *k0 = nullptr, *k1 = nullptr;
        XBFS_CUDA(g, cudaMalloc(&k0, nkeys * sizeof(unsigned long long)));
        XBFS_CUDA(g, cudaMalloc(&k1, nkeys * sizeof(unsigned long long)));
        xbfs_status s = o.id_bytes == 4
                            ? pack_edges<unsigned int>(g, src, dst, m, nb, o.edges_on_device != 0, k0, bad)
                            : pack_edges<long long>(g, src, dst, m, nb, o.edges_on_device != 0, k0, bad);
        if (s != XBFS_OK) { cudaFree(k0); cudaFree(k1); cudaFree(bad); return s; }
        int hbad = 0;
        XBFS_CUDA(g, cudaMemcpyAsync(&hbad, bad, sizeof(int), cudaMemcpyDeviceToHost, g->stream));
        XBFS_CUDA(g, cudaStreamSynchronize(g->stream));
        if (hbad) {
            cudaFree(k0); cudaFree(k1); cudaFree(bad);
            return set_error(XBFS_ERR_INVALID_ARG, "edge id out of range [0, %lld)", (long long)n);
        }
        // radix sort of the packed arcs (row-major, then neighbour id)
        cub::DoubleBuffer<unsigned long long> db(k0, k1);
        size_t tmp_bytes = 0;
        XBFS_CUDA(g, cub::DeviceRadixSort::SortKeys(nullptr, tmp_bytes, db, nkeys, 0, 2 * nb, g->stream));
        void* tmp = nullptr;
        XBFS_CUDA(g, cudaMalloc(&tmp, tmp_bytes));
        XBFS_CUDA(g, cub::DeviceRadixSort::SortKeys(tmp, tmp_bytes, db, nkeys, 0, 2 * nb, g->stream));
        cudaFree(tmp);
        unsigned long long* sorted = db.Current();
        unsigned long long* other = db.Alternate();
        long long* nsel = nullptr;
        XBFS_CUDA(g, cudaMalloc(&nsel, sizeof(long long)));
        unsigned long long* uniq = sorted;
        long long cnt = nkeys;
        if (!o.keep_duplicates) {
            size_t ub = 0;
            XBFS_CUDA(g, cub::DeviceSelect::Unique(nullptr, ub, sorted, other, nsel, nkeys, g->stream));
            XBFS_CUDA(g, cudaMalloc(&tmp, ub));
            XBFS_CUDA(g, cub::DeviceSelect::Unique(tmp, ub, sorted, other, nsel, nkeys, g->stream));
            cudaFree(tmp);
            XBFS_CUDA(g, cudaMemcpyAsync(&cnt, nsel, sizeof(long long), cudaMemcpyDeviceToHost, g->stream));
            uniq = other;
        }
        XBFS_CUDA(g, cudaStreamSynchronize(g->stream));
        // sentinels (self-loops) sort last: trim them
        const unsigned long long sentinel = (nb >= 32) ? ~0ull : ((1ull << (2 * nb)) - 1ull);
        arcs = cnt;
        {
            // binary search for the first sentinel among the last entries
            long long lo = 0, hi = cnt;
            while (lo < hi) {
                long long mid = (lo + hi) / 2;
                unsigned long long kv;
                XBFS_CUDA(g, cudaMemcpy(&kv, uniq + mid, sizeof(kv), cudaMemcpyDeviceToHost));
                if (kv == sentinel) hi = mid; else lo = mid + 1;
            }
            arcs = lo;
        }
        g->arcs = arcs;
        XBFS_CUDA(g, cudaMalloc(&g->col, std::max<long long>(arcs, 1) * sizeof(int)));
        if (arcs > 0) {
            k_split_keys<<<grid_for(arcs), kB, 0, g->stream>>>(uniq, arcs, n, nb, g->col, g->row_ptr);
            XBFS_CUDA(g, cudaGetLastError());
        } else {
            k_fill_rowptr<<<grid_for(n + 1), kB, 0, g->stream>>>(g->row_ptr, n, 0);
        }
        XBFS_CUDA(g, cudaStreamSynchronize(g->stream));
        cudaFree(k0);
        cudaFree(k1);
        cudaFree(nsel);
    } else {
        XBFS_CUDA(g, cudaMalloc(&g->col, sizeof(int)));
        k_fill_rowptr<<<grid_for(n + 1), kB, 0, g->stream>>>(g->row_ptr, n, 0);
        XBFS_CUDA(g, cudaGetLastError());
    }
    cudaFree(bad);
    if (g->directed) {
        xbfs_status st = build_transpose(g, nb);
        if (st != XBFS_OK) return st;
    }

    const long long words = (n + 31) / 32;
    XBFS_CUDA(g, cudaMalloc(&g->nonisolated, words * sizeof(unsigned int)));
    xbfs_status s = alloc_work(g);
    if (s != XBFS_OK) return s;
    unsigned long long facts[2];
    XBFS_CUDA(g, cudaMemsetAsync(g->red_scratch, 0, 8 * sizeof(unsigned long long), g->stream));
    k_degree_facts<<<grid_for(words), kB, 0, g->stream>>>(g->row_ptr, n, words, g->nonisolated, g->red_scratch);
    XBFS_CUDA(g, cudaGetLastError());
    XBFS_CUDA(g, cudaMemcpyAsync(facts, g->red_scratch, sizeof(facts), cudaMemcpyDeviceToHost, g->stream));
    XBFS_CUDA(g, cudaStreamSynchronize(g->stream));
    g->nonisolated_count = (long long)facts[0];
    g->max_deg = (int)facts[1];   // max (out-)degree: reorder key width, selector facts
    if (g->directed) {
        // BU candidates of a directed graph: vertices with an in-arc (reading R-9)
        XBFS_CUDA(g, cudaMemsetAsync(g->red_scratch, 0, 8 * sizeof(unsigned long long), g->stream));
        k_degree_facts<<<grid_for(words), kB, 0, g->stream>>>(g->in_row_ptr, n, words, g->nonisolated,
                                                              g->red_scratch);
        XBFS_CUDA(g, cudaGetLastError());
        XBFS_CUDA(g, cudaMemcpyAsync(facts, g->red_scratch, sizeof(facts), cudaMemcpyDeviceToHost, g->stream));
        XBFS_CUDA(g, cudaStreamSynchronize(g->stream));
        g->nonisolated_count = (long long)facts[0];
    }
    XBFS_CUDA(g, cudaMalloc(&g->head, n * sizeof(unsigned long long)));
    XBFS_CUDA(g, cudaMalloc(&g->head32, std::max<long long>(n, 1) * sizeof(unsigned)));
    g->idbits = std::max(1, bitlen((unsigned long long)(n - 1)));
    k_head<<<grid_for(n), kB, 0, g->stream>>>(g->row_ptr, g->col, n, g->head, g->head32, g->idbits);
    XBFS_CUDA(g, cudaGetLastError());
    if (g->directed) {
        XBFS_CUDA(g, cudaMalloc(&g->in_head32, std::max<long long>(n, 1) * sizeof(unsigned)));
        k_head<<<grid_for(n), kB, 0, g->stream>>>(g->in_row_ptr, g->in_col, n, nullptr, g->in_head32, g->idbits);
        XBFS_CUDA(g, cudaGetLastError());
    }
    if ((unsigned long long)arcs >= (1ull << g->dbits))
        return set_error(XBFS_ERR_INVALID_ARG, "graph too large for the packed queue counter");
    XBFS_TRY_B(prepare_drivers(g));
    XBFS_CUDA(g, cudaStreamSynchronize(g->stream));
    guard.keep = true;
    *out = g;
    return XBFS_OK;
}

extern "C" xbfs_status xbfs_reorder(xbfs_graph* g, int32_t mode) {
    if (!g) return set_error(XBFS_ERR_INVALID_ARG, "xbfs_reorder: NULL handle");
    if (mode != 0 && mode != 1) return set_error(XBFS_ERR_INVALID_ARG, "xbfs_reorder: mode must be 0 or 1");
    if (g->poisoned) return set_error(XBFS_ERR_STATE, "handle poisoned by an earlier failure");
    if (g->dist) return set_error(XBFS_ERR_STATE, "xbfs_reorder: a distributed handle is re-arranged at build time");
    if (g->arcs == 0) { g->reorder_mode = mode; return XBFS_OK; }
    XBFS_CUDA(g, cudaSetDevice(g->device));
    const long long n = g->n;
    XBFS_TRY_B(reorder_rows(g, g->row_ptr, &g->col, mode));
    if (g->directed) {
        XBFS_TRY_B(reorder_rows(g, g->in_row_ptr, &g->in_col, mode));
        k_head<<<grid_for(n), kB, 0, g->stream>>>(g->in_row_ptr, g->in_col, n, nullptr, g->in_head32, g->idbits);
        XBFS_CUDA(g, cudaGetLastError());
    }
    k_head<<<grid_for(n), kB, 0, g->stream>>>(g->row_ptr, g->col, n, g->head, g->head32, g->idbits);
    XBFS_CUDA(g, cudaGetLastError());
    XBFS_CUDA(g, cudaStreamSynchronize(g->stream));
    // the device-loop graph captured the old col pointer: re-instantiate it here (never in xbfs_run)
    XBFS_TRY_B(prepare_drivers(g));
    g->reorder_mode = mode;
    return XBFS_OK;
}
