// bu_core.cuh — the bottom-up step over a range of owned bitmap words, shared
// by the single-GPU kernel (k_bu_traverse, bfs.cu) and the multi-GPU one
// (dist.cu).  P:L122-131 §III-C; design notes in bfs.cu / DESIGN.md §5.
#pragma once
#include "common.cuh"

#ifndef XBFS_BU_PROF
#define XBFS_BU_PROF 0
#endif
// dense chunks: bit-parallel candidate compaction, one store per lane per word (B200 A/B:
// 815 vs 805 GTEPS)
#ifndef XBFS_BU_PCOMP
#define XBFS_BU_PCOMP 1
#endif

namespace xbfs {

// The frontier bitmap F_k is read-only during a BU step: its words are loaded through L1
// (the first probes of a dense step mostly hit the few words of the hubs).  Safe in the
// persistent kernel because the grid barrier before the step ends in an acquire load
// that invalidates the SM's L1 (CCTL.IVALL), and the per-level kernels start with a
// clean L1.  XBFS_BU_CUR_L1=0: through L2 (ld.cg) as the mutable arrays.
#ifndef XBFS_BU_CUR_L1
#define XBFS_BU_CUR_L1 1
#endif
__device__ __forceinline__ unsigned ld_cur(const unsigned* p) {
#if XBFS_BU_CUR_L1
    return __ldca(p);
#else
    return __ldcg(p);
#endif
}

// What a BU step reads and writes.  Vertex indices are LOCAL (the owned range
// starts at 0); col values and the frontier bitmap `cur` are GLOBAL.
struct BuView {
    const unsigned int* cur;          // F_k, global bitmap
    const unsigned int* nxt;          // F_{k+1} being written by this pass (look-ahead only)
    unsigned int* visited;            // owned words
    long long words;                  // owned words
    const unsigned long long* head;   // owned: deg << 32 | first stored neighbour
    const unsigned* head32;           // single GPU: min(deg, dmax) << idbits | first neighbour (H32)
    int idbits;
    const long long* row_ptr;         // owned rows
    const int* col;
    int* level;                       // owned
    int* parent;                      // owned (global ids)
    int lvl;                          // k + 1
    bool reverse;                     // walk the vertex range downwards (alternating BU steps)
#if XBFS_BU_PROF
    unsigned long long* prof;         // profiling build: per-phase cycle counters
#endif
};


// Per-warp shared-memory work lists of one block of WARPS warps (static in the
// per-level kernels, carved from dynamic shared memory in the persistent one).
template <int WARPS>
struct BuSmem {
    int list[WARPS][kBuChunkWords * 32];   // candidates of the warp's chunk
    int hard[WARPS][kBuChunkWords * 32];   // long unresolved rows (warp-cooperative)
    int hoff[WARPS][kBuChunkWords * 32];   // arcs already probed for each hard row
    unsigned found[WARPS][32];             // found words of the batch (by owning lane)
};

// ... plus the look-ahead lists (kept out of the default kernels' shared memory).
template <int WARPS>
struct BuSmemLa : BuSmem<WARPS> {
    int hlau[WARPS][kBuChunkWords * 32];   // F_{k+1} neighbour seen before a row went hard
    unsigned la[WARPS][32];                // look-ahead discoveries (level k+2)
};

// Look-ahead accumulators: vertices set to level k+2 by a BU pass.
struct BuLa {
    unsigned long long found = 0, edges = 0;
};

// publish(w, vis, found_word, la_word): store the owned word w of F_{k+1} (and of
// the look-ahead set) and update visited.
// Mutable state (visited) is read through L2 (__ldcg); F_k, read-only during the
// step, through L1 (ld_cur).
//
// LA ("since v7 is updated in this phase, v8, which
// belongs to the next level, can be updated in this bottom-up"): a candidate whose
// whole row holds no F_k vertex but some vertex already published into F_{k+1}
// by this same pass is at level k+2 exactly (no neighbour at level <= k, one at
// k+1: the exactness guard of reading C-9), with that neighbour as parent.  Only
// published F_{k+1} words are seen (whole-word stores), so a set bit is always a
// true level-(k+1) vertex; which candidates profit depends on the pass order.
//
// H32 (single GPU): the first probe reads the 4-byte head32[] word; a hit whose
// degree field saturated (deg >= dmax) is queued for pass 3 as ~v, where one
// row_ptr pair read (overlapping the misses' own) gives the degree for edgesF.
template <int WARPS, bool LA, bool H32, class Smem, class Publish>
__device__ __forceinline__ void bu_chunks(const BuView& b, Smem& sm, Publish publish,
                                          unsigned long long& found, unsigned long long& edges,
                                          unsigned long long& probes, unsigned& fmax, BuLa& la) {
    constexpr unsigned FULL = 0xffffffffu;
    const int lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const unsigned lt = (1u << lane) - 1u;
    constexpr int kCW = kBuChunkWords;
    auto& s_list = sm.list;
    auto& s_hard = sm.hard;
    auto& s_hoff = sm.hoff;
    auto& s_found = sm.found;
    const long long nchunks = (b.words + kCW - 1) / kCW;
    const long long gw = (blockIdx.x * (long long)blockDim.x + threadIdx.x) >> 5;
    const long long nw = ((long long)gridDim.x * blockDim.x) >> 5;
    // A group is 4 chunks (32 lanes = 4 chunks x kCW words): warp gw takes chunks gb + j*nw,
    // j < 4, for gb = gw, gw + 4 nw, ...  One load round trip tells which of the 4 chunks
    // hold candidates, and the next group's words are loaded one group ahead, so chunks
    // without candidates (most of them in late BU levels) cost no exposed latency.
    // (B200 A/B, round 2: a balanced contiguous word range per warp instead: s24 -0.8 %,
    // s20 -1 %; dynamic group scheduling from a step counter: 752 vs 788 GTEPS; an L2
    // prefetch of the next group's head32: 779 vs 806)
    static_assert(kCW == 8, "4 chunks of 8 words per warp load");
    auto load_group = [&](long long gbase, long long gst) -> unsigned {
        const long long cc = gbase + (long long)(lane >> 3) * gst;
        const long long ww = cc * kCW + (lane & 7);
        return (cc < nchunks && ww < b.words) ? __ldcg(b.visited + ww) : FULL;
    };
    // b.reverse: the grid walks the vertex range downwards (every warp its groups in reverse
    // order), so a BU step that follows another starts where the previous one ended, on the
    // head32 / level / parent lines still in L2
    const long long st = nw;
    const long long ng = gw < nchunks ? (nchunks - 1 - gw) / (4 * nw) + 1 : 0;   // this warp's groups
    const long long gstep = b.reverse ? -4 * nw : 4 * nw;
    long long gb = b.reverse && ng > 0 ? gw + (ng - 1) * 4 * nw : gw;
    unsigned grp_next = load_group(gb, st);
#if XBFS_BU_PROF
    long long pt[6] = {0, 0, 0, 0, 0, 0};
    long long tq = clock64();
#endif
    for (long long gi = 0; gi < ng; ++gi, gb += gstep) {
        const unsigned grp = grp_next;
        grp_next = gi + 1 < ng ? load_group(gb + gstep, nw) : FULL;
        const long long g0 = gb;
        // A sparse group (<= kCW*32 candidates over its 4 chunks, the late BU levels)
        // runs as ONE batch: one first-probe round trip for all of it instead of one
        // per chunk.  Dense groups run chunk by chunk.
        const int gcnt = (int)__reduce_add_sync(FULL, (unsigned)__popc(~grp));
        if (gcnt == 0) continue;
        const bool whole = gcnt <= kCW * 32;
        unsigned has = whole ? 1u : __ballot_sync(FULL, grp != FULL);   // lanes whose word has a candidate
        for (int j = 0; has; ++j, has >>= (whole ? 1 : 8)) {
            if (!whole && (has & 0xffu) == 0u) continue;
            const long long c = g0 + (long long)j * st;
            // 1. candidates of the batch's bitmap words: ballot/popc compaction into shared
            //    memory (the paper's count + prefix-sum + queue-write "double scan").
            long long w;
            bool own;
            unsigned vis;
            if (whole) {                 // lane l: word (l & 7) of chunk g0 + (l >> 3) * nw
                const long long cc = g0 + (long long)(lane >> 3) * st;
                w = cc * kCW + (lane & 7);
                own = cc < nchunks && w < b.words;
                vis = own ? grp : FULL;
            } else {                     // lanes 0..kCW-1: the words of chunk c
                const unsigned vis_j = __shfl_sync(FULL, grp, (j << 3) | (lane & 7));
                w = c * kCW + lane;
                own = lane < kCW && w < b.words;
                vis = own ? vis_j : FULL;
            }
            // the lane owning v's word (index into the found / look-ahead words)
            auto slot = [&](int v) -> int {
                const long long wv = v >> 5;
                if (whole) {
                    const long long cv = wv / kCW;
                    const int jj = st == 1 ? (int)(cv - g0) : (cv >= g0 + st) + (cv >= g0 + 2 * st) + (cv >= g0 + 3 * st);
                    return jj * kCW + (int)(wv & (kCW - 1));
                }
                return (int)(wv - c * kCW);
            };
            auto put = [&](int v, int pu) {
                st_out(b.level + v, b.lvl);
                st_out(b.parent + v, pu);
            };
            const unsigned cand = ~vis;
            // (chunks without a candidate were skipped above: F_{k+1} words start out
            // zero, the stale-bitmap clear of level k-1, so there is nothing to write)
            const int cnt = __popc(cand);
            int incl = cnt;
    #pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const int t = __shfl_up_sync(FULL, incl, o);
                if (lane >= o) incl += t;
            }
            const int total = __shfl_sync(FULL, incl, 31);
            int pos = incl - cnt;
            if (XBFS_BU_PCOMP && !whole) {
                // dense chunk: word i's candidates are written by the lanes of their bit
                // positions, one store per lane per word (kCW rounds instead of up to 32
                // serial ones in the busiest lane)
#pragma unroll
                for (int i = 0; i < kCW; ++i) {
                    const unsigned ci = __shfl_sync(FULL, cand, i);
                    const int pi = __shfl_sync(FULL, pos, i);
                    const long long wi = c * kCW + i;
                    if ((ci >> lane) & 1u) s_list[wib][pi + __popc(ci & lt)] = (int)(wi * 32 + lane);
                }
            } else {
                for (unsigned bits = cand; bits; bits &= bits - 1) s_list[wib][pos++] = (int)(w * 32 + __ffs(bits) - 1);
            }
            s_found[wib][lane] = 0;
            if constexpr (LA) sm.la[wib][lane] = 0;
            __syncwarp();
            // a look-ahead discovery of v (level k+2) with parent pu (F_{k+1})
            auto la_store = [&](int v, int pu, long long deg) {
                if constexpr (LA) {
                    b.level[v] = b.lvl + 1;
                    b.parent[v] = pu;
                    atomicOr(&sm.la[wib][slot(v)], 1u << (v & 31));
                    la.found += 1;
                    la.edges += (unsigned long long)deg;
                }
            };
#if XBFS_BU_PROF
            { const long long t = clock64(); pt[0] += t - tq; tq = t; }
#endif
            // 2. first probe of every candidate, kBuFirstIlp candidates per lane in flight:
            //    head[v] (deg << 32 | first stored neighbour) is a dense array read in
            //    candidate order, so a hit (the common case after the degree-desc
            //    re-arrangement) never touches row_ptr or col.  Misses with more
            //    arcs are compacted in place at the front of s_list.
            int nmiss = 0;
            const unsigned idmask = H32 ? (b.idbits >= 32 ? 0xffffffffu : ((1u << b.idbits) - 1u)) : 0u;
            const unsigned dmax = H32 ? (b.idbits >= 32 ? 0u : (0xffffffffu >> b.idbits)) : 0u;
            for (int base = 0; base < total; base += 32 * kBuFirstIlp) {
                int vv[kBuFirstIlp];
                unsigned long long hv[kBuFirstIlp];
                unsigned wd[kBuFirstIlp], wn[kBuFirstIlp];
    #pragma unroll
                for (int g = 0; g < kBuFirstIlp; ++g) {
                    const int idx = base + g * 32 + lane;
                    vv[g] = idx < total ? s_list[wib][idx] : -1;
                }
                if constexpr (H32) {
                    // unpack to the 64-bit head layout (deg << 32 | first); a saturated
                    // degree stays dmax (>= 2) and is resolved in pass 3 on a hit
    #pragma unroll
                    for (int g = 0; g < kBuFirstIlp; ++g) {
                        const unsigned h = vv[g] >= 0 ? ld_ro32<1>(b.head32 + vv[g]) : 0u;
                        hv[g] = ((unsigned long long)(b.idbits >= 32 ? 0u : (h >> b.idbits)) << 32) | (h & idmask);
                    }
                } else {
    #pragma unroll
                    for (int g = 0; g < kBuFirstIlp; ++g) hv[g] = vv[g] >= 0 ? __ldg(b.head + vv[g]) : 0ull;
                }
    #pragma unroll
                for (int g = 0; g < kBuFirstIlp; ++g) {
                    const int fu = (int)(unsigned)hv[g];
                    wd[g] = vv[g] >= 0 ? ld_cur(b.cur + (fu >> 5)) : 0u;
                    // look-ahead: a degree-1 miss needs its only neighbour's F_{k+1} bit
                    wn[g] = (LA && vv[g] >= 0 && (hv[g] >> 32) == 1) ? __ldcg(b.nxt + (fu >> 5)) : 0u;
                }
                __syncwarp();   // every read of this round is done before the in-place compaction
    #pragma unroll
                for (int g = 0; g < kBuFirstIlp; ++g) {
                    const int v = vv[g];
                    bool miss = false;
                    if (v >= 0) {
                        const int fu = (int)(unsigned)hv[g];
                        const long long d = (long long)(hv[g] >> 32);
                        if ((wd[g] >> (fu & 31)) & 1u) {
                            put(v, fu);
                            atomicOr(&s_found[wib][slot(v)], 1u << (v & 31));
                            if (!H32 || (unsigned)d < dmax) {
                                edges += (unsigned long long)d;
                                fmax = max(fmax, (unsigned)d);
                            } else {
                                miss = true;   // degree-only entry for pass 3 (stored as ~v)
                            }
                            ++found;
                            probes += 1;
                        } else if (d == 1 && (!H32 || dmax > 1)) {
                            probes += 1;
                            if (LA && ((wn[g] >> (fu & 31)) & 1u)) la_store(v, fu, 1);
                        } else {
                            miss = true;
                        }
                    }
                    const unsigned mm = __ballot_sync(FULL, miss);
                    if (miss) {
                        // H32: a hit with a saturated degree goes in as ~v (degree only)
                        const bool deg_only = H32 && ((wd[g] >> ((int)(unsigned)hv[g] & 31)) & 1u);
                        s_list[wib][nmiss + __popc(mm & lt)] = deg_only ? ~v : v;
                    }
                    nmiss += __popc(mm);
                }
            }
            __syncwarp();
#if XBFS_BU_PROF
            { const long long t = clock64(); pt[1] += t - tq; tq = t; pt[5] += nmiss; }
#endif
            // 3. the misses: lane-per-candidate, kBuBatch arcs per step in stored
            //    order from the second arc on (look-ahead: from the first, whose
            //    F_{k+1} bit pass 1 did not read); a lane that finishes takes the
            //    next candidate, so lanes stay busy.
            int v = -1, nxt = 0, nhard = 0, lau = -1;
            long long rs = 0, re = 0, p = 0;
            for (;;) {
                const unsigned need = __ballot_sync(FULL, v < 0);
                if (v < 0) {
                    const int idx = nxt + __popc(need & lt);
                    if (idx < nmiss) {
                        v = s_list[wib][idx];
                        if (H32 && v < 0) {          // found at the first probe; its degree only
                            const int u0 = ~v;
                            const long long dd = b.row_ptr[u0 + 1] - b.row_ptr[u0];
                            edges += (unsigned long long)dd;
                            fmax = max(fmax, (unsigned)dd);
                            v = -1;
                        } else {
                            rs = ld_ro64<4>(b.row_ptr + v);
                            re = ld_ro64<4>(b.row_ptr + v + 1);
                            p = LA ? rs : rs + 1;
                            lau = -1;
                        }
                    }
                }
                nxt += __popc(need);
                if (!__any_sync(FULL, v >= 0) && nxt >= nmiss) break;   // (degree-only entries leave v < 0)
                bool to_hard = false;
                if (v >= 0) {
                    const long long end = min(re, p + kBuBatch);
                    int u[kBuBatch];
                    unsigned wd[kBuBatch], wn[kBuBatch];
    #pragma unroll
                    for (int j = 0; j < kBuBatch; ++j) u[j] = (p + j < end) ? ld_ro32<2>(b.col + p + j) : -1;
    #pragma unroll
                    for (int j = 0; j < kBuBatch; ++j) {
                        wd[j] = u[j] >= 0 ? ld_cur(b.cur + (u[j] >> 5)) : 0u;
                        wn[j] = (LA && lau < 0 && u[j] >= 0) ? __ldcg(b.nxt + (u[j] >> 5)) : 0u;
                    }
                    int hit = -1;
    #pragma unroll
                    for (int j = kBuBatch - 1; j >= 0; --j)
                        if (u[j] >= 0 && ((wd[j] >> (u[j] & 31)) & 1u)) hit = j;   // first hit in row order
                    if (LA && lau < 0) {
    #pragma unroll
                        for (int j = kBuBatch - 1; j >= 0; --j)
                            if (u[j] >= 0 && ((wn[j] >> (u[j] & 31)) & 1u)) lau = u[j];
                    }
                    if (hit >= 0) {
                        int pu = u[0];
    #pragma unroll
                        for (int j = 1; j < kBuBatch; ++j) if (j == hit) pu = u[j];
                        put(v, pu);
                        atomicOr(&s_found[wib][slot(v)], 1u << (v & 31));
                        edges += (unsigned long long)(re - rs);
                        fmax = max(fmax, (unsigned)(re - rs));
                        ++found;
                        probes += (unsigned long long)(p + hit + 1 - rs);
                        v = -1;
                    } else if (end == re) {
                        probes += (unsigned long long)(re - rs);
                        if (LA && lau >= 0) la_store(v, lau, re - rs);
                        v = -1;
                    } else if (re - end > kBuHardMin) {
                        to_hard = true;
                    } else {
                        p = end;
                    }
                }
                const unsigned hm = __ballot_sync(FULL, to_hard);
                if (to_hard) {
                    const int hi = nhard + __popc(hm & lt);
                    s_hard[wib][hi] = v;
                    s_hoff[wib][hi] = (int)(p + kBuBatch - rs);
                    if constexpr (LA) sm.hlau[wib][hi] = lau;
                    v = -1;
                }
                nhard += __popc(hm);
            }
            __syncwarp();
#if XBFS_BU_PROF
            { const long long t = clock64(); pt[2] += t - tq; tq = t; }
#endif
            // 4. long unresolved rows: the whole warp probes 32 arcs per step, first hit wins
            for (int h = 0; h < nhard; ++h) {
                const int hv = s_hard[wib][h];
                const long long hrs = b.row_ptr[hv], hre = b.row_ptr[hv + 1];
                int hl = -1;
                if constexpr (LA) hl = sm.hlau[wib][h];
                bool hit_any = false;
                for (long long base = hrs + s_hoff[wib][h]; base < hre; base += 32) {
                    const long long pp = base + lane;
                    const int u = pp < hre ? __ldg(b.col + pp) : -1;
                    const bool hit = u >= 0 && ((ld_cur(b.cur + (u >> 5)) >> (u & 31)) & 1u);
                    const unsigned m = __ballot_sync(FULL, hit);
                    if (m) {
                        const int first = __ffs(m) - 1;
                        if (lane == first) {
                            put(hv, u);
                            atomicOr(&s_found[wib][slot(hv)], 1u << (hv & 31));
                            edges += (unsigned long long)(hre - hrs);
                            fmax = max(fmax, (unsigned)(hre - hrs));
                            ++found;
                            probes += (unsigned long long)(pp + 1 - hrs);
                        }
                        hit_any = true;
                        break;
                    }
                    if (LA && hl < 0) {
                        const bool nb = u >= 0 && ((__ldcg(b.nxt + (u >> 5)) >> (u & 31)) & 1u);
                        const unsigned mn = __ballot_sync(FULL, nb);
                        if (mn) hl = __shfl_sync(FULL, u, __ffs(mn) - 1);
                    }
                }
                if (!hit_any && lane == 0) {
                    probes += (unsigned long long)(hre - hrs);
                    if (LA && hl >= 0) la_store(hv, hl, hre - hrs);
                }
            }
            __syncwarp();
#if XBFS_BU_PROF
            { const long long t = clock64(); pt[3] += t - tq; tq = t; }
#endif
            if (own) {
                const unsigned f = s_found[wib][lane];
                unsigned lf = 0u;
                if constexpr (LA) lf = sm.la[wib][lane];
                if (f | lf) publish(w, vis, f, lf);   // zero words are already zero in every replica
            }
            __syncwarp();
#if XBFS_BU_PROF
            { const long long t = clock64(); pt[4] += t - tq; tq = t; }
#endif
        }
    }
#if XBFS_BU_PROF
    // per-warp phase cycles: [0] scan+compaction, [1] first probes, [2] miss loop, [3] hard rows,
    // [4] publish, [5] misses; [6] warps, [7] max warp total (imbalance)
    if (lane == 0 && b.prof) {
        long long tot = 0;
        for (int i = 0; i < 6; ++i) { atomicAdd(b.prof + i, (unsigned long long)pt[i]); if (i < 5) tot += pt[i]; }
        atomicAdd(b.prof + 6, 1ull);
        atomicMax(b.prof + 7, (unsigned long long)tot);
    }
#endif
}

}  // namespace xbfs
