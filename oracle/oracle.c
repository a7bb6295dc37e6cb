/*
 * oracle.c — plain, slow, obviously-correct CPU oracle for the XBFS hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this library.
 * It shares no code, header, table or helper with the CUDA path
 * (paper_conf_sc_yangls0w24_b200/csrc); neither includes the other.
 *
 * What it computes (PAPER.md = "P", line numbers; SURVEY.md §8(c) readings):
 *   oracle_build_csr   O-3: symmetric CSR of the input tuples, self-loops and
 *                      duplicate arcs dropped, each row sorted by id.  The paper
 *                      stores graphs symmetric (Tab II |M| = 2x undirected
 *                      edges; reading C-2, C-3) with 8-byte edge
 *                      offsets and 4-byte vertex ids.
 *   oracle_reorder     a2: degree-aware neighbour re-arrangement (P:L153
 *                      §IV-B): each row sorted by neighbour degree descending,
 *                      ties by id ascending (reading C-12).
 *   oracle_reorder_by  the same with degrees from another CSR (directed in-arc
 *                      rows ordered by the in-neighbour's out-degree, R-9).
 *   oracle_first_parents  reading R-12: parent[v] = the first vertex of v's
 *                      stored row one level up (the CUDA path's deterministic
 *                      choice among the valid parents of C-14).
 *   oracle_bfs         O-4: textbook FIFO-queue BFS; the "status array" holds
 *                      the visit level, level[s] = 0 (C-6), -1 = not
 *                      reached (C-1), parent[s] = s.
 *   oracle_validate    O-5: Graph500 validation V1..V5 of a (level, parent)
 *                      pair against the input tuples.
 *   oracle_input_edges O-6: Graph500 m = #tuples (i,j) with level[i] >= 0.
 *   oracle_level_stats per level k: |F_k|, edgesF_k = sum of deg over F_k
 *                      (the numerator of the paper's ratio).
 *   oracle_select      the paper's strategy rule (§III): BU iff
 *                      edgesF_k / |M| > alpha; otherwise SF/SS by frontier growth
 *                      (rule unstated in the paper: reading C-10), plus the
 *                      optional stay-in-BU hysteresis of reading C-11.
 *   oracle_select_sequence  the selector replayed level by level over a BFS:
 *                      |F_k|, edgesF_k, U_k from the level array, the rule above.
 *   oracle_byte_replay O-8: algorithmic bytes of one BFS given the per-level
 *                      strategy sequence, exactly SURVEY §8(d) D-3 (not any
 *                      kernel's traffic model).
 *   oracle_build_csr_directed  f4 (directed graphs; reading
 *                      R-9): out-arc CSR of the tuples taken as arcs i -> j,
 *                      self-loops and duplicate arcs dropped, rows id-sorted.
 *                      oracle_bfs / oracle_level_stats / oracle_reorder apply
 *                      unchanged to it (BFS follows out-arcs).
 *   oracle_validate_directed  the Graph500 checks restated for arcs: V1, V2,
 *                      V3 as undirected; V4 the tree arc parent[v] -> v exists;
 *                      V5 for every tuple (i,j), i != j: i reached implies j
 *                      reached with level[j] <= level[i] + 1.
 *   (validate_omp.c, liboracle_omp.so) oracle_validate_tuples: the same V1-V5
 *                      restated over the tuple list only (no CSR), OpenMP-parallel,
 *                      for the s27 sizes where the serial oracle is too slow.
 *
 * Parity pins: tests/test_oracle.py (closed forms, scipy brute force,
 * validator mutation tests, hand-computed byte replay).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ---------------------------------------------------------------- O-3 CSR */

/* row_ptr: int64[n+1]; col: int32 capacity >= 2*m.  *arcs_out = A.
 * Two counting-sort passes (textbook LSD order): first group every arc by its
 * source row (unsorted rows), then walk rows v = 0..n-1 and append v to the row
 * of each neighbour u; since the arc set is symmetric, row u then receives its
 * neighbours in ascending id order.  Duplicates are adjacent and dropped. */
int oracle_build_csr(int64_t n, int64_t m, const uint32_t* src, const uint32_t* dst,
                     int64_t* row_ptr, int32_t* col, int64_t* arcs_out) {
    if (n <= 0 || m < 0 || !row_ptr || !col || !arcs_out) return 1;
    for (int64_t e = 0; e < m; ++e)
        if (src[e] >= (uint64_t)n || dst[e] >= (uint64_t)n) return 1;
    int64_t* start = (int64_t*)calloc((size_t)n + 1, sizeof(int64_t));
    int64_t* cur = (int64_t*)malloc(((size_t)n + 1) * sizeof(int64_t));
    int32_t* tmp = (int32_t*)malloc((size_t)(2 * m > 0 ? 2 * m : 1) * sizeof(int32_t));
    if (!start || !cur || !tmp) { free(start); free(cur); free(tmp); return 2; }
    for (int64_t e = 0; e < m; ++e) {
        if (src[e] == dst[e]) continue;              /* self-loop dropped */
        start[src[e] + 1]++; start[dst[e] + 1]++;    /* both arcs (undirected) */
    }
    for (int64_t v = 0; v < n; ++v) start[v + 1] += start[v];
    /* pass 1: arcs grouped by source row, unsorted */
    memcpy(cur, start, (size_t)n * sizeof(int64_t));
    for (int64_t e = 0; e < m; ++e) {
        uint32_t u = src[e], v = dst[e];
        if (u == v) continue;
        tmp[cur[u]++] = (int32_t)v;
        tmp[cur[v]++] = (int32_t)u;
    }
    /* pass 2: row u receives v for every arc (v,u), v ascending */
    memcpy(cur, start, (size_t)n * sizeof(int64_t));
    for (int64_t v = 0; v < n; ++v)
        for (int64_t p = start[v]; p < start[v + 1]; ++p)
            col[cur[tmp[p]]++] = (int32_t)v;
    /* drop duplicate arcs (adjacent in each sorted row), compact */
    int64_t out = 0;
    for (int64_t v = 0; v < n; ++v) {
        int64_t b = start[v], e = start[v + 1];
        row_ptr[v] = out;
        for (int64_t i = b; i < e; ++i) {
            if (i > b && col[i] == col[i - 1]) continue;
            col[out++] = col[i];
        }
    }
    row_ptr[n] = out;
    *arcs_out = out;
    free(start); free(cur); free(tmp);
    return 0;
}

/* ---------------------------------------------------- a2 degree reorder */

static const int64_t* g_rp;   /* degree lookup for the comparator (single-threaded) */

static int cmp_deg_desc(const void* a, const void* b) {
    int32_t x = *(const int32_t*)a, y = *(const int32_t*)b;
    int64_t dx = g_rp[x + 1] - g_rp[x], dy = g_rp[y + 1] - g_rp[y];
    if (dx != dy) return dx > dy ? -1 : 1;   /* larger degree first */
    return (x > y) - (x < y);                 /* tie: id ascending (C-12) */
}

/* Rows of (row_ptr, col) sorted by the neighbour's degree in deg_row_ptr's CSR,
 * descending, ties id ascending.  Undirected: deg_row_ptr = row_ptr.  Directed
 * (R-9): the in-arc rows are ordered by the in-neighbour's OUT-degree. */
int oracle_reorder_by(int64_t n, const int64_t* row_ptr, int32_t* col, const int64_t* deg_row_ptr) {
    if (n <= 0 || !row_ptr || !col || !deg_row_ptr) return 1;
    g_rp = deg_row_ptr;
    for (int64_t v = 0; v < n; ++v)
        qsort(col + row_ptr[v], (size_t)(row_ptr[v + 1] - row_ptr[v]), sizeof(int32_t), cmp_deg_desc);
    g_rp = NULL;
    return 0;
}

int oracle_reorder(int64_t n, const int64_t* row_ptr, int32_t* col) {
    return oracle_reorder_by(n, row_ptr, col, row_ptr);
}

/* ------------------------------------------------------------- O-4 BFS */

/* level, parent: int32[n].  Returns the number of levels (max level + 1). */
int32_t oracle_bfs(int64_t n, const int64_t* row_ptr, const int32_t* col, int64_t s,
                   int32_t* level, int32_t* parent) {
    if (n <= 0 || s < 0 || s >= n) return -1;
    int32_t* Q = (int32_t*)malloc((size_t)n * sizeof(int32_t));
    if (!Q) return -2;
    for (int64_t v = 0; v < n; ++v) { level[v] = -1; parent[v] = -1; }
    int64_t head = 0, tail = 0;
    level[s] = 0; parent[s] = (int32_t)s; Q[tail++] = (int32_t)s;
    int32_t maxl = 0;
    while (head < tail) {
        int32_t u = Q[head++];
        for (int64_t p = row_ptr[u]; p < row_ptr[u + 1]; ++p) {
            int32_t v = col[p];
            if (level[v] == -1) {
                level[v] = level[u] + 1;
                parent[v] = u;
                if (level[v] > maxl) maxl = level[v];
                Q[tail++] = v;
            }
        }
    }
    free(Q);
    return maxl + 1;
}

/* Reading R-12 (C-14 "any valid parent", made deterministic): parent[s] = s;
 * for every other reached v, the FIRST u in v's stored row (row_ptr/col as
 * given: the re-arranged rows; the in-arc rows of a directed graph)
 * with level[u] == level[v] - 1; -1 if unreached.  Returns the number of
 * reached v != s without such a neighbour (0 for a true BFS level array). */
int64_t oracle_first_parents(int64_t n, const int64_t* row_ptr, const int32_t* col, const int32_t* level,
                             int64_t s, int32_t* parent) {
    int64_t orphans = 0;
    for (int64_t v = 0; v < n; ++v) {
        parent[v] = -1;
        if (level[v] < 0) continue;
        if (v == s) { parent[v] = (int32_t)s; continue; }
        for (int64_t p = row_ptr[v]; p < row_ptr[v + 1]; ++p)
            if (level[col[p]] == level[v] - 1) { parent[v] = col[p]; break; }
        if (parent[v] < 0) orphans++;
    }
    return orphans;
}

/* ------------------------------------------------- O-5 Graph500 checks */

enum { V1_ROOT = 1, V2_REACH_CONSISTENT = 2, V3_LEVEL_STEP = 4, V4_TREE_EDGE = 8,
       V5_EDGE_SPAN = 16, V_RANGE = 32 };

static int has_arc(const int64_t* row_ptr, const int32_t* col, int32_t u, int32_t v) {
    int64_t lo = row_ptr[u], hi = row_ptr[u + 1];       /* rows sorted by id */
    while (lo < hi) {
        int64_t mid = lo + (hi - lo) / 2;
        if (col[mid] < v) lo = mid + 1; else hi = mid;
    }
    return lo < row_ptr[u + 1] && col[lo] == v;
}

/* Returns a bitmask of failed checks (0 = valid).  row_ptr/col must be the
 * oracle's own id-sorted CSR (oracle_build_csr), not a reordered copy. */
int oracle_validate(int64_t n, const int64_t* row_ptr, const int32_t* col,
                    int64_t m, const uint32_t* src, const uint32_t* dst, int64_t s,
                    const int32_t* level, const int32_t* parent) {
    int bad = 0;
    if (s < 0 || s >= n) return V_RANGE;
    if (parent[s] != s || level[s] != 0) bad |= V1_ROOT;                      /* V1 */
    for (int64_t v = 0; v < n; ++v) {
        int reached_l = level[v] >= 0, reached_p = parent[v] >= 0;
        if (reached_l != reached_p) { bad |= V2_REACH_CONSISTENT; continue; } /* V2 */
        /* V2 (§8(b) semantics, reading C-1): unreached means exactly level = parent = -1 */
        if (!reached_l && (level[v] != -1 || parent[v] != -1)) { bad |= V2_REACH_CONSISTENT; continue; }
        if (parent[v] >= n || level[v] < -1) { bad |= V_RANGE; continue; }
        if (!reached_l || v == s) continue;
        int32_t p = parent[v];
        if (level[p] != level[v] - 1) bad |= V3_LEVEL_STEP;                   /* V3 */
        if (!has_arc(row_ptr, col, p, (int32_t)v)) bad |= V4_TREE_EDGE;       /* V4 */
    }
    for (int64_t e = 0; e < m; ++e) {                                          /* V5 */
        int32_t li = level[src[e]], lj = level[dst[e]];
        if ((li >= 0) != (lj >= 0)) { bad |= V5_EDGE_SPAN; continue; }
        if (li >= 0 && (li - lj > 1 || lj - li > 1)) bad |= V5_EDGE_SPAN;
    }
    return bad;
}

/* O-6: Graph500 m = number of input tuples whose first endpoint is reached. */
int64_t oracle_input_edges(int64_t m, const uint32_t* src, const int32_t* level) {
    int64_t c = 0;
    for (int64_t e = 0; e < m; ++e) c += level[src[e]] >= 0;
    return c;
}

/* Per-level |F_k| and edgesF_k (P:L87 ratio numerator) from a level array.
 * Arrays sized >= nlevels.  Returns nlevels. */
int32_t oracle_level_stats(int64_t n, const int64_t* row_ptr, const int32_t* level,
                           int32_t cap, int64_t* fsize, int64_t* fedges) {
    int32_t nl = 0;
    for (int64_t v = 0; v < n; ++v) if (level[v] + 1 > nl) nl = level[v] + 1;
    if (nl > cap) return -1;
    for (int32_t k = 0; k < nl; ++k) { fsize[k] = 0; fedges[k] = 0; }
    for (int64_t v = 0; v < n; ++v) {
        if (level[v] < 0) continue;
        fsize[level[v]]++;
        fedges[level[v]] += row_ptr[v + 1] - row_ptr[v];
    }
    return nl;
}

/* ---------------------------------------------------- strategy selector */
/* P:L87 §III: "if the ratio of neighbors to the total number of edges in the
 * graph exceeds alpha, XBFS selects the bottom-up strategy.  Otherwise, it
 * switches between the scan-free and single-scan strategies based on the
 * growth rate of the number of nodes in the frontier queue."  alpha = 0.1
 * (0.04 on B200, reading C-13/R-4).  Strict '>' (C-8).  Growth rule
 * (unstated; reading C-10): single-scan iff |F_k| > grow * |F_{k-1}| and
 * ratio > ratio_min.  Reading C-11 (optional hysteresis, bu_stay > 0): after a
 * bottom-up step stay bottom-up while |U_k| * bu_stay < edgesF_k.
 * prev = strategy of step k-1 (-1 at k = 0).  0 = SF, 1 = SS, 2 = BU. */
int32_t oracle_select(int64_t f_size, int64_t f_prev, int64_t f_edges, int64_t arcs,
                      double alpha, double grow, double ratio_min,
                      double bu_stay, int32_t prev, int64_t unvisited) {
    double ratio = arcs > 0 ? (double)f_edges / (double)arcs : 0.0;
    if (ratio > alpha) return 2;
    if (bu_stay > 0.0 && prev == 2 && (double)unvisited * bu_stay < (double)f_edges) return 2;
    if ((double)f_size > grow * (double)f_prev && ratio > ratio_min) return 1;
    return 0;
}

/* The selector replayed over one BFS, in level order (P:L87 per level): from
 * the exact level array, |F_k| = #{v : level v = k}, edgesF_k = sum of deg over
 * F_k, U_k = non-isolated vertices not reached at levels <= k (the BU
 * candidates of step k), and strategy[k] = oracle_select(|F_k|, |F_{k-1}|,
 * edgesF_k, A, ..., strategy[k-1], U_k).  Arrays sized >= nlevels.
 * Returns nlevels, or -1 if cap is too small. */
int32_t oracle_select_sequence(int64_t n, const int64_t* row_ptr, const int32_t* level, int32_t cap,
                               double alpha, double grow, double ratio_min, double bu_stay,
                               int8_t* strategy, int64_t* unvisited_out) {
    int32_t nl = 0;
    for (int64_t v = 0; v < n; ++v) if (level[v] + 1 > nl) nl = level[v] + 1;
    if (nl > cap) return -1;
    int64_t* fsize = (int64_t*)calloc((size_t)nl + 1, sizeof(int64_t));
    int64_t* fedges = (int64_t*)calloc((size_t)nl + 1, sizeof(int64_t));
    int64_t* noniso_at = (int64_t*)calloc((size_t)nl + 1, sizeof(int64_t));
    if (!fsize || !fedges || !noniso_at) { free(fsize); free(fedges); free(noniso_at); return -2; }
    int64_t nonisolated = 0;
    for (int64_t v = 0; v < n; ++v) {
        int64_t d = row_ptr[v + 1] - row_ptr[v];
        if (d > 0) nonisolated++;
        if (level[v] < 0) continue;
        fsize[level[v]]++;
        fedges[level[v]] += d;
        if (d > 0) noniso_at[level[v]]++;
    }
    const int64_t arcs = row_ptr[n];
    int64_t reached_noniso = 0;
    int32_t prev = -1;
    for (int32_t k = 0; k < nl; ++k) {
        reached_noniso += noniso_at[k];                 /* visited before step k: levels <= k */
        int64_t u = nonisolated - reached_noniso;
        int32_t s = oracle_select(fsize[k], k > 0 ? fsize[k - 1] : 0, fedges[k], arcs,
                                  alpha, grow, ratio_min, bu_stay, prev, u);
        strategy[k] = (int8_t)s;
        if (unvisited_out) unvisited_out[k] = u;
        prev = s;
    }
    free(fsize); free(fedges); free(noniso_at);
    return nl;
}

/* ------------------------------------------------------ O-8 byte replay */
/* Algorithmic bytes of one BFS, SURVEY §8(d) D-3 exactly, given the strategy
 * used at each level (0 SF, 1 SS, 2 BU) and the (reordered) CSR the GPU
 * traversed.  The D-3 terms (bitmap probes are L2 traffic, not counted):
 *   init       : 8N (level + parent) + 3N/8 (three N-bit bitmaps)
 *   TD step k  : 20|F_k| (queue entry + row_ptr pair) + 4 edgesF_k (col)
 *                + 28|F_{k+1}| (level 4, parent 4, queue 4, row_ptr pair 16 for binning)
 *   SS step k  : the TD terms + N/8 (single-scan generation over the N-bit status bitmap)
 *   BU step k  : N/4 (two bitmaps) + 24|U_k| + 4 probes_k (col) + 8|F_{k+1}| (level, parent)
 * N/8 is rounded up to whole bytes (reading R-11): bm = ceil(N/8), N/4 = 2 bm,
 * 3N/8 = 3 bm.  probes(v) = 1 + index of the first level-k neighbour in v's
 * stored row, or deg(v) if none (BU tests only level k: reading C-9); U_k =
 * non-isolated vertices not reached at levels <= k.  per_level[k] gets the
 * bytes of step k; the return value includes init. */
int64_t oracle_byte_replay(int64_t n, const int64_t* row_ptr, const int32_t* col,
                           const int32_t* level, int32_t nlevels, const int8_t* strategy,
                           int64_t* per_level) {
    const int64_t bm = (n + 7) / 8;
    int64_t total = 8 * n + 3 * bm;
    int64_t* fsize = (int64_t*)calloc((size_t)nlevels + 1, sizeof(int64_t));
    int64_t* fedges = (int64_t*)calloc((size_t)nlevels + 1, sizeof(int64_t));
    if (!fsize || !fedges) { free(fsize); free(fedges); return -1; }
    int64_t nonisolated = 0;
    for (int64_t v = 0; v < n; ++v) {
        int64_t d = row_ptr[v + 1] - row_ptr[v];
        nonisolated += d > 0;
        if (level[v] >= 0 && level[v] < nlevels) { fsize[level[v]]++; fedges[level[v]] += d; }
    }
    int64_t unvisited = nonisolated;     /* U_0: non-isolated vertices other than the source */
    for (int64_t v = 0; v < n; ++v)
        if (level[v] == 0 && row_ptr[v + 1] > row_ptr[v]) unvisited--;
    for (int32_t k = 0; k < nlevels; ++k) {
        int64_t bytes = 0;
        int64_t found = fsize[k + 1];                        /* |F_{k+1}| (0 past the end) */
        if (strategy[k] == 2) {
            int64_t probes = 0;
            for (int64_t v = 0; v < n; ++v) {
                if (row_ptr[v + 1] == row_ptr[v]) continue;      /* isolated: not a candidate */
                if (level[v] >= 0 && level[v] <= k) continue;     /* visited before step k */
                int64_t pr = row_ptr[v + 1] - row_ptr[v];
                for (int64_t p = row_ptr[v]; p < row_ptr[v + 1]; ++p)
                    if (level[col[p]] == k) { pr = p - row_ptr[v] + 1; break; }
                probes += pr;
            }
            bytes = 2 * bm + 24 * unvisited + 4 * probes + 8 * found;
        } else {
            bytes = 20 * fsize[k] + 4 * fedges[k] + 28 * found;
            if (strategy[k] == 1) bytes += bm;                  /* SS: the single scan */
        }
        unvisited -= found;
        if (per_level) per_level[k] = bytes;
        total += bytes;
    }
    free(fsize); free(fedges);
    return total;
}

/* Arcs a bottom-up step at level k probes (P:L124-131 early termination): over
 * the candidates (non-isolated, not reached by level k), 1 + index of the first
 * neighbour at level k in the stored row, or the whole degree if none. */
int64_t oracle_bu_probes(int64_t n, const int64_t* row_ptr, const int32_t* col,
                         const int32_t* level, int32_t k) {
    int64_t probes = 0;
    for (int64_t v = 0; v < n; ++v) {
        if (row_ptr[v + 1] == row_ptr[v]) continue;
        if (level[v] >= 0 && level[v] <= k) continue;
        int64_t pr = row_ptr[v + 1] - row_ptr[v];
        for (int64_t p = row_ptr[v]; p < row_ptr[v + 1]; ++p)
            if (level[col[p]] == k) { pr = p - row_ptr[v] + 1; break; }
        probes += pr;
    }
    return probes;
}

/* ------------------------------------------- f4: directed graphs (R-9) */

/* Out-arc CSR: every tuple (i,j), i != j, is the arc i -> j.  Same two-pass
 * counting sort as oracle_build_csr, one arc per tuple: pass 1 groups arcs by
 * target j, pass 2 walks targets j = 0..n-1 and appends j to the row of each
 * source i, so every row receives its targets in ascending id order;
 * duplicates are then adjacent and dropped.  col capacity >= m. */
int oracle_build_csr_directed(int64_t n, int64_t m, const uint32_t* src, const uint32_t* dst,
                              int64_t* row_ptr, int32_t* col, int64_t* arcs_out) {
    if (n <= 0 || m < 0 || !row_ptr || !col || !arcs_out) return 1;
    for (int64_t e = 0; e < m; ++e)
        if (src[e] >= (uint64_t)n || dst[e] >= (uint64_t)n) return 1;
    int64_t* tstart = (int64_t*)calloc((size_t)n + 1, sizeof(int64_t));   /* by target */
    int64_t* start = (int64_t*)calloc((size_t)n + 1, sizeof(int64_t));    /* by source */
    int64_t* cur = (int64_t*)malloc(((size_t)n + 1) * sizeof(int64_t));
    int32_t* tmp = (int32_t*)malloc((size_t)(m > 0 ? m : 1) * sizeof(int32_t));
    if (!tstart || !start || !cur || !tmp) { free(tstart); free(start); free(cur); free(tmp); return 2; }
    for (int64_t e = 0; e < m; ++e) {
        if (src[e] == dst[e]) continue;              /* self-loop dropped */
        tstart[dst[e] + 1]++;
        start[src[e] + 1]++;
    }
    for (int64_t v = 0; v < n; ++v) { tstart[v + 1] += tstart[v]; start[v + 1] += start[v]; }
    /* pass 1: sources grouped by target */
    memcpy(cur, tstart, (size_t)n * sizeof(int64_t));
    for (int64_t e = 0; e < m; ++e) {
        if (src[e] == dst[e]) continue;
        tmp[cur[dst[e]]++] = (int32_t)src[e];
    }
    /* pass 2: row i receives j for every arc i -> j, j ascending */
    memcpy(cur, start, (size_t)n * sizeof(int64_t));
    for (int64_t j = 0; j < n; ++j)
        for (int64_t p = tstart[j]; p < tstart[j + 1]; ++p)
            col[cur[tmp[p]]++] = (int32_t)j;
    int64_t out = 0;
    for (int64_t v = 0; v < n; ++v) {
        int64_t b = start[v], e = start[v + 1];
        row_ptr[v] = out;
        for (int64_t i = b; i < e; ++i) {
            if (i > b && col[i] == col[i - 1]) continue;
            col[out++] = col[i];
        }
    }
    row_ptr[n] = out;
    *arcs_out = out;
    free(tstart); free(start); free(cur); free(tmp);
    return 0;
}

/* Validation of a BFS over arcs.  row_ptr/col: oracle_build_csr_directed's
 * id-sorted out-arc CSR.  Same bitmask as oracle_validate. */
int oracle_validate_directed(int64_t n, const int64_t* row_ptr, const int32_t* col,
                             int64_t m, const uint32_t* src, const uint32_t* dst, int64_t s,
                             const int32_t* level, const int32_t* parent) {
    int bad = 0;
    if (s < 0 || s >= n) return V_RANGE;
    if (parent[s] != s || level[s] != 0) bad |= V1_ROOT;                      /* V1 */
    for (int64_t v = 0; v < n; ++v) {
        int reached_l = level[v] >= 0, reached_p = parent[v] >= 0;
        if (reached_l != reached_p) { bad |= V2_REACH_CONSISTENT; continue; } /* V2 */
        /* V2 (§8(b) semantics, reading C-1): unreached means exactly level = parent = -1 */
        if (!reached_l && (level[v] != -1 || parent[v] != -1)) { bad |= V2_REACH_CONSISTENT; continue; }
        if (parent[v] >= n || level[v] < -1) { bad |= V_RANGE; continue; }
        if (!reached_l || v == s) continue;
        int32_t p = parent[v];
        if (level[p] != level[v] - 1) bad |= V3_LEVEL_STEP;                   /* V3 */
        if (!has_arc(row_ptr, col, p, (int32_t)v)) bad |= V4_TREE_EDGE;       /* V4: arc p -> v */
    }
    for (int64_t e = 0; e < m; ++e) {                                          /* V5 */
        if (src[e] == dst[e]) continue;
        int32_t li = level[src[e]], lj = level[dst[e]];
        if (li < 0) continue;                        /* nothing follows from an unreached tail */
        if (lj < 0 || lj > li + 1) bad |= V5_EDGE_SPAN;
    }
    return bad;
}
