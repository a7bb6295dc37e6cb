/*
 * validate_omp.c — Graph500 validation O-5 (V1..V5) over the input TUPLE LIST,
 * OpenMP-parallel, for sizes where the serial oracle CSR is too slow (s27:
 * 134 M vertices, 2.1 G tuples).
 *
 * TEST INFRASTRUCTURE ONLY (part of oracle/, same rules as oracle.c): only
 * tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / reference legs
 * load it.  Shares nothing with the CUDA path.
 *
 * SURVEY §8(c) O-5, restated over tuples (src[e], dst[e]) instead of a CSR:
 *   V1  parent[s] == s and level[s] == 0
 *   V2  level[v] >= 0  <=>  parent[v] >= 0; an unreached vertex has exactly
 *       level = parent = -1 (§8(b) semantics, reading C-1)
 *   V3  every reached v != s: level[parent[v]] == level[v] - 1
 *   V4  every reached v != s: (parent[v], v) is an input edge, i.e. some tuple
 *       (i, j), i != j, has {i, j} = {parent[v], v}  (directed: (i, j) = (parent[v], v))
 *   V5  every tuple (i, j): both or neither endpoint reached and
 *       |level[i] - level[j]| <= 1  (directed, i != j: i reached => j reached
 *       with level[j] <= level[i] + 1)
 * V4 is checked the way the Graph500 reference does it: one pass over the
 * tuples marks every vertex whose tree edge it is; every reached v != s must be
 * marked.  V1..V5 together pin level[v] = dist(s, v) exactly (the certificate
 * in SURVEY §8(c) O-5), so this validates the levels of roots the serial BFS
 * cannot afford.  Same bitmask as oracle_validate (oracle.c).
 */
#include <stdint.h>
#include <stdlib.h>

enum { V1_ROOT = 1, V2_REACH_CONSISTENT = 2, V3_LEVEL_STEP = 4, V4_TREE_EDGE = 8,
       V5_EDGE_SPAN = 16, V_RANGE = 32 };

int oracle_validate_tuples(int64_t n, int64_t m, const uint32_t* src, const uint32_t* dst, int64_t s,
                           const int32_t* level, const int32_t* parent, int32_t directed, int32_t threads) {
    if (n <= 0 || s < 0 || s >= n) return V_RANGE;
    if (threads <= 0) threads = 1;
    int bad = 0;
    if (parent[s] != s || level[s] != 0) bad |= V1_ROOT;                          /* V1 */
    /* V2, range, V3: one pass over the vertices */
#pragma omp parallel for num_threads(threads) reduction(| : bad) schedule(static)
    for (int64_t v = 0; v < n; ++v) {
        const int32_t lv = level[v], pv = parent[v];
        if ((lv >= 0) != (pv >= 0)) { bad |= V2_REACH_CONSISTENT; continue; }
        if (lv < 0) {
            if (lv != -1 || pv != -1) bad |= V2_REACH_CONSISTENT;
            continue;
        }
        if (pv >= n) { bad |= V_RANGE; continue; }
        if (v != s && level[pv] != lv - 1) bad |= V3_LEVEL_STEP;                  /* V3 */
    }
    /* V4 marks + V5: one pass over the tuples */
    uint8_t* ok = (uint8_t*)calloc((size_t)n, 1);
    if (!ok) return -1;
#pragma omp parallel for num_threads(threads) reduction(| : bad) schedule(static)
    for (int64_t e = 0; e < m; ++e) {
        const uint32_t i = src[e], j = dst[e];
        if (i >= (uint64_t)n || j >= (uint64_t)n) { bad |= V_RANGE; continue; }
        const int32_t li = level[i], lj = level[j];
        if (directed) {
            if (i == j) continue;
            if (li >= 0 && (lj < 0 || lj > li + 1)) bad |= V5_EDGE_SPAN;       /* V5 (arcs) */
            if (lj >= 0 && parent[j] == (int32_t)i) __atomic_store_n(&ok[j], 1, __ATOMIC_RELAXED);
        } else {
            if ((li >= 0) != (lj >= 0)) { bad |= V5_EDGE_SPAN; continue; }     /* V5 */
            if (li >= 0 && (li - lj > 1 || lj - li > 1)) bad |= V5_EDGE_SPAN;
            if (i == j || li < 0) continue;
            if (parent[j] == (int32_t)i) __atomic_store_n(&ok[j], 1, __ATOMIC_RELAXED);
            if (parent[i] == (int32_t)j) __atomic_store_n(&ok[i], 1, __ATOMIC_RELAXED);
        }
    }
#pragma omp parallel for num_threads(threads) reduction(| : bad) schedule(static)
    for (int64_t v = 0; v < n; ++v)
        if (v != s && level[v] >= 0 && !ok[v]) bad |= V4_TREE_EDGE;               /* V4 */
    free(ok);
    return bad;
}
