/*
 * synth.c — seeded synthetic graph generators (INPUTS ONLY).
 *
 * This module is shared by the CUDA path's harness (bench.py) and by the
 * oracle-based tests.  It holds none of the BFS method's arithmetic: it only
 * produces edge tuples and root vertices.  Recipe fixed in SURVEY.md §8(c) O-1,
 * O-2, O-7 (the paper gives no generator parameters: PAPER.md L194-195,
 * Tab II "Rmat23 / Rmat25"), restated in DESIGN.md §3.
 *
 *   splitmix64(x)      : the standard 64-bit finaliser (Steele/Vigna).
 *   U(seed, e, k)      : (splitmix64(splitmix64(seed) ^ (e*2s + k)) >> 11) * 2^-53
 *   Kronecker tuple e  : s bit-levels, quadrant probabilities A,B,C,D =
 *                        0.57, 0.19, 0.19, 0.05 (Graph500), then both endpoints
 *                        relabelled by the seeded bijection pi on s-bit ints.
 *   grid (W x H)       : 4-neighbour lattice, id(x,y) = y*W + x.
 *   roots              : stream splitmix64(root_seed + t) mod N, skipping
 *                        repeats and vertices with no non-self-loop tuple.
 *
 * Build: gcc -O3 -fopenmp -shared -fPIC (see __graft_entry__.build()).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

static inline uint64_t splitmix64(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

uint64_t synth_splitmix64(uint64_t x) { return splitmix64(x); }

/* U(seed,e,k) with hs = splitmix64(seed) precomputed. */
static inline double unif(uint64_t hs, uint64_t ctr) {
    return (double)(splitmix64(hs ^ ctr) >> 11) * (1.0 / 9007199254740992.0);
}

double synth_uniform(uint64_t seed, uint64_t e, uint64_t k, int32_t scale) {
    return unif(splitmix64(seed), e * 2ull * (uint64_t)scale + k);
}

/* pi: 4 rounds of  v ^= c_r & mask; v = (v*K_r) & mask; v ^= v >> ceil(s/2).
 * c_r = splitmix64(seed ^ (2r+1)), K_r = splitmix64(seed ^ (2r+2)) | 1. */
typedef struct { uint64_t c[4], k[4], mask; int sh; } perm_t;

static void perm_init(perm_t* p, uint64_t seed, int scale) {
    p->mask = (scale >= 64) ? ~0ull : ((1ull << scale) - 1ull);
    p->sh = (scale + 1) / 2;
    for (int r = 0; r < 4; ++r) {
        p->c[r] = splitmix64(seed ^ (uint64_t)(2 * r + 1));
        p->k[r] = splitmix64(seed ^ (uint64_t)(2 * r + 2)) | 1ull;
    }
}

static inline uint64_t perm_apply(const perm_t* p, uint64_t v) {
    for (int r = 0; r < 4; ++r) {
        v ^= p->c[r] & p->mask;
        v = (v * p->k[r]) & p->mask;
        if (p->sh > 0) v ^= v >> p->sh;
    }
    return v;
}

uint64_t synth_perm(uint64_t seed, int32_t scale, uint64_t v) {
    perm_t p; perm_init(&p, seed, scale);
    return perm_apply(&p, v);
}

/* Graph500 Kronecker: tuples [e_begin, e_end) of the M = ef*2^s stream.
 * Writes uint32 endpoints (requires scale <= 32).  permute=0 skips pi
 * (used by the generator's own statistical tests of the quadrant law). */
int synth_kronecker(int32_t scale, uint64_t seed, int64_t e_begin, int64_t e_end,
                    int32_t permute, uint32_t* src, uint32_t* dst) {
    if (scale < 1 || scale > 32 || e_end < e_begin || !src || !dst) return 1;
    const double A = 0.57, B = 0.19, C = 0.19;
    const double ab = A + B, a_norm = A / ab, c_norm = C / (1.0 - ab);
    const uint64_t hs = splitmix64(seed);
    perm_t p; perm_init(&p, seed, scale);
    const uint64_t two_s = 2ull * (uint64_t)scale;
#pragma omp parallel for schedule(static)
    for (int64_t e = e_begin; e < e_end; ++e) {
        uint64_t i = 0, j = 0;
        const uint64_t base = (uint64_t)e * two_s;
        for (int b = 0; b < scale; ++b) {
            double r1 = unif(hs, base + 2ull * b);
            double r2 = unif(hs, base + 2ull * b + 1ull);
            uint64_t ii = r1 > ab;
            uint64_t jj = r2 > (ii ? c_norm : a_norm);
            i |= ii << b;
            j |= jj << b;
        }
        if (permute) { i = perm_apply(&p, i); j = perm_apply(&p, j); }
        src[e - e_begin] = (uint32_t)i;
        dst[e - e_begin] = (uint32_t)j;
    }
    return 0;
}

/* Number of tuples the grid generator emits for a W x H box. */
int64_t synth_grid_count(int32_t W, int32_t H) {
    return 2ll * W * H - W - H;
}

/* 2D 4-neighbour grid, row-major ids; for each (y,x) in row-major order emit
 * the right neighbour (if any) then the down neighbour (if any).
 * perm_scale > 0 relabels ids by pi on perm_scale bits (W*H must be 2^perm_scale).
 * keep_prob < 1 drops tuple e unless U(seed,e,0) < keep_prob ("road-like"); the
 * kept count is returned through *m_out. */
int synth_grid(int32_t W, int32_t H, uint64_t seed, int32_t perm_scale, double keep_prob,
               uint32_t* src, uint32_t* dst, int64_t* m_out) {
    if (W < 1 || H < 1 || !src || !dst || !m_out) return 1;
    perm_t p; if (perm_scale > 0) perm_init(&p, seed, perm_scale);
    const uint64_t hs = splitmix64(seed);
    int64_t e = 0, kept = 0;
    for (int64_t y = 0; y < H; ++y) {
        for (int64_t x = 0; x < W; ++x) {
            uint64_t a = (uint64_t)(y * W + x);
            for (int d = 0; d < 2; ++d) {
                uint64_t b;
                if (d == 0) { if (x + 1 >= W) continue; b = a + 1; }
                else        { if (y + 1 >= H) continue; b = a + (uint64_t)W; }
                int keep = keep_prob >= 1.0 || unif(hs, (uint64_t)e * 2ull * 24ull) < keep_prob;
                ++e;
                if (!keep) continue;
                uint64_t u = a, v = b;
                if (perm_scale > 0) { u = perm_apply(&p, u); v = perm_apply(&p, v); }
                src[kept] = (uint32_t)u; dst[kept] = (uint32_t)v; ++kept;
            }
        }
    }
    *m_out = kept;
    return 0;
}

/* Roots: candidates splitmix64(root_seed + t) mod N for
 * t = 0,1,...; skip repeats and vertices that touch no non-self-loop tuple
 * (degree 0 in the symmetric, self-loop-free CSR).  Returns how many roots
 * were written (< count only if fewer eligible vertices exist). */
int64_t synth_roots(int64_t n, int64_t m, const uint32_t* src, const uint32_t* dst,
                    uint64_t root_seed, int64_t count, int64_t* roots) {
    if (n <= 0 || count <= 0) return 0;
    uint8_t* ok = (uint8_t*)calloc((size_t)n, 1);
    uint8_t* used = (uint8_t*)calloc((size_t)n, 1);
    if (!ok || !used) { free(ok); free(used); return -1; }
    for (int64_t e = 0; e < m; ++e) {
        if (src[e] != dst[e]) { ok[src[e]] = 1; ok[dst[e]] = 1; }
    }
    int64_t eligible = 0;
    for (int64_t v = 0; v < n; ++v) eligible += ok[v];
    int64_t want = count < eligible ? count : eligible, got = 0;
    for (uint64_t t = 0; got < want; ++t) {
        int64_t v = (int64_t)(splitmix64(root_seed + t) % (uint64_t)n);
        if (!ok[v] || used[v]) continue;
        used[v] = 1; roots[got++] = v;
    }
    free(ok); free(used);
    return got;
}
