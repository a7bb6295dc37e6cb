"""Pins for the CPU oracle (oracle/): every check here is fixed by something
other than the oracle itself — a closed form, an independent library routine
(scipy.sparse.csgraph), a brute-force matrix-power BFS, a hand-computed value,
or a number printed in the paper (tests/golden/).  CPU only."""
import itertools
import json
import os

import numpy as np
import pytest
import scipy.sparse as sp
from scipy.sparse.csgraph import shortest_path

import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _graph(n, edges):
    e = np.asarray(edges, dtype=np.int64).reshape(-1, 2)
    return n, e[:, 0].astype(np.uint32), e[:, 1].astype(np.uint32)


def _levels(n, edges, s):
    n, src, dst = _graph(n, edges)
    g = oracle.build_csr(n, src, dst)
    level, parent, nl = oracle.bfs(g, s)
    assert oracle.validate(g, src, dst, s, level, parent) == 0
    return level, parent, nl


# ---------------------------------------------------------------- closed forms

def test_path_levels():
    n = 37
    for s in (0, 5, 36):
        level, parent, nl = _levels(n, [(i, i + 1) for i in range(n - 1)], s)
        assert np.array_equal(level, np.abs(np.arange(n) - s))
        assert nl == max(s, n - 1 - s) + 1


def test_cycle_levels():
    n = 41
    d = np.arange(n)
    for s in (0, 17):
        level, _, _ = _levels(n, [(i, (i + 1) % n) for i in range(n)], s)
        assert np.array_equal(level, np.minimum(np.abs(d - s), n - np.abs(d - s)))


def test_star_levels_and_parents():
    n = 50
    edges = [(0, i) for i in range(1, n)]
    level, parent, _ = _levels(n, edges, 0)
    assert level[0] == 0 and np.all(level[1:] == 1) and np.all(parent[1:] == 0)
    level, parent, _ = _levels(n, edges, 7)          # from a leaf
    expect = np.full(n, 2); expect[7] = 0; expect[0] = 1
    assert np.array_equal(level, expect)
    assert parent[0] == 7 and all(parent[v] == 0 for v in range(1, n) if v != 7)


def test_complete_graph():
    n = 16
    level, _, nl = _levels(n, list(itertools.combinations(range(n), 2)), 3)
    assert level[3] == 0 and np.all(np.delete(level, 3) == 1) and nl == 2


def test_binary_tree():
    n = 255
    level, parent, _ = _levels(n, [((v - 1) // 2, v) for v in range(1, n)], 0)
    assert np.array_equal(level, np.floor(np.log2(np.arange(n) + 1)).astype(int))
    assert all(parent[v] == (v - 1) // 2 for v in range(1, n))


def test_hypercube_popcount():
    d = 8
    n = 1 << d
    edges = [(v, v ^ (1 << b)) for v in range(n) for b in range(d) if v < v ^ (1 << b)]
    for s in (0, 0b10110011):
        level, _, nl = _levels(n, edges, s)
        assert np.array_equal(level, [bin(v ^ s).count("1") for v in range(n)])
        assert nl == d + 1


def test_grid_manhattan():
    W, H = 23, 17
    idx = lambda x, y: y * W + x
    edges = [(idx(x, y), idx(x + 1, y)) for y in range(H) for x in range(W - 1)]
    edges += [(idx(x, y), idx(x, y + 1)) for y in range(H - 1) for x in range(W)]
    sx, sy = 5, 11
    level, _, _ = _levels(W * H, edges, idx(sx, sy))
    xs, ys = np.meshgrid(np.arange(W), np.arange(H))
    assert np.array_equal(level, (np.abs(xs - sx) + np.abs(ys - sy)).ravel())


def test_disjoint_union_unreached():
    a = [(i, i + 1) for i in range(9)]           # 0..9 path
    b = [(10 + i, 10 + i + 1) for i in range(4)]  # 10..14 path
    level, parent, _ = _levels(20, a + b, 3)      # 15..19 isolated
    assert np.all(level[10:] == -1) and np.all(parent[10:] == -1)
    assert np.array_equal(level[:10], np.abs(np.arange(10) - 3))


def test_isolated_source():
    level, parent, nl = _levels(6, [(0, 1), (1, 2)], 5)
    assert level[5] == 0 and parent[5] == 5 and nl == 1
    assert np.all(np.delete(level, 5) == -1)


def test_self_loops_and_multi_edges_have_no_effect():
    base = [(i, i + 1) for i in range(11)]
    noisy = base + [(3, 3), (7, 7), (2, 3), (3, 2), (2, 3), (0, 1)]
    l1, _, _ = _levels(12, base, 0)
    l2, _, _ = _levels(12, noisy, 0)
    assert np.array_equal(l1, l2)
    n, src, dst = _graph(12, noisy)
    assert oracle.build_csr(n, src, dst).arcs == 22


# ------------------------------------------------- brute force / library pins

def _random_graph(rng, n, m):
    e = rng.integers(0, n, size=(m, 2))
    return e


@pytest.mark.parametrize("seed", range(12))
def test_bfs_matches_scipy_shortest_path(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.integers(2, 64))
    e = _random_graph(rng, n, int(rng.integers(0, 3 * n)))
    n, src, dst = _graph(n, e)
    g = oracle.build_csr(n, src, dst)
    mask = src != dst
    A = sp.coo_matrix((np.ones(mask.sum()), (src[mask], dst[mask])), shape=(n, n)).tocsr()
    D = shortest_path(A, directed=False, unweighted=True)
    for s in range(n):
        level, parent, _ = oracle.bfs(g, s)
        expect = np.where(np.isinf(D[s]), -1, D[s]).astype(np.int64)
        assert np.array_equal(level, expect)
        assert oracle.validate(g, src, dst, s, level, parent) == 0


@pytest.mark.parametrize("seed", range(6))
def test_bfs_matches_boolean_matrix_powers(seed):
    """Textbook brute force: level k set = vertices first reached by A^k."""
    rng = np.random.default_rng(100 + seed)
    n = int(rng.integers(2, 60))
    e = _random_graph(rng, n, int(rng.integers(n // 2, 2 * n + 1)))
    n, src, dst = _graph(n, e)
    adj = np.zeros((n, n), dtype=bool)
    adj[src, dst] = True
    adj[dst, src] = True
    np.fill_diagonal(adj, False)
    g = oracle.build_csr(n, src, dst)
    for s in range(0, n, 3):
        dist = np.full(n, -1)
        reach = np.zeros(n, dtype=bool)
        reach[s] = True
        dist[s] = 0
        k = 0
        while True:
            k += 1
            nxt = (adj[reach].any(axis=0)) & ~reach & (dist == -1)
            if not nxt.any():
                break
            dist[nxt] = k
            reach = nxt
        level, _, _ = oracle.bfs(g, s)
        assert np.array_equal(level, dist)


@pytest.mark.parametrize("seed", range(5))
def test_csr_matches_set_build(seed):
    rng = np.random.default_rng(200 + seed)
    n = int(rng.integers(1, 1 << 12))
    e = _random_graph(rng, n, int(rng.integers(0, 8 * n)))
    n, src, dst = _graph(n, e)
    g = oracle.build_csr(n, src, dst)
    rows = [set() for _ in range(n)]
    for u, v in zip(src.tolist(), dst.tolist()):
        if u != v:
            rows[u].add(v)
            rows[v].add(u)
    rp = np.concatenate([[0], np.cumsum([len(r) for r in rows])])
    col = np.array([c for r in rows for c in sorted(r)], dtype=np.int32)
    assert np.array_equal(g.row_ptr, rp)
    assert np.array_equal(g.col, col)


def test_reorder_invariants():
    rng = np.random.default_rng(7)
    n = 500
    e = np.concatenate([rng.integers(0, n, (3000, 2)), np.stack([np.zeros(200, int), rng.integers(0, n, 200)], 1)])
    n, src, dst = _graph(n, e)
    g = oracle.build_csr(n, src, dst)
    r = oracle.reorder(g)
    deg = g.degree()
    for v in range(n):
        a, b = g.row_ptr[v], g.row_ptr[v + 1]
        row = r.col[a:b]
        assert sorted(row.tolist()) == g.col[a:b].tolist()                 # multiset preserved
        keys = [(-int(deg[c]), int(c)) for c in row]
        assert keys == sorted(keys)                                         # deg desc, id asc
    # levels are invariant under the reorder (only parents change)
    for s in (0, 13, 77):
        assert np.array_equal(oracle.bfs(g, s)[0], oracle.bfs(r, s)[0])


# ------------------------------------------------------------ validator pins

def _valid_case():
    rng = np.random.default_rng(11)
    n = 220                                   # vertices 200..219 are isolated (never reached)
    e = rng.integers(0, 200, (800, 2))
    n, src, dst = _graph(n, e)
    g = oracle.build_csr(n, src, dst)
    s = int(src[0])
    level, parent, _ = oracle.bfs(g, s)
    return g, src, dst, s, level, parent


def test_validator_accepts_oracle_tree():
    g, src, dst, s, level, parent = _valid_case()
    assert oracle.validate(g, src, dst, s, level, parent) == 0


def test_validator_rejects_mutations():
    g, src, dst, s, level, parent = _valid_case()
    reached = np.flatnonzero((level >= 2))
    v = int(reached[0])

    p = parent.copy(); p[s] = int(reached[1])                        # wrong root parent
    assert oracle.validate(g, src, dst, s, level, p) & oracle.V1_ROOT

    # parent = a non-neighbour at the right level (tree edge missing)
    same = [u for u in np.flatnonzero(level == level[v] - 1) if not
            np.isin(v, g.col[g.row_ptr[u]:g.row_ptr[u + 1]])]
    p = parent.copy(); p[v] = int(same[0])
    assert oracle.validate(g, src, dst, s, level, p) & oracle.V4_TREE_EDGE

    # parent at the same level (level step broken)
    p = parent.copy(); p[v] = int(np.flatnonzero(level == level[v])[0 if np.flatnonzero(level == level[v])[0] != v else 1])
    assert oracle.validate(g, src, dst, s, level, p) & (oracle.V3_LEVEL_STEP | oracle.V4_TREE_EDGE)

    # 2-cycle between two reached vertices
    u = int(parent[v]); p = parent.copy(); p[u] = v
    assert oracle.validate(g, src, dst, s, level, p) != 0

    # reached vertex marked unreached in level only
    lv = level.copy(); lv[v] = -1
    assert oracle.validate(g, src, dst, s, lv, parent) & oracle.V2_REACH

    # level off by one everywhere at depth >= 2 (tree still consistent? no: V3/V5)
    lv = level.copy(); lv[level >= 2] += 1
    assert oracle.validate(g, src, dst, s, lv, parent) != 0

    # an unreached vertex marked reached with a bogus parent
    un = np.flatnonzero(level == -1)
    assert un.size
    lv = level.copy(); p = parent.copy(); lv[un[0]] = 1; p[un[0]] = s
    assert oracle.validate(g, src, dst, s, lv, p) != 0

    # §8(b): an unreached vertex holds exactly level = parent = -1 (any other negative fails)
    for bad_l, bad_p in ((-1, -2), (-7, -1), (-7, -7), (-1, -2147483648)):
        lv = level.copy(); p = parent.copy(); lv[un[0]] = bad_l; p[un[0]] = bad_p
        assert oracle.validate(g, src, dst, s, lv, p) & oracle.V2_REACH, (bad_l, bad_p)


# ----------------------------------------------------------- TEPS / stats pins

def test_input_edges_grid_equals_m():
    W, H = 9, 7
    idx = lambda x, y: y * W + x
    edges = [(idx(x, y), idx(x + 1, y)) for y in range(H) for x in range(W - 1)]
    edges += [(idx(x, y), idx(x, y + 1)) for y in range(H - 1) for x in range(W)]
    n, src, dst = _graph(W * H, edges)
    g = oracle.build_csr(n, src, dst)
    level, _, _ = oracle.bfs(g, 0)
    assert oracle.input_edges(src, level) == 2 * W * H - W - H


def test_input_edges_counts_duplicates_and_self_loops():
    # component {0,1,2} + {3,4}; tuples with reached first endpoint from s=0
    edges = [(0, 1), (1, 0), (0, 1), (2, 2), (1, 2), (3, 4), (4, 4)]
    n, src, dst = _graph(5, edges)
    g = oracle.build_csr(n, src, dst)
    level, _, _ = oracle.bfs(g, 0)
    assert oracle.input_edges(src, level) == 5


def test_level_stats_star_hand_values():
    n = 11
    n, src, dst = _graph(n, [(0, i) for i in range(1, n)])
    g = oracle.build_csr(n, src, dst)
    level, _, _ = oracle.bfs(g, 0)
    fs, fe = oracle.level_stats(g, level)
    assert fs.tolist() == [1, 10] and fe.tolist() == [10, 10]


def test_selector_paper_rule_on_table3():
    """P:L87 + alpha = 0.1: on the Tab III ratios the rule selects BU
    exactly at levels 3 and 4 — the levels where Tab VI's best is BU."""
    gold = json.load(open(os.path.join(GOLDEN, "paper_r25.json")))
    arcs = gold["rmat25_edges"]["value"]
    ratios = gold["tab3_ratios"]["value"]
    best = gold["tab6_best"]["value"]
    picks = [oracle.select(1, 1, int(round(r * arcs)), arcs, alpha=gold["alpha"]["value"]) for r in ratios]
    assert [p == 2 for p in picks] == [b == "BU" for b in best]
    # strict '>' (reading C-8): ratio exactly alpha stays top-down
    assert oracle.select(5, 1, 10, 100, alpha=0.1) != 2
    assert oracle.select(5, 1, 11, 100, alpha=0.1) == 2
    # growth rule (reading C-10): growing frontier -> SS, shrinking -> SF
    assert oracle.select(100, 10, 50, 100000, alpha=0.1, grow=2.0, ratio_min=1e-4) == 1
    assert oracle.select(10, 100, 50, 100000, alpha=0.1, grow=2.0, ratio_min=1e-4) == 0


def test_byte_replay_hand_computed():
    """SURVEY §8(d) D-3 by hand.  Path 0-1-2-3 from s=0 (N=4: N/8 -> bm = 1 byte,
    reading R-11), strategies SF, BU, SF, SF.  deg = [1,2,2,1]; F = {0},{1},{2},{3}.
      init      8N + 3N/8                                  = 32 + 3         = 35
      L0 SF     20|F0| + 4 edgesF0 + 28|F1|                = 20 + 4 + 28    = 52
      L1 BU     N/4 + 24|U1| + 4 probes + 8|F2|, U1 = {2,3}
                probes: v2's reordered row [1 (deg 2), 3 (deg 1)] -> 1
                        v3's row [2]: no level-1 neighbour -> deg 1  => 2
                                                           = 2 + 48 + 8 + 8 = 66
      L2 SF     20 + 4*2 + 28                                               = 56
      L3 SF     20 + 4*1 + 0                                                = 24
    SS at L2 adds the single scan N/8: 57; D-3 charges no queue rebuild after BU.
    """
    n, src, dst = _graph(4, [(0, 1), (1, 2), (2, 3)])
    g = oracle.reorder(oracle.build_csr(n, src, dst))
    level, _, nl = oracle.bfs(g, 0)
    assert nl == 4
    tot, per = oracle.byte_replay(g, level, [0, 2, 0, 0])
    assert per.tolist() == [52, 66, 56, 24]
    assert tot == 35 + 52 + 66 + 56 + 24
    _, per2 = oracle.byte_replay(g, level, [0, 2, 1, 0])
    assert per2.tolist() == [52, 66, 57, 24]


def test_byte_replay_hand_computed_star_rounding():
    """Star, centre 0 with leaves 1..19 (N = 20: bm = ceil(20/8) = 3 bytes), from
    s = 1, strategies SF, BU, SF.  F = {1}, {0}, {2..19}.
      init   8*20 + 3*3                                  = 169
      L0 SF  20*1 + 4*1 + 28*1                           = 52
      L1 BU  U1 = 18 leaves, each row [0] hits at once (18 probes), 18 found:
             2*3 + 24*18 + 4*18 + 8*18                   = 654
      L2 SF  20*18 + 4*18 + 0                            = 432
    All-BU instead: L0 BU: U0 = 19 (every vertex but the source), probes: v0's row
    [1, ...] hits at index 0 -> 1, 18 leaves scan their whole row [0] -> 18 => 19;
      2*3 + 24*19 + 4*19 + 8*1 = 546."""
    n, src, dst = _graph(20, [(0, i) for i in range(1, 20)])
    g = oracle.reorder(oracle.build_csr(n, src, dst))
    level, _, nl = oracle.bfs(g, 1)
    assert nl == 3
    tot, per = oracle.byte_replay(g, level, [0, 2, 0])
    assert per.tolist() == [52, 654, 432] and tot == 169 + 52 + 654 + 432
    _, per_bu = oracle.byte_replay(g, level, [2, 2, 2])
    assert per_bu[0] == 546


def test_select_hysteresis_and_sequence_hand_computed():
    """Reading C-11: after a BU step stay BU while |U_k| * bu_stay < edgesF_k;
    never from a top-down step.  Sequence replay by hand on the star of the
    previous test (A = 38 arcs) from s = 1, alpha = 0.1:
      k=0: |F|=1, edgesF=1  (ratio 0.026)  -> growth 1 > 2*0 and ratio > 1e-3: SS
      k=1: |F|=1, edgesF=19 (ratio 0.5)    -> BU
      k=2: |F|=18, edgesF=18 (ratio 0.47)  -> BU;  U = [19, 18, 0]."""
    assert oracle.select(10, 10, 50, 100000, alpha=0.1, bu_stay=1.0, prev=2, unvisited=49) == 2
    assert oracle.select(10, 10, 50, 100000, alpha=0.1, bu_stay=1.0, prev=2, unvisited=50) == 0
    assert oracle.select(10, 10, 50, 100000, alpha=0.1, bu_stay=1.0, prev=0, unvisited=1) == 0
    assert oracle.select(10, 10, 50, 100000, alpha=0.1, bu_stay=0.0, prev=2, unvisited=1) == 0
    n, src, dst = _graph(20, [(0, i) for i in range(1, 20)])
    g = oracle.build_csr(n, src, dst)
    level, _, _ = oracle.bfs(g, 1)
    st, un = oracle.select_sequence(g, level, alpha=0.1, grow=2.0, ratio_min=1e-3, bu_stay=1.0)
    assert st.tolist() == [1, 2, 2] and un.tolist() == [19, 18, 0]
    # path 0..9 from 0 (A = 18): edgesF_k = 1 at k = 0 and 9, 2 elsewhere; BU iff
    # edgesF_k / 18 > 0.1; level 0 grows (1 > 2*0) -> SS, level 9 does not -> SF
    n, src, dst = _graph(10, [(i, i + 1) for i in range(9)])
    g = oracle.build_csr(n, src, dst)
    level, _, _ = oracle.bfs(g, 0)
    st, un = oracle.select_sequence(g, level, alpha=0.1, grow=2.0, ratio_min=1e-3, bu_stay=0.0)
    assert st.tolist() == [1, 2, 2, 2, 2, 2, 2, 2, 2, 0]
    # every step equals the single-step rule on the exact per-level counters
    fs, fe = oracle.level_stats(g, level)
    prev = -1
    for k in range(len(st)):
        expect = oracle.select(int(fs[k]), int(fs[k - 1]) if k else 0, int(fe[k]), g.arcs, alpha=0.1, grow=2.0,
                               ratio_min=1e-3, bu_stay=0.0, prev=prev, unvisited=int(un[k]))
        assert st[k] == expect
        prev = expect
    assert un.tolist() == [9 - k for k in range(10)]


# ------------------------------------------------------- paper byte model pin

def test_paper_bandwidth_model_reproduces_13_7_percent():
    from paper_conf_sc_yangls0w24_b200 import metrics
    gold = json.load(open(os.path.join(GOLDEN, "paper_r25.json")))
    V, M = gold["rmat25_vertices"]["value"], gold["rmat25_edges"]["value"]
    b = metrics.model_bytes(V, M)
    assert b == 2_684_335_432
    # 43 GTEPS over |M| arcs gives the runtime; both efficiencies follow.
    t = M / (gold["gteps"]["value"] * 1e9)
    bw = gold["bandwidth_tbs"]["value"] * 1e12
    assert abs(metrics.bandwidth_efficiency(b, t, bw) - gold["predicted_efficiency"]["value"]) < 0.005
    hw = gold["hardware_bytes_gb"]["value"] * 1e9
    assert abs(metrics.bandwidth_efficiency(hw, t, bw) - gold["hardware_efficiency"]["value"]) < 0.005
    # Tab I "Sum" = levels 0..5 (reading C-21)
    kb = gold["tab1_fetch_kb_rearranged"]["value"]
    assert abs(sum(kb[:6]) - gold["tab1_sum_kb_rearranged"]["value"]) < 0.02
    # Tab III ratios sum to ~1: every arc of the root's component expanded once
    assert abs(sum(gold["tab3_ratios"]["value"]) - 0.999855) < 1e-5


def test_harmonic_mean_and_quartiles():
    from paper_conf_sc_yangls0w24_b200 import metrics
    assert metrics.harmonic_mean([1.0, 2.0, 4.0]) == pytest.approx(3 / (1 + 0.5 + 0.25))
    q = metrics.quartiles([1, 2, 3, 4, 5])
    assert (q["min"], q["q1"], q["median"], q["q3"], q["max"]) == (1, 2, 3, 4, 5)


def test_bu_probes_hand_computed():
    """Star centre 0 with leaves 1..4 plus path 4-5-6, from s = 1.
    levels: 1:0, 0:1, 2/3/4:2, 5:3, 6:4.  Reordered rows (deg desc, id asc):
      0: [1,2,3,4] (all deg 1 except 4 with deg 2) -> [4,1,2,3];  4: [0,5] (deg 4, 2);
      5: [4,6] (deg 2, 1); 6: [5].
    BU at k=1 (candidates: 2,3,4,5,6): v2 row [0] hit at 1; v3 same 1; v4 row [0,5]: 0 hit -> 1;
      v5 row [4,6]: no level-1 neighbour -> 2; v6 row [5] -> 1.  Total 6.
    BU at k=2 (candidates 5,6): v5 row [4,...]: 4 at level 2 -> 1; v6 row [5] -> 1.  Total 2."""
    n, src, dst = _graph(7, [(0, 1), (0, 2), (0, 3), (0, 4), (4, 5), (5, 6)])
    g = oracle.reorder(oracle.build_csr(n, src, dst))
    assert g.col[g.row_ptr[0]:g.row_ptr[1]].tolist() == [4, 1, 2, 3]
    level, _, _ = oracle.bfs(g, 1)
    assert level.tolist() == [1, 0, 2, 2, 2, 3, 4]
    assert oracle.bu_probes(g, level, 1) == 6
    assert oracle.bu_probes(g, level, 2) == 2
    # k=0 (F_0 = {1}): v0 row [4,1,2,3] hits 1 at index 1 -> 2; v2, v3 -> 1 each (deg);
    # v4 -> 2; v5 -> 2; v6 -> 1
    assert oracle.bu_probes(g, level, 0) == 2 + 1 + 1 + 2 + 2 + 1


# ------------------------------------------------- f4: directed graphs (R-9)

def test_directed_path_one_way():
    """0 -> 1 -> 2 -> 3: levels from 0 are 0..3; from 3 nothing else is reachable
    (the undirected build would reach all four)."""
    n, src, dst = _graph(4, [(0, 1), (1, 2), (2, 3)])
    g = oracle.build_csr_directed(n, src, dst)
    assert g.row_ptr.tolist() == [0, 1, 2, 3, 3] and g.col.tolist() == [1, 2, 3]
    lv, pa, nl = oracle.bfs(g, 0)
    assert lv.tolist() == [0, 1, 2, 3] and pa.tolist() == [0, 0, 1, 2] and nl == 4
    lv, pa, nl = oracle.bfs(g, 3)
    assert lv.tolist() == [-1, -1, -1, 0] and nl == 1
    assert oracle.validate_directed(g, src, dst, 3, lv, pa) == 0


def test_directed_cycle_closed_form():
    """Directed n-cycle i -> i+1 (mod n): level(v) = (v - s) mod n."""
    n = 37
    e = [(i, (i + 1) % n) for i in range(n)]
    n, src, dst = _graph(n, e)
    g = oracle.build_csr_directed(n, src, dst)
    for s in (0, 5, 36):
        lv, pa, nl = oracle.bfs(g, s)
        assert lv.tolist() == [(v - s) % n for v in range(n)] and nl == n
        assert oracle.validate_directed(g, src, dst, s, lv, pa) == 0


@pytest.mark.parametrize("seed", range(8))
def test_directed_bfs_matches_scipy(seed):
    rng = np.random.default_rng(500 + seed)
    n = int(rng.integers(2, 64))
    e = _random_graph(rng, n, int(rng.integers(0, 4 * n)))
    n, src, dst = _graph(n, e)
    g = oracle.build_csr_directed(n, src, dst)
    mask = src != dst
    A = sp.coo_matrix((np.ones(mask.sum()), (src[mask], dst[mask])), shape=(n, n)).tocsr()
    D = shortest_path(A, directed=True, unweighted=True)
    for s in range(n):
        level, parent, _ = oracle.bfs(g, s)
        expect = np.where(np.isinf(D[s]), -1, D[s]).astype(np.int64)
        assert np.array_equal(level, expect)
        assert oracle.validate_directed(g, src, dst, s, level, parent) == 0


@pytest.mark.parametrize("seed", range(4))
def test_directed_csr_matches_set_build(seed):
    rng = np.random.default_rng(600 + seed)
    n = int(rng.integers(1, 1 << 11))
    e = _random_graph(rng, n, int(rng.integers(0, 8 * n)))
    n, src, dst = _graph(n, e)
    g = oracle.build_csr_directed(n, src, dst)
    rows = [set() for _ in range(n)]
    for u, v in zip(src.tolist(), dst.tolist()):
        if u != v:
            rows[u].add(v)
    rp = np.concatenate([[0], np.cumsum([len(r) for r in rows])])
    col = np.array([c for r in rows for c in sorted(r)], dtype=np.int32)
    assert np.array_equal(g.row_ptr, rp)
    assert np.array_equal(g.col, col)


def test_directed_validator_rejects_mutations():
    rng = np.random.default_rng(21)
    n = 300
    n, src, dst = _graph(n, rng.integers(0, n, (1500, 2)))
    g = oracle.build_csr_directed(n, src, dst)
    s = int(src[0])
    level, parent, _ = oracle.bfs(g, s)
    assert oracle.validate_directed(g, src, dst, s, level, parent) == 0
    # a tree arc used backwards: v's parent replaced by a vertex one level up that v
    # only has an IN-arc from... pick u at level(v)-1 with arc v -> u but not u -> v
    out = lambda u: set(g.col[g.row_ptr[u]:g.row_ptr[u + 1]].tolist())
    done = False
    for v in np.flatnonzero(level >= 2):
        for u in np.flatnonzero(level == level[v] - 1):
            if u in out(v) and v not in out(u):
                p = parent.copy(); p[v] = int(u)
                assert oracle.validate_directed(g, src, dst, s, level, p) & oracle.V4_TREE_EDGE
                done = True
                break
        if done:
            break
    assert done
    # an arc i -> j skipping levels: pretend j is two levels deeper than allowed
    i = int(np.flatnonzero(level == 1)[0])
    j = next(iter(out(i)))
    lv = level.copy(); lv[j] = level[i] + 2
    assert oracle.validate_directed(g, src, dst, s, lv, parent) != 0
    # unreached head of a reached tail
    lv = level.copy(); p = parent.copy(); lv[j] = -1; p[j] = -1
    if j != s:
        assert oracle.validate_directed(g, src, dst, s, lv, p) & oracle.V5_EDGE_SPAN
    # an unreached vertex holds exactly level = parent = -1
    un = np.flatnonzero(level == -1)
    assert un.size
    for bad_l, bad_p in ((-1, -2), (-7, -7)):
        lv = level.copy(); p = parent.copy(); lv[un[0]] = bad_l; p[un[0]] = bad_p
        assert oracle.validate_directed(g, src, dst, s, lv, p) & oracle.V2_REACH
    # the undirected validator would reject a valid directed tree of a one-way path
    n2, s2, d2 = _graph(3, [(0, 1), (1, 2)])
    g2 = oracle.build_csr_directed(n2, s2, d2)
    lv2, pa2, _ = oracle.bfs(g2, 1)
    assert oracle.validate_directed(g2, s2, d2, 1, lv2, pa2) == 0
    assert oracle.validate(oracle.build_csr(n2, s2, d2), s2, d2, 1, lv2, pa2) & oracle.V5_EDGE_SPAN


# ------------------------------------- O-5 over the tuple list (s27 validator)

def _mutations(g, src, dst, s, level, parent):
    """(level, parent) variants: the valid tree plus one mutation per V-check."""
    out = [(level, parent)]
    reached = np.flatnonzero(level >= 2)
    v = int(reached[0])
    p = parent.copy(); p[s] = int(reached[1]); out.append((level, p))
    same = [u for u in np.flatnonzero(level == level[v] - 1)
            if not np.isin(v, g.col[g.row_ptr[u]:g.row_ptr[u + 1]])]
    p = parent.copy(); p[v] = int(same[0]); out.append((level, p))
    u = int(parent[v]); p = parent.copy(); p[u] = v; out.append((level, p))
    lv = level.copy(); lv[v] = -1; out.append((lv, parent))
    lv = level.copy(); lv[level >= 2] += 1; out.append((lv, parent))
    un = np.flatnonzero(level == -1)
    lv = level.copy(); p = parent.copy(); lv[un[0]] = 1; p[un[0]] = s; out.append((lv, p))
    lv = level.copy(); p = parent.copy(); p[un[0]] = -2; out.append((lv, p))
    lv = level.copy(); p = parent.copy(); lv[un[0]] = -7; p[un[0]] = -7; out.append((lv, p))
    lv = level.copy(); lv[s] = 1; out.append((lv, parent))
    return out


def test_validate_tuples_agrees_with_csr_validator():
    """The OpenMP tuple-list validator (oracle_validate_tuples) is pinned to the
    CSR validator: same bitmask on the valid tree and on every mutation, and zero
    exactly when the CSR validator says valid; 1 and 4 threads agree."""
    g, src, dst, s, level, parent = _valid_case()
    for lv, pa in _mutations(g, src, dst, s, level, parent):
        want = oracle.validate(g, src, dst, s, lv, pa)
        for t in (1, 4):
            got = oracle.validate_tuples(g.n, src, dst, s, lv, pa, threads=t)
            assert got == want, (got, want)


@pytest.mark.parametrize("seed", range(6))
def test_validate_tuples_random_graphs(seed):
    rng = np.random.default_rng(900 + seed)
    n = int(rng.integers(2, 300))
    e = rng.integers(0, n, (int(rng.integers(1, 4 * n)), 2))
    n, src, dst = _graph(n, e)
    g = oracle.build_csr(n, src, dst)
    gd = oracle.build_csr_directed(n, src, dst)
    for s in rng.integers(0, n, 4):
        lv, pa, _ = oracle.bfs(g, int(s))
        assert oracle.validate_tuples(n, src, dst, int(s), lv, pa) == 0
        lvd, pad, _ = oracle.bfs(gd, int(s))
        assert oracle.validate_tuples(n, src, dst, int(s), lvd, pad, directed=True) == 0
        # the undirected tree is not a valid directed one unless the arcs allow it, and vice versa
        assert (oracle.validate_tuples(n, src, dst, int(s), lvd, pad) == 0) == \
            (oracle.validate(g, src, dst, int(s), lvd, pad) == 0)
        assert (oracle.validate_tuples(n, src, dst, int(s), lv, pa, directed=True) == 0) == \
            (oracle.validate_directed(gd, src, dst, int(s), lv, pa) == 0)


# ------------------------------------------ R-12: deterministic first parents

def test_first_parents_hand_computed():
    """Reading R-12: parent[v] = the first vertex of v's RE-ARRANGED row one level up.
    Diamond 0-1, 0-2, 1-3, 2-3 plus 2-4 from s = 0: levels 0,1,1,2,2; deg(2) = 3 >
    deg(1) = 2, so row 3 is [2, 1] and parent[3] = 2 (id order would give 1).
    Without 2-4 the degrees tie and the id-ascending tie-break gives 1."""
    n, src, dst = _graph(5, [(0, 1), (0, 2), (1, 3), (2, 3), (2, 4)])
    g = oracle.reorder(oracle.build_csr(n, src, dst))
    level, _, _ = oracle.bfs(g, 0)
    par, orphans = oracle.first_parents(g, level, 0)
    assert par.tolist() == [0, 0, 0, 2, 2] and orphans == 0
    n, src, dst = _graph(5, [(0, 1), (0, 2), (1, 3), (2, 3)])
    g = oracle.reorder(oracle.build_csr(n, src, dst))
    level, _, _ = oracle.bfs(g, 0)
    par, _ = oracle.first_parents(g, level, 0)
    assert par.tolist() == [0, 0, 0, 1, -1]
    # path from 0: parent[v] = v - 1 (closed form)
    n, src, dst = _graph(9, [(i, i + 1) for i in range(8)])
    g = oracle.reorder(oracle.build_csr(n, src, dst))
    level, _, _ = oracle.bfs(g, 0)
    assert oracle.first_parents(g, level, 0)[0].tolist() == [0] + list(range(8))
    # directed (R-9): in-arc row of 3 = {1, 2} ordered by OUT-degree (2 has 2, 1 has 1)
    n, src, dst = _graph(5, [(0, 1), (0, 2), (1, 3), (2, 3), (2, 4)])
    gd = oracle.build_csr_directed(n, src, dst)
    tin = oracle.reorder(oracle.transpose_directed(n, src, dst), deg_from=gd)
    assert tin.col[tin.row_ptr[3]:tin.row_ptr[4]].tolist() == [2, 1]
    lv, _, _ = oracle.bfs(gd, 0)
    assert oracle.first_parents(tin, lv, 0)[0].tolist() == [0, 0, 0, 2, 2]


@pytest.mark.parametrize("seed", range(4))
def test_first_parents_are_valid_bfs_parents(seed):
    """On random graphs the R-12 parents pass Graph500 validation (V1-V5) and no
    reached vertex is left without a parent; directed likewise over in-arc rows."""
    rng = np.random.default_rng(1300 + seed)
    n = int(rng.integers(2, 400))
    e = rng.integers(0, n, (int(rng.integers(1, 5 * n)), 2))
    n, src, dst = _graph(n, e)
    g = oracle.build_csr(n, src, dst)
    r = oracle.reorder(g)
    gd = oracle.build_csr_directed(n, src, dst)
    tin = oracle.reorder(oracle.transpose_directed(n, src, dst), deg_from=gd)
    for s in rng.integers(0, n, 5):
        lv, _, _ = oracle.bfs(g, int(s))
        par, orphans = oracle.first_parents(r, lv, int(s))
        assert orphans == 0 and oracle.validate(g, src, dst, int(s), lv, par) == 0
        lvd, _, _ = oracle.bfs(gd, int(s))
        pard, orphans = oracle.first_parents(tin, lvd, int(s))
        assert orphans == 0 and oracle.validate_directed(gd, src, dst, int(s), lvd, pard) == 0
