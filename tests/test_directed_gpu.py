"""GPU parity for directed graphs (reading R-9): the CUDA path
through the C ABI against the oracle's out-arc CSR, textbook BFS and arc-wise
Graph500 validation.  Levels must match BIT-EXACTLY; parents must validate and
equal reading R-12's choice (the first in-neighbour of the re-arranged in-arc
row one level up, oracle_first_parents) BIT-EXACTLY;
the per-level counters (|F_k|, edgesF_k over OUT-degrees), vertices reached,
arcs traversed and Graph500 m must equal the oracle's.  Every strategy is
forced on every level besides the adaptive selector, so the in-arc bottom-up
search is checked on its own."""
import numpy as np
import pytest

import oracle
from paper_conf_sc_yangls0w24_b200 import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

MODES = [dict(), dict(force_strategy=0), dict(force_strategy=1), dict(force_strategy=2),
         dict(alpha=0.005), dict(alpha=0.3, grow=1.0, ratio_min=0.0), dict(bu_stay=0.0),
         dict(driver=3, force_strategy=2)]


@pytest.fixture(scope="module")
def xb():
    from paper_conf_sc_yangls0w24_b200 import xbfs
    return xbfs


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a).view(np.int32)).cuda()


_ROWS = {}


def in_rows(og, src, dst, reordered=True):
    """R-12 parent rows of a directed graph: the in-arc CSR, re-arranged by the
    in-neighbour's out-degree (R-9) when the library's graph is (cached)."""
    key = (id(og), reordered)
    if key not in _ROWS or _ROWS[key][0] is not og:
        t = oracle.transpose_directed(og.n, src, dst)
        _ROWS[key] = (og, oracle.reorder(t, deg_from=og) if reordered else t)
    return _ROWS[key][1]


def check_parents_directed(og, src, dst, root, lv, pa, reordered=True, strategy=None):
    """Parents: arc-wise V1-V5 everywhere; R-12 exact where a bottom-up step found the vertex."""
    assert oracle.validate_directed(og, src, dst, int(root), lv, pa) == 0, f"validation (root {root})"
    want, orphans = oracle.first_parents(in_rows(og, src, dst, reordered), lv, int(root))
    assert orphans == 0
    exact = lv <= 1
    if strategy is not None:
        st = np.asarray(list(strategy) + [-1], dtype=np.int64)
        idx = np.clip(lv - 1, 0, len(st) - 1)
        exact |= (lv >= 2) & (lv - 1 < len(strategy)) & (st[idx] == 2)
    bad = np.flatnonzero(exact & (want != pa))
    assert bad.size == 0, f"parents differ from R-12 at {bad[:5]} (root {root})"


def _check(g, og, src, dst, root, **opts):
    level, parent, st = g.run(int(root), stats=True, **opts)
    lv, pa = level.cpu().numpy(), parent.cpu().numpy()
    ref, _, nl = oracle.bfs(og, int(root))
    assert np.array_equal(lv, ref), f"levels differ (root {root}, {opts})"
    check_parents_directed(og, src, dst, root, lv, pa, g.reordered, st.strategy)
    fs, fe = oracle.level_stats(og, ref)
    assert st.num_levels == nl
    cap = len(st.frontier_vertices)
    assert st.frontier_vertices == fs.tolist()[:cap]
    assert st.frontier_edges == fe.tolist()[:cap]
    assert st.vertices_reached == int((ref >= 0).sum())
    assert st.arcs_traversed == int(fe.sum())
    assert st.input_edges_traversed == oracle.input_edges(src, ref)
    if "force_strategy" in opts and nl > 1:
        assert set(st.strategy) == {opts["force_strategy"]}
    return st


def _one_way_grid(w, h):
    """Arcs right and down only: from (r, c) the reachable set is the lower-right
    quadrant at Manhattan distance."""
    v = np.arange(w * h).reshape(h, w)
    right = np.stack([v[:, :-1].ravel(), v[:, 1:].ravel()], 1)
    down = np.stack([v[:-1, :].ravel(), v[1:, :].ravel()], 1)
    e = np.concatenate([right, down]).astype(np.uint32)
    return e[:, 0].copy(), e[:, 1].copy(), w * h


@pytest.mark.parametrize("scale", [10, 14])
def test_directed_csr_bit_exact(xb, scale):
    src, dst, n = synth.kronecker(scale, seed=4)
    og = oracle.build_csr_directed(n, src, dst)
    g = xb.Graph(_dev(src), _dev(dst), n, reorder=False, directed=True)
    rp, col = g.csr()
    assert g.arcs == og.arcs
    assert np.array_equal(rp, og.row_ptr) and np.array_equal(col[: og.arcs], og.col)
    g.reorder(1)
    r = oracle.reorder(og)
    rp, col = g.csr()
    assert np.array_equal(col[: og.arcs], r.col)
    g.close()


@pytest.mark.parametrize("scale", [12, 15])
def test_directed_kronecker(xb, scale):
    src, dst, n = synth.kronecker(scale, seed=5)
    og = oracle.build_csr_directed(n, src, dst)
    g = xb.Graph(_dev(src), _dev(dst), n, directed=True)
    roots = synth.roots(n, src, dst, 3)
    seen_bu = False
    for root in roots:
        for opts in MODES:
            st = _check(g, og, src, dst, root, **opts)
            seen_bu |= 2 in st.strategy
    assert seen_bu
    g.close()


def test_directed_random_with_sources_and_sinks(xb):
    """Sparse random arcs: many vertices have no in-arc (never BU candidates) or
    no out-arc; roots include a pure source and a pure sink."""
    rng = np.random.default_rng(9)
    n = 20000
    e = rng.integers(0, n, size=(3 * n, 2)).astype(np.uint32)
    src, dst = e[:, 0].copy(), e[:, 1].copy()
    og = oracle.build_csr_directed(n, src, dst)
    indeg = np.bincount(dst[src != dst], minlength=n)
    outdeg = og.degree()
    pure_src = int(np.flatnonzero((indeg == 0) & (outdeg > 0))[0])
    pure_sink = int(np.flatnonzero((indeg > 0) & (outdeg == 0))[0])
    g = xb.Graph(src, dst, n, directed=True)
    for root in (int(src[0]), pure_src, pure_sink):
        for opts in MODES:
            _check(g, og, src, dst, root, **opts)
    g.close()


def test_directed_one_way_grid_and_cycle(xb):
    src, dst, n = _one_way_grid(96, 80)
    og = oracle.build_csr_directed(n, src, dst)
    g = xb.Graph(src, dst, n, directed=True)
    for root in (0, 96 * 40 + 50):
        for opts in MODES:
            _check(g, og, src, dst, root, **opts)
    lv, _, _ = g.run(0)
    r, c = np.divmod(np.arange(n), 96)
    assert np.array_equal(lv.cpu().numpy(), r + c)       # closed form from the corner
    g.close()
    # directed cycle: N levels, one vertex each (deep-path driver case)
    n = 3000
    src = np.arange(n, dtype=np.uint32)
    dst = ((src + 1) % n).astype(np.uint32)
    og = oracle.build_csr_directed(n, src, dst)
    g = xb.Graph(src, dst, n, directed=True)
    for opts in (dict(), dict(force_strategy=2)):
        st = _check(g, og, src, dst, 17, **opts)
        assert st.num_levels == n
    g.close()


def test_directed_unsupported_modes(xb):
    src, dst, n = synth.kronecker(8, seed=1)
    g = xb.Graph(src, dst, n, directed=True)
    for opts in (dict(driver=1), dict(driver=2), dict(lookahead=1)):
        with pytest.raises(xb.XbfsError) as ei:
            g.run(int(src[0]), **opts)
        assert ei.value.status == xb.XBFS_ERR_UNSUPPORTED
    g.run(int(src[0]))                                     # the handle still works
    g.close()


def test_symmetric_input_directed_equals_undirected(xb):
    """Both arcs of every tuple given as a directed graph = the undirected graph."""
    src, dst, n = synth.kronecker(12, seed=6)
    s2 = np.concatenate([src, dst]); d2 = np.concatenate([dst, src])
    gd = xb.Graph(s2, d2, n, directed=True)
    gu = xb.Graph(src, dst, n)
    for root in synth.roots(n, src, dst, 3):
        ld, _, _ = gd.run(int(root))
        lu, _, _ = gu.run(int(root))
        assert torch.equal(ld, lu)
    gd.close(); gu.close()


def test_directed_kronecker_s20_saturated_head(xb):
    """Scale 20: head32 holds 20-bit ids, so in-degrees >= 4095 saturate and the
    bottom-up resolves them from in_row_ptr (the s24 bench case has dmax = 255)."""
    src, dst, n = synth.kronecker(20, seed=1)
    og = oracle.build_csr_directed(n, src, dst)
    g = xb.Graph(src, dst, n, directed=True)
    for root in synth.roots(n, src, dst, 2):
        for opts in (dict(), dict(force_strategy=2)):
            _check(g, og, src, dst, root, **opts)
    g.close()


def test_directed_sinks_fill_a_tile(xb):
    """Many out-degree-0 vertices discovered in one top-down level (a hub with
    20000 arcs into sinks plus a few real rows): the queue holds only vertices
    with arcs, so a 2048-arc tile never spans more entries than it has arcs."""
    hub, nsink = 0, 20000
    sinks = np.arange(1, nsink + 1)
    chain = np.arange(nsink + 1, nsink + 50)
    extra = sinks[::97]                       # a few of them do have out-arcs (into the chain)
    src = np.concatenate([np.full(nsink, hub), np.full(chain.size, hub), chain[:-1], extra])
    dst = np.concatenate([sinks, chain, chain[1:], nsink + 1 + np.arange(extra.size) % chain.size])
    n = nsink + 50
    src, dst = src.astype(np.uint32), dst.astype(np.uint32)
    og = oracle.build_csr_directed(n, src, dst)
    g = xb.Graph(src, dst, n, directed=True)
    for opts in MODES:
        _check(g, og, src, dst, hub, **opts)
    g.close()


def test_bench_workload_s24d_full_size(xb):
    """The directed bench workload at full size (bench.py --config s24d: the s24 Kronecker
    tuples as arcs, 16.8 M vertices / 263 M arcs), persistent driver, default options:
    levels bit-exact against the oracle's serial BFS, parents arc-validated, per-level
    counters exact, one launch per BFS; roots are bench's candidates, including ones
    whose forward reach is tiny (the bench screens those out; parity must hold anyway)."""
    import bench
    src, dst, n = bench.make_graph("s24d", pinned=False)
    og = oracle.build_csr_directed(n, src, dst)
    g = xb.Graph(_dev(src), _dev(dst), n, directed=True)
    for root in bench.pick_roots("s24d", n, src, dst, 3):
        st = _check(g, og, src, dst, root)
        assert st.kernel_launches == 1
    g.close()


def test_directed_int64_device_edges_and_host_batch(xb):
    """Directed build from int64 ids resident on the device (id_bytes 8,
    edges_on_device 1) equals the oracle; the pipelined host-output batch call
    returns every root's exact levels on it."""
    src, dst, n = synth.kronecker(13, seed=8)
    og = oracle.build_csr_directed(n, src, dst)
    s64 = torch.from_numpy(src.astype(np.int64)).cuda()
    d64 = torch.from_numpy(dst.astype(np.int64)).cuda()
    g = xb.Graph(s64, d64, n, reorder=False, directed=True)
    rp, col = g.csr()
    assert np.array_equal(rp, og.row_ptr) and np.array_equal(col[: og.arcs], og.col)
    g.reorder(1)
    roots = [int(r) for r in synth.roots(n, src, dst, 4, root_seed=5)]
    lh = np.empty(4 * n, np.int32)
    ph = np.empty(4 * n, np.int32)
    g.run_host_batch(roots, lh, ph)
    for i, r in enumerate(roots):
        ref, _, _ = oracle.bfs(og, r)
        assert np.array_equal(lh[i * n:(i + 1) * n], ref)
        check_parents_directed(og, src, dst, r, lh[i * n:(i + 1) * n], ph[i * n:(i + 1) * n])
    g.close()
