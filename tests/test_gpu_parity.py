"""GPU parity: the CUDA path (through the C ABI) against the oracle.

Levels are unique (hop distances) and must match the oracle BIT-EXACTLY.
Parents are not unique in general (C-14); the library makes them
deterministic (reading R-12: the first vertex of the re-arranged row one level
up), so they must equal the oracle's oracle_first_parents BIT-EXACTLY and also
pass Graph500 validation V1-V5 against the input tuples.
Every strategy is forced on every level (SF-only, SS-only, BU-only) besides the
adaptive selector, so each kernel is checked on its own."""
import numpy as np
import pytest

import oracle
from paper_conf_sc_yangls0w24_b200 import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

MODES = [dict(), dict(force_strategy=0), dict(force_strategy=1), dict(force_strategy=2),
         dict(alpha=0.02), dict(alpha=0.3, grow=1.0, ratio_min=0.0), dict(bu_stay=4.0),
         dict(driver=1), dict(driver=1, force_strategy=1), dict(driver=1, force_strategy=2),
         dict(driver=2), dict(driver=2, force_strategy=1), dict(driver=2, force_strategy=2),
         dict(driver=3, force_strategy=0)]


@pytest.fixture(scope="module")
def xb():
    from paper_conf_sc_yangls0w24_b200 import xbfs
    return xbfs


def _dev(a):
    return torch.from_numpy(np.ascontiguousarray(a).view(np.int32)).cuda()


_ROWS = {}


def parent_rows(og, reordered=True):
    """The rows R-12 parents are searched in: the oracle's re-arranged CSR (cached)."""
    if not reordered:
        return og
    key = id(og)
    if key not in _ROWS or _ROWS[key][0] is not og:
        _ROWS[key] = (og, oracle.reorder(og))
    return _ROWS[key][1]


def check_parents(og, src, dst, root, lv, pa, reordered=True, strategy=None):
    """Parents: Graph500 V1-V5 everywhere, and R-12 exact (the first vertex of the
    re-arranged row one level up) at every vertex a bottom-up step found
    (strategy[level-1] == BU; top-down steps keep the vertex that discovered it)."""
    assert oracle.validate(og, src, dst, int(root), lv, pa) == 0, f"validation failed (root {root})"
    want, orphans = oracle.first_parents(parent_rows(og, reordered), lv, int(root))
    assert orphans == 0
    exact = lv <= 1
    if strategy is not None:
        st = np.asarray(list(strategy) + [-1], dtype=np.int64)
        idx = np.clip(lv - 1, 0, len(st) - 1)
        exact |= (lv >= 2) & (lv - 1 < len(strategy)) & (st[idx] == 2)
    bad = np.flatnonzero(exact & (want != pa))
    assert bad.size == 0, f"parents differ from R-12 at {bad[:5]} (root {root}): {pa[bad[:5]]} vs {want[bad[:5]]}"


def _check_run(g, og, src, dst, root, **opts):
    level, parent, st = g.run(int(root), stats=True, **opts)
    lv, pa = level.cpu().numpy(), parent.cpu().numpy()
    ref, _, nl = oracle.bfs(og, int(root))
    assert np.array_equal(lv, ref), f"levels differ (root {root}, opts {opts})"
    # (look-ahead vertices keep the F_{k+1} neighbour the pass saw: validated, not R-12)
    check_parents(og, src, dst, root, lv, pa, g.reordered, None if opts.get("lookahead") else st.strategy)
    # counters against the oracle's per-level facts
    fs, fe = oracle.level_stats(og, ref)
    assert st.num_levels == nl
    cap = len(st.frontier_vertices)          # per-level log: the first min(nl, capacity) levels
    assert cap == min(nl, 1 << 14)
    assert st.frontier_vertices == fs.tolist()[:cap]
    assert st.frontier_edges == fe.tolist()[:cap]
    assert st.vertices_reached == int((ref >= 0).sum())
    assert st.arcs_traversed == int(fe.sum())
    assert st.input_edges_traversed == oracle.input_edges(src, ref)
    if "force_strategy" in opts:
        assert set(st.strategy) == {opts["force_strategy"]}
    return st


@pytest.mark.parametrize("scale", [10, 14])
def test_csr_build_and_reorder_bit_exact(xb, scale):
    src, dst, n = synth.kronecker(scale, seed=1)
    og = oracle.build_csr(n, src, dst)
    g = xb.Graph(_dev(src), _dev(dst), n, reorder=False)
    rp, col = g.csr()
    assert np.array_equal(rp, og.row_ptr) and np.array_equal(col, og.col)
    assert g.arcs == og.arcs and g.max_degree == og.degree().max() and g.m_input == src.shape[0]
    g.reorder(1)
    rp2, col2 = g.csr()
    ro = oracle.reorder(og)
    assert np.array_equal(rp2, og.row_ptr) and np.array_equal(col2, ro.col)
    g.reorder(1)                                  # idempotent
    assert np.array_equal(g.csr()[1], ro.col)
    g.reorder(0)                                  # back to id order
    assert np.array_equal(g.csr()[1], og.col)
    g.close()


def test_csr_build_host_int64_edges(xb):
    src, dst, n = synth.kronecker(11, seed=4)
    og = oracle.build_csr(n, src, dst)
    g = xb.Graph(src.astype(np.int64), dst.astype(np.int64), n, reorder=False)
    rp, col = g.csr()
    assert np.array_equal(rp, og.row_ptr) and np.array_equal(col, og.col)
    g.close()


@pytest.mark.parametrize("opts", MODES)
def test_kronecker_s10_all_roots_all_strategies(xb, opts):
    src, dst, n = synth.kronecker(10, seed=1)
    og = oracle.build_csr(n, src, dst)
    g = xb.Graph(_dev(src), _dev(dst), n)
    for root in synth.roots(n, src, dst, 16, root_seed=2):
        _check_run(g, og, src, dst, root, **opts)
    g.close()


@pytest.mark.parametrize("opts", MODES[:4])
def test_kronecker_s16_strategies(xb, opts):
    src, dst, n = synth.kronecker(16, seed=3)
    og = oracle.build_csr(n, src, dst)
    g = xb.Graph(_dev(src), _dev(dst), n)
    for root in synth.roots(n, src, dst, 6, root_seed=5):
        _check_run(g, og, src, dst, root, **opts)
    g.close()


def test_kronecker_s20_adaptive(xb):
    src, dst, n = synth.kronecker(20, seed=1)
    og = oracle.build_csr(n, src, dst)
    g = xb.Graph(_dev(src), _dev(dst), n)
    for root in synth.roots(n, src, dst, 8, root_seed=2):
        st = _check_run(g, og, src, dst, root)
        assert 2 in st.strategy     # a BU level happens on Kronecker s20 with the default alpha (0.04)
    for root in synth.roots(n, src, dst, 2, root_seed=9):
        for f in (0, 1, 2):
            _check_run(g, og, src, dst, root, force_strategy=f)
    g.close()


@pytest.mark.parametrize("perm", [0, 10])
def test_grid_levels(xb, perm):
    W = H = 32 if perm else 48
    src, dst, n = synth.grid(W, H, seed=3, perm_scale=perm)
    og = oracle.build_csr(n, src, dst)
    g = xb.Graph(_dev(src), _dev(dst), n)
    for root in (0, n // 2 + W // 2, n - 1, 17):
        for opts in MODES[:4]:
            _check_run(g, og, src, dst, root, **opts)
    g.close()


def test_edge_cases(xb):
    # N not a multiple of 32; isolated vertices; 2-vertex component; self loops; duplicates
    n = 77
    e = [(i, i + 1) for i in range(30)] + [(40, 41)] + [(50, 50), (3, 4), (4, 3), (3, 4)] + \
        [(60, j) for j in range(61, 77)]
    src = np.array([a for a, _ in e], np.uint32)
    dst = np.array([b for _, b in e], np.uint32)
    og = oracle.build_csr(n, src, dst)
    g = xb.Graph(_dev(src), _dev(dst), n)
    for root in (0, 29, 40, 50, 33, 60, 76):      # 50: self-loop only (isolated); 33: isolated
        for opts in MODES:
            _check_run(g, og, src, dst, root, **opts)
    g.close()


def test_empty_and_tiny_graphs(xb):
    for n, e in [(1, []), (5, []), (2, [(0, 1)]), (33, [(0, 32)])]:
        src = np.array([a for a, _ in e], np.uint32)
        dst = np.array([b for _, b in e], np.uint32)
        og = oracle.build_csr(n, src, dst)
        g = xb.Graph(_dev(src) if len(e) else src, _dev(dst) if len(e) else dst, n)
        for root in range(n):
            for opts in MODES[:4]:
                _check_run(g, og, src, dst, root, **opts)
        g.close()


def test_hub_root_and_random_graphs(xb):
    rng = np.random.default_rng(0)
    n = 5000
    hub = np.stack([np.zeros(4000, np.int64), rng.integers(1, n, 4000)], 1)
    rnd = rng.integers(0, n, (20000, 2))
    e = np.concatenate([hub, rnd]).astype(np.uint32)
    src, dst = e[:, 0].copy(), e[:, 1].copy()
    og = oracle.build_csr(n, src, dst)
    g = xb.Graph(_dev(src), _dev(dst), n)
    for root in (0, 1, 4999):
        for opts in MODES:
            _check_run(g, og, src, dst, root, **opts)
    g.close()


def test_run_host_matches_device(xb):
    src, dst, n = synth.kronecker(12, seed=2)
    og = oracle.build_csr(n, src, dst)
    g = xb.Graph(_dev(src), _dev(dst), n)
    root = int(synth.roots(n, src, dst, 1)[0])
    lh = np.empty(n, np.int32)
    ph = np.empty(n, np.int32)
    st = g.run_host(root, lh, ph, stats=True)
    ref, _, nl = oracle.bfs(og, root)
    assert np.array_equal(lh, ref)
    check_parents(og, src, dst, root, lh, ph, True, st.strategy)
    assert st.num_levels == nl
    g.close()


@pytest.mark.parametrize("slots", [None, 2, 1])
def test_run_host_batch_matches_oracle(xb, slots):
    """Pipelined multi-root host call: every root's (last, when slots wrap) result equals
    the oracle's levels and validates; slot reuse across the two device buffers is exercised
    with 5 roots."""
    src, dst, n = synth.kronecker(12, seed=3)
    og = oracle.build_csr(n, src, dst)
    g = xb.Graph(_dev(src), _dev(dst), n)
    roots = [int(r) for r in synth.roots(n, src, dst, 5)]
    k = len(roots)
    ns = k if slots is None else slots
    lh = np.full(ns * n, -7, np.int32)
    ph = np.full(ns * n, -7, np.int32)
    g.run_host_batch(roots, lh, ph, host_slots=slots)
    for s in range(ns):
        i = max(j for j in range(k) if j % ns == s)      # the last root written to slot s
        ref, _, _ = oracle.bfs(og, roots[i])
        lv, pa = lh[s * n:(s + 1) * n], ph[s * n:(s + 1) * n]
        assert np.array_equal(lv, ref), (slots, s)
        check_parents(og, src, dst, roots[i], lv, pa)
    with pytest.raises(xb.XbfsError) as ei:
        g.run_host_batch([roots[0], n], lh, ph, host_slots=1)
    assert ei.value.status == xb.XBFS_ERR_INVALID_ARG
    g.run_host_batch([], lh, ph)                          # empty batch: a no-op
    g.close()


def test_errors(xb):
    src, dst, n = synth.kronecker(8, seed=1)
    g = xb.Graph(_dev(src), _dev(dst), n)
    lv = torch.empty(n, dtype=torch.int32, device="cuda")
    with pytest.raises(xb.XbfsError) as ei:
        xb.xbfs_run(g.handle, n, lv, lv)
    assert ei.value.status == xb.XBFS_ERR_INVALID_ARG
    with pytest.raises(xb.XbfsError):
        xb.xbfs_run(g.handle, -1, lv, lv)
    bad = np.array([0, n], np.uint32)
    with pytest.raises(xb.XbfsError) as ei:
        xb.Graph(bad, bad, n)
    assert ei.value.status == xb.XBFS_ERR_INVALID_ARG
    # the handle still works after rejected arguments
    level, parent, _ = g.run(int(src[0]))
    g.close()


@pytest.mark.parametrize("scale", [12, 16])
def test_bu_probes_and_parents_match_definition(xb, scale):
    """Bottom-up with early termination over degree-ordered rows
    (P:L153): the GPU's per-level probe count equals the oracle's definition,
    and a BU parent is exactly the first stored neighbour one level up."""
    src, dst, n = synth.kronecker(scale, seed=7)
    og = oracle.build_csr(n, src, dst)
    ro = oracle.reorder(og)
    g = xb.Graph(_dev(src), _dev(dst), n)
    for root in synth.roots(n, src, dst, 3, root_seed=11):
        for opts in (dict(force_strategy=2), dict(), dict(alpha=0.01)):
            level, parent, st = g.run(int(root), stats=True, **opts)
            ref, _, nl = oracle.bfs(og, int(root))
            lv, pa = level.cpu().numpy(), parent.cpu().numpy()
            assert np.array_equal(lv, ref)
            for k in range(nl):
                if st.strategy[k] == 2:
                    assert st.bu_probes[k] == oracle.bu_probes(ro, ref, k), (k, opts)
                    for v in np.flatnonzero(ref == k + 1)[:3000]:
                        row = ro.col[ro.row_ptr[v]:ro.row_ptr[v + 1]]
                        assert pa[v] == row[np.argmax(ref[row] == k)]
    g.close()


@pytest.mark.parametrize("small", [0, 200, 65536])
def test_small_frontier_cluster_mode(xb, small):
    """Small-frontier cluster mode (f3) hands levels back and forth with the
    level kernels; levels stay bit-exact and stats consistent for any threshold."""
    for graph in ("grid", "kron"):
        if graph == "grid":
            src, dst, n = synth.grid(64, 48, seed=5)
        else:
            src, dst, n = synth.kronecker(14, seed=21)
        og = oracle.build_csr(n, src, dst)
        g = xb.Graph(_dev(src), _dev(dst), n)
        roots = [0, n - 1, n // 2] if graph == "grid" else synth.roots(n, src, dst, 5, root_seed=3)
        for root in roots:
            for opts in (dict(small_edges=small), dict(small_edges=small, driver=1),
                         dict(small_edges=small, driver=2),
                         dict(small_edges=small, force_strategy=0), dict(small_edges=small, bu_stay=0.0)):
                _check_run(g, og, src, dst, root, **opts)
        g.close()


def test_per_level_strategy_plan(xb):
    """A per-level plan (forced-strategy studies) is followed level by level,
    including random mixes of SF/SS/BU; levels stay exact."""
    src, dst, n = synth.kronecker(14, seed=8)
    og = oracle.build_csr(n, src, dst)
    g = xb.Graph(_dev(src), _dev(dst), n)
    rng = np.random.default_rng(1)
    for root in synth.roots(n, src, dst, 4, root_seed=13):
        for _ in range(4):
            plan = rng.integers(0, 3, 12).tolist()
            st = _check_run(g, og, src, dst, root, plan=plan)
            assert st.strategy == plan[:st.num_levels]
        st = _check_run(g, og, src, dst, root, plan=[-1, 2, -1])
        assert st.strategy[1] == 2
    g.close()


def test_persistent_driver_level_times(xb):
    """The persistent driver (one cooperative launch per BFS) logs a %globaltimer
    stamp per level: the per-level times are positive and sum to at most the
    event-timed BFS; the other drivers report zeros."""
    src, dst, n = synth.kronecker(16, seed=4)
    og = oracle.build_csr(n, src, dst)
    g = xb.Graph(_dev(src), _dev(dst), n)
    for root in synth.roots(n, src, dst, 3, root_seed=5):
        st = _check_run(g, og, src, dst, root, driver=3)
        assert st.kernel_launches == 1
        assert all(t > 0 for t in st.level_ms)
        assert sum(st.level_ms) <= st.elapsed_ms * 1.01
        st = _check_run(g, og, src, dst, root, driver=1)
        assert st.kernel_launches > 1 and all(t == 0 for t in st.level_ms)
    g.close()


def test_deep_path_beyond_the_level_log(xb):
    """A path of 65,600 levels, deeper than the device's per-level log (kLogCap =
    65,536 entries) and than any 16-bit level encoding: levels and parents stay
    exact past the log's end, for the persistent (adaptive, forced BU / SS) and
    host-loop drivers and a source in the middle."""
    n = 65_600
    src = np.arange(n - 1, dtype=np.uint32)
    dst = src + 1
    og = oracle.build_csr(n, src, dst)
    g = xb.Graph(_dev(src), _dev(dst), n)
    for root, opts in ((0, dict()), (0, dict(force_strategy=2)), (n - 1, dict(force_strategy=1)),
                       (0, dict(driver=1, small_edges=0)), (n // 2, dict())):
        st = _check_run(g, og, src, dst, root, **opts)
        assert st.num_levels == max(root, n - 1 - root) + 1
    g.close()


def test_unaligned_output_arrays(xb):
    """The init fill writes 32-byte groups only when both outputs are 32-byte
    aligned (else 16-byte groups, else scalars); offset views of odd length
    still get every element right."""
    src, dst, n = synth.kronecker(11, seed=9)
    n += 3                                   # N not a multiple of 4; 3 isolated vertices
    og = oracle.build_csr(n, src, dst)
    g = xb.Graph(_dev(src), _dev(dst), n)
    lbuf = torch.full((n + 1,), 7, dtype=torch.int32, device="cuda")
    pbuf = torch.full((n + 1,), 7, dtype=torch.int32, device="cuda")
    for root in synth.roots(n - 3, src, dst, 3, root_seed=1):
        for opts in (dict(), dict(driver=1), dict(force_strategy=2)):
            level, parent, st = g.run(int(root), lbuf[1:], pbuf[1:], stats=True, **opts)
            lv, pa = level.cpu().numpy(), parent.cpu().numpy()
            ref, _, _ = oracle.bfs(og, int(root))
            assert np.array_equal(lv, ref)
            check_parents(og, src, dst, root, lv, pa, True, st.strategy)
            assert int(lbuf[0]) == 7 and int(pbuf[0]) == 7
    g.close()


@pytest.mark.parametrize("graph", ["kron", "grid", "hub"])
def test_bu_lookahead(xb, graph):
    """BU look-ahead: a BU step also settles level k+2
    vertices whose whole row misses F_k but hits a vertex this pass already put
    into F_{k+1}.  Levels stay bit-exact, parents valid, per-level frontier sizes
    exact (the look-ahead vertices are merged into F_{k+2} before step k+1, for
    a BU, SS or SF step k+1 alike), and the look-ahead does fire."""
    if graph == "kron":
        src, dst, n = synth.kronecker(15, seed=6)
        roots = synth.roots(n, src, dst, 4, root_seed=9)
    elif graph == "grid":
        src, dst, n = synth.grid(40, 30, seed=2)
        roots = [0, n // 2, n - 1]
    else:
        rng = np.random.default_rng(3)
        n = 6000
        e = np.concatenate([np.stack([np.zeros(3000, np.int64), rng.integers(1, n, 3000)], 1),
                            rng.integers(0, n, (15000, 2))]).astype(np.uint32)
        src, dst = e[:, 0].copy(), e[:, 1].copy()
        roots = [0, 1, 5999]
    og = oracle.build_csr(n, src, dst)
    g = xb.Graph(_dev(src), _dev(dst), n)
    fired = 0
    for root in roots:
        for opts in (dict(lookahead=1), dict(lookahead=1, force_strategy=2), dict(lookahead=1, alpha=0.005),
                     dict(lookahead=1, alpha=0.3, bu_stay=0.0), dict(lookahead=1, driver=3, bu_stay=8.0)):
            st = _check_run(g, og, src, dst, root, **opts)
            assert all(x == 0 for k, x in enumerate(st.lookahead_found) if st.strategy[k] != 2)
            fired += sum(st.lookahead_found)
    assert fired > 0
    # without the option nothing is set ahead
    st = _check_run(g, og, src, dst, roots[0], force_strategy=2)
    assert sum(st.lookahead_found) == 0
    with pytest.raises(xb.XbfsError):
        g.run(int(roots[0]), lookahead=1, driver=1)
    g.close()


@pytest.mark.parametrize("cfg", ["s24", "grid"])
def test_bench_workload_full_size(xb, cfg):
    """The exact graphs and roots bench.py times (BASELINE configs 3 and 5 at full
    size: Kronecker s24 ef16 seed 1, 16.8 M vertices / 521 M arcs; the 4096^2
    grid), in bench's launch configuration (persistent driver, default options):
    levels bit-exact against the oracle's serial BFS of the whole graph, parents
    Graph500-valid, per-level counters exact."""
    import bench
    src, dst, n = bench.make_graph(cfg, pinned=False)
    og = oracle.build_csr(n, src, dst)
    g = xb.Graph(_dev(src), _dev(dst), n)
    roots = bench.pick_roots(cfg, n, src, dst, 4 if cfg == "s24" else 2)
    for root in roots:
        st = _check_run(g, og, src, dst, root)
        assert st.kernel_launches == 1          # one cooperative launch per BFS
    g.close()


@pytest.mark.parametrize("scale", [16, 20])
def test_selector_decisions_match_the_rule(xb, scale):
    """The device selector (every CTA of the persistent kernel steps a replica of it)
    against oracle_select_sequence: the paper's rule (strict '>' C-8) with
    the growth rule C-10 and the stay-in-BU hysteresis C-11, replayed on the
    oracle's exact per-level counters.  The strategy of every level and U_k (the
    BU candidates before step k) must be identical, for the default options and
    for other (alpha, grow, ratio_min, bu_stay) settings."""
    src, dst, n = synth.kronecker(scale, seed=1)
    og = oracle.build_csr(n, src, dst)
    g = xb.Graph(_dev(src), _dev(dst), n)
    d = xb.xbfs_run_opts_default()
    settings = [dict(alpha=d.alpha, grow=d.grow, ratio_min=d.ratio_min, bu_stay=d.bu_stay),
                dict(alpha=0.1, grow=2.0, ratio_min=1e-3, bu_stay=0.0),      # the paper's rule
                dict(alpha=0.01, grow=1.5, ratio_min=1e-4, bu_stay=4.0)]
    for root in synth.roots(n, src, dst, 6, root_seed=17):
        ref, _, nl = oracle.bfs(og, int(root))
        for opt in settings:
            for drv in (3, 1):
                _, _, st = g.run(int(root), stats=True, driver=drv, small_edges=0, **opt)
                want, unv = oracle.select_sequence(og, ref, **opt)
                assert st.num_levels == nl
                assert st.strategy == want.tolist(), (root, opt, drv)
                assert st.unvisited == unv.tolist(), (root, opt, drv)
    g.close()


def test_run_host_batch_pinned_overlap(xb):
    """xbfs_run_host_batch into PINNED host buffers (the copy of root i really
    overlaps the BFS of root i+1, so the two device slots' reuse ordering is
    exercised): 7 roots, every slot's levels exact and parents valid."""
    src, dst, n = synth.kronecker(14, seed=12)
    og = oracle.build_csr(n, src, dst)
    g = xb.Graph(_dev(src), _dev(dst), n)
    roots = [int(r) for r in synth.roots(n, src, dst, 7, root_seed=21)]
    k = len(roots)
    lh = torch.full((k * n,), -7, dtype=torch.int32, pin_memory=True).numpy()
    ph = torch.full((k * n,), -7, dtype=torch.int32, pin_memory=True).numpy()
    for _ in range(2):
        g.run_host_batch(roots, lh, ph)
        for i, r in enumerate(roots):
            ref, _, _ = oracle.bfs(og, r)
            lv, pa = lh[i * n:(i + 1) * n], ph[i * n:(i + 1) * n]
            assert np.array_equal(lv, ref), i
            assert oracle.validate(og, src, dst, r, lv, pa) == 0, i
        lh[:] = -7
        ph[:] = -7
    with pytest.raises(ValueError):
        g.run_host_batch(roots, lh[: n], ph[: n])          # too small for k slots: refused in the binding
    g.close()


def test_bench_workload_s27_full_size(xb):
    """BASELINE config 4's graph (Kronecker s27 ef16 seed 1: 134 M vertices, 2.1 G
    tuples, 4.2 G arcs) on one B200 in bench's launch configuration.  Every root
    checked passes the OpenMP tuple-list Graph500 validator (V1-V5 over all 2.1 G
    input tuples, which certifies the levels exactly: SURVEY §8(c) O-5), and the
    first root's levels equal the oracle's serial BFS over its own CSR bit-exactly."""
    import gc

    import bench
    src, dst, n = bench.make_graph("s27", pinned=False)
    roots = [int(r) for r in bench.pick_roots("s27", n, src, dst, 3)]
    g = xb.Graph(torch.from_numpy(src.view(np.int32)), torch.from_numpy(dst.view(np.int32)), n)
    results = []
    for root in roots:
        level, parent, st = g.run(root, stats=True)
        assert st.kernel_launches == 1
        lv, pa = level.cpu().numpy(), parent.cpu().numpy()
        del level, parent
        assert oracle.validate_tuples(n, src, dst, root, lv, pa) == 0, root
        assert st.vertices_reached == int((lv >= 0).sum())
        results.append((root, lv if not results else None, st))
    g.close()
    torch.cuda.empty_cache()
    gc.collect()
    root, lv0, st0 = results[0]
    og = oracle.build_csr(n, src, dst)
    ref, _, nl = oracle.bfs(og, root)
    assert np.array_equal(lv0, ref)
    assert st0.num_levels == nl
    assert st0.input_edges_traversed == oracle.input_edges(src, ref)
