"""Harness arithmetic against the oracle: the bench's per-BFS algorithmic byte
count (metrics.bfs_level_bytes, the persistent kernel's roofline numerator)
equals the oracle's byte replay (O-8, itself pinned by hand in test_oracle.py)
for any strategy sequence."""
import numpy as np

import oracle
from paper_conf_sc_yangls0w24_b200 import metrics, synth


def test_bfs_level_bytes_equals_oracle_replay():
    src, dst, n = synth.kronecker(11, seed=3)
    g = oracle.reorder(oracle.build_csr(n, src, dst))
    rng = np.random.default_rng(0)
    nonisolated = int((np.diff(g.row_ptr) > 0).sum())
    for root in synth.roots(n, src, dst, 3, root_seed=4):
        level, _, nl = oracle.bfs(g, int(root))
        fs, fe = oracle.level_stats(g, level)
        for _ in range(6):
            strat = rng.integers(0, 3, nl).tolist()
            _, per = oracle.byte_replay(g, level, strat)
            unv, probes = [], []
            u = nonisolated - int(np.diff(g.row_ptr)[root] > 0)
            for k in range(nl):
                unv.append(u)
                probes.append(oracle.bu_probes(g, level, k) if strat[k] == 2 else 0)
                u -= int(fs[k + 1]) if k + 1 < nl else 0
            mine = metrics.bfs_level_bytes(n, strat, fs.tolist(), fe.tolist(), unv, probes)
            assert mine == per.tolist()
            assert metrics.bfs_alg_bytes(n, strat, fs.tolist(), fe.tolist(), unv, probes) == \
                oracle.byte_replay(g, level, strat)[0]


def test_directed_bu_level_adds_the_count_pass():
    """R-9: a directed BU step reads in-arc rows, so edgesF_{k+1} comes from the
    out-arc head[] word of every found vertex (8 B each, read where the vertex is
    published): added to the BU level, nothing else changes."""
    from paper_conf_sc_yangls0w24_b200 import metrics
    n = 1 << 12
    strat, fv, fe, un, pr = [0, 2, 2, 0], [1, 50, 900, 30], [50, 900, 4000, 60], [4000, 3950, 3000, 2100], \
        [0, 7000, 5000, 0]
    u = metrics.bfs_level_bytes(n, strat, fv, fe, un, pr)
    d = metrics.bfs_level_bytes(n, strat, fv, fe, un, pr, directed=True)
    assert d[0] == u[0] and d[3] == u[3]
    assert d[1] - u[1] == 8 * 900 and d[2] - u[2] == 8 * 30
