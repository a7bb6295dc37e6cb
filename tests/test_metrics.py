"""Harness arithmetic against the oracle: the bench's roofline numerator
(metrics.d3_level_bytes / d3_bytes) equals the oracle's byte
replay (O-8, itself pinned by hand in test_oracle.py) for any strategy
sequence, given the per-level counters the library logs."""
import numpy as np

import oracle
from paper_conf_sc_yangls0w24_b200 import metrics, synth


def test_d3_bytes_equal_oracle_replay():
    src, dst, n = synth.kronecker(11, seed=3)
    n = n + 5                                   # N not a multiple of 8 (R-11 rounding) + isolated tail
    g = oracle.reorder(oracle.build_csr(n, src, dst))
    rng = np.random.default_rng(0)
    nonisolated = int((np.diff(g.row_ptr) > 0).sum())
    for root in synth.roots(n - 5, src, dst, 3, root_seed=4):
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
            mine = metrics.d3_level_bytes(n, strat, fs.tolist(), fe.tolist(), unv, probes)
            assert mine == per.tolist()
            assert metrics.d3_bytes(n, strat, fs.tolist(), fe.tolist(), unv, probes) == \
                oracle.byte_replay(g, level, strat)[0]


def test_d3_terms_by_hand():
    """D-3 at N = 4096 (N/8 = 512): init 8N + 3N/8; an SF, an SS and a BU level."""
    n = 1 << 12
    strat, fv, fe, un, pr = [0, 1, 2], [1, 50, 900], [50, 900, 4000], [4000, 3950, 3000], [0, 0, 5000]
    assert metrics.d3_init(n) == 8 * 4096 + 3 * 512
    lv = metrics.d3_level_bytes(n, strat, fv, fe, un, pr)
    assert lv == [20 * 1 + 4 * 50 + 28 * 50, 20 * 50 + 4 * 900 + 28 * 900 + 512, 1024 + 24 * 3000 + 4 * 5000]
