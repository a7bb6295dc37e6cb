"""Generator checks (inputs module): closed-form counts, the Graph500 quadrant
law within 5 sigma, self-loop rate M*(A+D)^s, determinism, bijective relabel."""
import numpy as np
import pytest

from paper_conf_sc_yangls0w24_b200 import synth


def test_splitmix64_reference_values():
    # splitmix64 as published (Vigna): state 0 -> first output after one increment
    assert synth.splitmix64(0) == 0xE220A8397B1DCDAF
    assert synth.splitmix64(0x9E3779B97F4A7C15 * 0) == 0xE220A8397B1DCDAF


def test_kronecker_shape_and_determinism():
    s = 12
    a_src, a_dst, n = synth.kronecker(s, seed=5)
    b_src, b_dst, _ = synth.kronecker(s, seed=5)
    c_src, _, _ = synth.kronecker(s, seed=6)
    assert n == 1 << s and a_src.shape[0] == 16 * n
    assert a_src.max() < n and a_dst.max() < n
    assert np.array_equal(a_src, b_src) and np.array_equal(a_dst, b_dst)
    assert not np.array_equal(a_src, c_src)
    # sub-range generation is the same stream
    p_src, p_dst, _ = synth.kronecker(s, seed=5, e_begin=1000, e_end=3000)
    assert np.array_equal(p_src, a_src[1000:3000]) and np.array_equal(p_dst, a_dst[1000:3000])


def test_kronecker_quadrant_law():
    s = 10
    src, dst, n = synth.kronecker(s, seed=3, permute=False)
    M = src.shape[0]
    probs = {(0, 0): 0.57, (0, 1): 0.19, (1, 0): 0.19, (1, 1): 0.05}
    for b in range(s):
        i = (src >> b) & 1
        j = (dst >> b) & 1
        for (qi, qj), p in probs.items():
            c = int(np.sum((i == qi) & (j == qj)))
            sigma = np.sqrt(M * p * (1 - p))
            assert abs(c - M * p) < 5 * sigma, (b, qi, qj, c, M * p)


def test_kronecker_self_loop_rate():
    s = 14
    src, dst, n = synth.kronecker(s, seed=9)
    M = src.shape[0]
    loops = int(np.sum(src == dst))
    p = 0.62 ** s
    sigma = np.sqrt(M * p * (1 - p))
    assert abs(loops - M * p) < 5 * sigma


@pytest.mark.parametrize("s", [1, 5, 10, 16])
def test_perm_is_bijection(s):
    vals = {synth.perm(77, s, v) for v in range(1 << s)} if s <= 10 else None
    if vals is not None:
        assert vals == set(range(1 << s))
    else:
        src, dst, n = synth.kronecker(s, seed=77, permute=True)
        assert src.max() < n


def test_grid_counts():
    W, H = 13, 9
    src, dst, n = synth.grid(W, H)
    assert n == W * H and src.shape[0] == 2 * W * H - W - H
    pairs = set(zip(src.tolist(), dst.tolist()))
    assert (0, 1) in pairs and (0, W) in pairs and len(pairs) == src.shape[0]
    src2, dst2, _ = synth.grid(16, 16, perm_scale=8, seed=4)
    assert src2.shape[0] == 2 * 256 - 32 and max(src2.max(), dst2.max()) < 256
    src3, _, _ = synth.grid(64, 64, keep_prob=0.8, seed=4)
    assert 0.75 * (2 * 4096 - 128) < src3.shape[0] < 0.85 * (2 * 4096 - 128)


def test_roots_distinct_and_non_isolated():
    src = np.array([0, 1, 2, 5, 5], dtype=np.uint32)
    dst = np.array([1, 2, 0, 5, 6], dtype=np.uint32)
    r = synth.roots(10, src, dst, 100, root_seed=2)
    assert sorted(r.tolist()) == [0, 1, 2, 5, 6]
    r2 = synth.roots(10, src, dst, 3, root_seed=2)
    assert len(set(r2.tolist())) == 3 and set(r2.tolist()) <= {0, 1, 2, 5, 6}
