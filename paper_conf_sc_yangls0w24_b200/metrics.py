"""Harness arithmetic: TEPS conventions, Graph500 statistics, roofline bytes.

Pure Python; no BFS arithmetic.  Citations are PAPER.md lines ("P:L…").
"""
from __future__ import annotations

import math
from typing import Sequence


def model_bytes(n: int, arcs: int) -> int:
    """The paper's predicted memory read for one BFS: 8*2|V| + 4*|M| bytes
    (§V-F: every vertex's two 8-byte edge offsets + every arc's 4-byte
    id; reading C-24).  |M| = stored arcs (reading C-4)."""
    return 16 * n + 4 * arcs


def bandwidth_efficiency(nbytes: float, seconds: float, peak_bytes_per_s: float) -> float:
    """(bytes / runtime) / peak, the paper's efficiency."""
    return nbytes / seconds / peak_bytes_per_s


def teps(edges: int, seconds: float) -> float:
    return edges / seconds


def harmonic_mean(xs: Sequence[float]) -> float:
    """Graph500 reports the harmonic mean of per-root TEPS."""
    xs = list(xs)
    return len(xs) / sum(1.0 / x for x in xs)


def quartiles(xs: Sequence[float]):
    """min, Q1, median, Q3, max (Graph500 statistics; linear interpolation)."""
    s = sorted(xs)

    def q(p):
        if len(s) == 1:
            return s[0]
        pos = p * (len(s) - 1)
        lo = math.floor(pos)
        hi = min(lo + 1, len(s) - 1)
        return s[lo] + (s[hi] - s[lo]) * (pos - lo)

    return {"min": s[0], "q1": q(0.25), "median": q(0.5), "q3": q(0.75), "max": s[-1]}


# --------------------------------------------------------------------------
# the ALGORITHMIC bytes of one BFS given the strategies the
# selector took (the roofline numerator; replayed independently by the oracle's
# oracle_byte_replay, tests/test_metrics.py).  Bitmap probes are L2 traffic and
# are not counted.  N/8 is rounded up to whole bytes (reading R-11).
# --------------------------------------------------------------------------

def d3_bitmap(n: int) -> int:
    """N/8 bytes (one N-bit bitmap), rounded up."""
    return (n + 7) // 8


def d3_init(n: int) -> int:
    """level + parent (8N) + three N-bit bitmaps (3N/8)."""
    return 8 * n + 3 * d3_bitmap(n)


def d3_level_bytes(n: int, strategy, fv, fe, unvisited, probes):
    """Per level k: TD (SF/SS) 20|F_k| + 4 edgesF_k + 28|F_{k+1}| (+ N/8 for the
    single scan of SS); BU N/4 + 24|U_k| + 4 probes_k + 8|F_{k+1}|."""
    bm = d3_bitmap(n)
    out = []
    L = len(strategy)
    for k in range(L):
        found = fv[k + 1] if k + 1 < L else 0
        if strategy[k] == 2:
            out.append(2 * bm + 24 * unvisited[k] + 4 * probes[k] + 8 * found)
        else:
            out.append(20 * fv[k] + 4 * fe[k] + 28 * found + (bm if strategy[k] == 1 else 0))
    return out


def d3_bytes(n: int, strategy, fv, fe, unvisited, probes) -> int:
    """Init + every level: D-3 algorithmic bytes of one whole BFS."""
    return d3_init(n) + sum(d3_level_bytes(n, strategy, fv, fe, unvisited, probes))


# --------------------------------------------------------------------------
# KERNEL TRAFFIC MODEL (reported as the bench line's `kernel_model`, never as
# the roofline numerator): what this build's kernels move per launch
# (DESIGN.md §5).  B = 4*ceil(n/32) bytes is one pass over an n-bit bitmap.
# --------------------------------------------------------------------------

def bitmap_bytes(n: int) -> int:
    return 4 * ((n + 31) // 32)


def bytes_init(n: int) -> int:
    """level + parent fill (8n) + visited write, non-isolated read, 3 frontier maps."""
    return 8 * n + 5 * bitmap_bytes(n)


def bytes_td_sf(n: int, f_size: int, f_edges: int, found: int) -> int:
    """Scan-free expansion: stale-map clear + 20 B per queue entry (id + two int64)
    + 4 B per arc (col) + 44 B per discovered vertex (level, parent, row_ptr pair,
    next-queue entry)."""
    return bitmap_bytes(n) + 20 * f_size + 4 * f_edges + 44 * found


def bytes_td_ss(n: int, f_size: int, f_edges: int, found: int) -> int:
    """Single-scan expansion: as SF but only level + parent per discovered vertex."""
    return bitmap_bytes(n) + 20 * f_size + 4 * f_edges + 8 * found


def bytes_generate(n: int, count: int, post: bool) -> int:
    """Bitmap -> queue: bitmap read (+ visited OR when post) + 36 B per vertex
    (row_ptr pair + queue entry)."""
    return (2 if post else 1) * bitmap_bytes(n) + 36 * count


def bytes_bu(n: int, unvisited: int, probes: int, found: int) -> int:
    """Bottom-up step: 4 bitmap passes (visited read + write, next write, stale
    clear) + 16 B row_ptr pair per candidate + 4 B per probed arc + 8 B
    level+parent per found vertex."""
    return 4 * bitmap_bytes(n) + 16 * unvisited + 4 * probes + 8 * found


def bytes_ss_count(n: int, found: int) -> int:
    """Single-scan count pass: next-frontier bitmap read + 8 B head[] per vertex."""
    return bitmap_bytes(n) + 8 * found


def kernel_model_level_bytes(n: int, strategy, fv, fe, unvisited, probes, directed: bool = False):
    """Algorithmic bytes of every level of one BFS given the strategies the
    selector took (the phases of the persistent kernel): SF and SS
    read a queue that exists after an SF level (No-Frontier-Generation) and is
    generated from the frontier bitmap otherwise; SS adds its count pass."""
    out = []
    L = len(strategy)
    for k in range(L):
        found = fv[k + 1] if k + 1 < L else 0
        s = strategy[k]
        queue_valid = k == 0 or strategy[k - 1] == 0
        b = 0
        if s != 2 and not queue_valid:
            b += bytes_generate(n, fv[k], post=False)
        if s == 0:
            b += bytes_td_sf(n, fv[k], fe[k], found)
        elif s == 1:
            b += bytes_td_ss(n, fv[k], fe[k], found) + bytes_ss_count(n, found)
        else:
            b += bytes_bu(n, unvisited[k], probes[k], found)
            if directed:     # in-arc rows do not give out-degrees: head[] of every found vertex (R-9)
                b += 8 * found
        out.append(b)
    return out


def kernel_model_bytes(n: int, strategy, fv, fe, unvisited, probes, directed: bool = False) -> int:
    """Init + every level: the algorithmic bytes of one persistent-kernel launch."""
    return bytes_init(n) + sum(kernel_model_level_bytes(n, strategy, fv, fe, unvisited, probes, directed))
