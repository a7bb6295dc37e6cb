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
# Algorithmic bytes per kernel launch.  Inputs are the per-level
# counters the library logs; used for the bench's live roofline figure.
# --------------------------------------------------------------------------

def bytes_td_expand(f_size: int, f_edges: int, found: int) -> int:
    """Top-down expansion of F_k: 20 B per frontier queue entry (id + two
    int64 offsets) + 4 B per expanded arc (col) + per discovered vertex 4 B
    level + 4 B parent + 16 B row_ptr pair + 20 B next-queue entry (SF)."""
    return 20 * f_size + 4 * f_edges + 44 * found


def bytes_generate(n: int, f_size: int) -> int:
    """Bitmap scan (n/8 B) + per frontier vertex 16 B row_ptr pair + 20 B queue
    entry."""
    return n // 8 + 36 * f_size


def bytes_bu(n: int, unvisited: int, probes: int, found: int) -> int:
    """Bottom-up step: visited + non-isolated words read (n/4 B), next and
    visited words written (n/4 B), 16 B row_ptr pair per candidate, 4 B per
    probed arc, 8 B level+parent per found vertex."""
    return n // 4 + n // 4 + 16 * unvisited + 4 * probes + 8 * found


def bytes_init(n: int) -> int:
    """level + parent fill (8n) and four n-bit bitmaps cleared."""
    return 8 * n + 4 * ((n + 7) // 8)
