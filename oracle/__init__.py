"""CPU oracle for the XBFS hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_sc_yangls0w24_b200``) never imports it and shares no code with
it.  Every function follows the plain definition it cites (see oracle.c's
header and DESIGN.md §3); pins live in ``tests/test_oracle.py``.

Parity status per function:
  build_csr, reorder, bfs, validate, input_edges, level_stats, select,
  select_sequence, byte_replay, build_csr_directed,
  validate_directed, validate_tuples (OpenMP, liboracle_omp.so) — all pinned
  (closed forms, scipy brute force, mutation tests, hand-computed replay,
  agreement of the two validators).  The paper's own worked example (Figs 1-4) is lost:
  "parity unpinned" for that example only.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_SRC_OMP = os.path.join(_HERE, "validate_omp.c")
_LIB_OMP = os.path.join(_HERE, "liboracle_omp.so")

V1_ROOT, V2_REACH, V3_LEVEL_STEP, V4_TREE_EDGE, V5_EDGE_SPAN, V_RANGE = 1, 2, 4, 8, 16, 32


def build(force: bool = False) -> str:
    """Compile oracle.c with plain gcc (no OpenMP, no CUDA)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-shared", "-fPIC", "-o", _LIB, _SRC])
    # the tuple-list validator for s27-size roots: OpenMP over the host cores
    if force or not os.path.exists(_LIB_OMP) or os.path.getmtime(_LIB_OMP) < os.path.getmtime(_SRC_OMP):
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-fopenmp", "-shared", "-fPIC", "-o", _LIB_OMP,
                               _SRC_OMP])
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        i64, i32, f64 = ctypes.c_int64, ctypes.c_int32, ctypes.c_double
        L.oracle_build_csr.argtypes = [i64, i64, P, P, P, P, P]
        L.oracle_build_csr.restype = ctypes.c_int
        L.oracle_reorder.argtypes = [i64, P, P]
        L.oracle_reorder.restype = ctypes.c_int
        L.oracle_reorder_by.argtypes = [i64, P, P, P]
        L.oracle_reorder_by.restype = ctypes.c_int
        L.oracle_first_parents.argtypes = [i64, P, P, P, i64, P]
        L.oracle_first_parents.restype = i64
        L.oracle_bfs.argtypes = [i64, P, P, i64, P, P]
        L.oracle_bfs.restype = i32
        L.oracle_validate.argtypes = [i64, P, P, i64, P, P, i64, P, P]
        L.oracle_validate.restype = ctypes.c_int
        L.oracle_input_edges.argtypes = [i64, P, P]
        L.oracle_input_edges.restype = i64
        L.oracle_level_stats.argtypes = [i64, P, P, i32, P, P]
        L.oracle_level_stats.restype = i32
        L.oracle_select.argtypes = [i64, i64, i64, i64, f64, f64, f64, f64, i32, i64]
        L.oracle_select.restype = i32
        L.oracle_select_sequence.argtypes = [i64, P, P, i32, f64, f64, f64, f64, P, P]
        L.oracle_select_sequence.restype = i32
        L.oracle_byte_replay.argtypes = [i64, P, P, P, i32, P, P]
        L.oracle_byte_replay.restype = i64
        L.oracle_bu_probes.argtypes = [i64, P, P, P, i32]
        L.oracle_bu_probes.restype = i64
        L.oracle_build_csr_directed.argtypes = [i64, i64, P, P, P, P, P]
        L.oracle_build_csr_directed.restype = ctypes.c_int
        L.oracle_validate_directed.argtypes = [i64, P, P, i64, P, P, i64, P, P]
        L.oracle_validate_directed.restype = ctypes.c_int
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _u32(a) -> np.ndarray:
    return np.ascontiguousarray(a, dtype=np.uint32)


class CSR:
    """Oracle CSR: row_ptr int64[n+1], col int32[A]; rows id-sorted (O-3)."""

    def __init__(self, n: int, row_ptr: np.ndarray, col: np.ndarray):
        self.n, self.row_ptr, self.col = n, row_ptr, col

    @property
    def arcs(self) -> int:
        return int(self.row_ptr[-1])

    def degree(self) -> np.ndarray:
        return np.diff(self.row_ptr)


def build_csr(n: int, src, dst) -> CSR:
    src, dst = _u32(src), _u32(dst)
    m = src.shape[0]
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    col = np.zeros(max(2 * m, 1), dtype=np.int32)
    arcs = ctypes.c_int64(0)
    rc = lib().oracle_build_csr(n, m, _p(src), _p(dst), _p(row_ptr), _p(col), ctypes.byref(arcs))
    if rc != 0:
        raise ValueError(f"oracle_build_csr failed rc={rc}")
    return CSR(n, row_ptr, col[: arcs.value].copy())


def build_csr_directed(n: int, src, dst) -> CSR:
    """f4 / reading R-9: out-arc CSR of the tuples taken as arcs src -> dst."""
    src, dst = _u32(src), _u32(dst)
    m = src.shape[0]
    row_ptr = np.zeros(n + 1, dtype=np.int64)
    col = np.zeros(max(m, 1), dtype=np.int32)
    arcs = ctypes.c_int64(0)
    rc = lib().oracle_build_csr_directed(n, m, _p(src), _p(dst), _p(row_ptr), _p(col), ctypes.byref(arcs))
    if rc != 0:
        raise ValueError(f"oracle_build_csr_directed failed rc={rc}")
    return CSR(n, row_ptr, col[: arcs.value].copy())


def validate_directed(g: CSR, src, dst, source: int, level, parent) -> int:
    """Graph500 checks restated for arcs (oracle.c); g = build_csr_directed's CSR."""
    src, dst = _u32(src), _u32(dst)
    level = np.ascontiguousarray(level, dtype=np.int32)
    parent = np.ascontiguousarray(parent, dtype=np.int32)
    return lib().oracle_validate_directed(g.n, _p(g.row_ptr), _p(g.col), src.shape[0], _p(src), _p(dst),
                                          int(source), _p(level), _p(parent))


def reorder(g: CSR, deg_from: CSR | None = None) -> CSR:
    """a2: per-row degree-descending, id-ascending ties (C-12).  deg_from:
    take the neighbour degrees from this CSR instead (directed in-arc rows by the
    in-neighbour's out-degree, R-9)."""
    col = g.col.copy()
    if deg_from is None:
        rc = lib().oracle_reorder(g.n, _p(g.row_ptr), _p(col))
    else:
        rc = lib().oracle_reorder_by(g.n, _p(g.row_ptr), _p(col), _p(deg_from.row_ptr))
    if rc != 0:
        raise ValueError("oracle_reorder failed")
    return CSR(g.n, g.row_ptr, col)


def transpose_directed(n: int, src, dst) -> CSR:
    """In-arc CSR of the directed tuple graph: row j lists every i with an arc i -> j."""
    return build_csr_directed(n, dst, src)


def first_parents(rows: CSR, level, source: int):
    """Reading R-12: parent[v] = first vertex of v's stored row at level[v] - 1
    (rows = the re-arranged CSR the GPU searches).  Returns (parent int32[n], orphans)."""
    level = np.ascontiguousarray(level, dtype=np.int32)
    parent = np.empty(rows.n, dtype=np.int32)
    orphans = lib().oracle_first_parents(rows.n, _p(rows.row_ptr), _p(rows.col), _p(level), int(source),
                                         _p(parent))
    return parent, int(orphans)


def bfs(g: CSR, source: int):
    """O-4 plain FIFO BFS.  Returns (level int32[n], parent int32[n], nlevels)."""
    level = np.empty(g.n, dtype=np.int32)
    parent = np.empty(g.n, dtype=np.int32)
    nl = lib().oracle_bfs(g.n, _p(g.row_ptr), _p(g.col), int(source), _p(level), _p(parent))
    if nl < 0:
        raise ValueError("oracle_bfs: bad source")
    return level, parent, nl


def validate(g: CSR, src, dst, source: int, level, parent) -> int:
    """O-5 Graph500 V1..V5; returns a bitmask of failed checks (0 = valid)."""
    src, dst = _u32(src), _u32(dst)
    level = np.ascontiguousarray(level, dtype=np.int32)
    parent = np.ascontiguousarray(parent, dtype=np.int32)
    return lib().oracle_validate(g.n, _p(g.row_ptr), _p(g.col), src.shape[0], _p(src), _p(dst),
                                 int(source), _p(level), _p(parent))


def input_edges(src, level) -> int:
    """O-6 Graph500 m: tuples (i, j) with level[i] >= 0."""
    src = _u32(src)
    level = np.ascontiguousarray(level, dtype=np.int32)
    return int(lib().oracle_input_edges(src.shape[0], _p(src), _p(level)))


def level_stats(g: CSR, level):
    """Per level k: |F_k| and edgesF_k (P:L87 ratio numerator)."""
    level = np.ascontiguousarray(level, dtype=np.int32)
    cap = int(level.max()) + 2 if level.size else 1
    fs = np.zeros(cap, dtype=np.int64)
    fe = np.zeros(cap, dtype=np.int64)
    nl = lib().oracle_level_stats(g.n, _p(g.row_ptr), _p(level), cap, _p(fs), _p(fe))
    return fs[:nl].copy(), fe[:nl].copy()


def select(f_size: int, f_prev: int, f_edges: int, arcs: int, alpha=0.1, grow=2.0, ratio_min=1e-3,
           bu_stay=0.0, prev=-1, unvisited=0) -> int:
    """P:L87 strategy rule (0 SF, 1 SS, 2 BU); growth rule is reading C-10, the
    optional stay-in-BU hysteresis (bu_stay > 0, after a BU step) reading C-11."""
    return int(lib().oracle_select(f_size, f_prev, f_edges, arcs, alpha, grow, ratio_min, bu_stay, prev,
                                   unvisited))


def select_sequence(g: CSR, level, alpha=0.1, grow=2.0, ratio_min=1e-3, bu_stay=0.0):
    """The selector replayed over one BFS (exact levels): returns (strategy int8[nl],
    U_k int64[nl]) where U_k = non-isolated vertices unreached before step k."""
    level = np.ascontiguousarray(level, dtype=np.int32)
    cap = int(level.max()) + 2 if level.size else 1
    st = np.zeros(cap, dtype=np.int8)
    un = np.zeros(cap, dtype=np.int64)
    nl = lib().oracle_select_sequence(g.n, _p(g.row_ptr), _p(level), cap, alpha, grow, ratio_min, bu_stay,
                                      _p(st), _p(un))
    if nl < 0:
        raise ValueError("oracle_select_sequence failed")
    return st[:nl].copy(), un[:nl].copy()


_lib_omp = None


def validate_tuples(n: int, src, dst, source: int, level, parent, directed: bool = False,
                    threads: int | None = None) -> int:
    """O-5 V1..V5 over the tuple list (no CSR), OpenMP-parallel: the s27 validator.
    Same bitmask as validate()."""
    global _lib_omp
    if _lib_omp is None:
        build()
        L = ctypes.CDLL(_LIB_OMP)
        P = ctypes.c_void_p
        L.oracle_validate_tuples.argtypes = [ctypes.c_int64, ctypes.c_int64, P, P, ctypes.c_int64, P, P,
                                             ctypes.c_int32, ctypes.c_int32]
        L.oracle_validate_tuples.restype = ctypes.c_int
        _lib_omp = L
    src, dst = _u32(src), _u32(dst)
    level = np.ascontiguousarray(level, dtype=np.int32)
    parent = np.ascontiguousarray(parent, dtype=np.int32)
    t = threads if threads else (os.cpu_count() or 1)
    return _lib_omp.oracle_validate_tuples(n, src.shape[0], _p(src), _p(dst), int(source), _p(level), _p(parent),
                                           int(bool(directed)), int(t))


def byte_replay(g: CSR, level, strategy):
    """O-8 algorithmic bytes of one BFS for a strategy sequence (reordered CSR),
    exactly SURVEY §8(d) D-3.  Returns (total incl. init, per-level int64[])."""
    level = np.ascontiguousarray(level, dtype=np.int32)
    strategy = np.ascontiguousarray(strategy, dtype=np.int8)
    per = np.zeros(max(len(strategy), 1), dtype=np.int64)
    tot = lib().oracle_byte_replay(g.n, _p(g.row_ptr), _p(g.col), _p(level), len(strategy),
                                   _p(strategy), _p(per))
    return int(tot), per[: len(strategy)].copy()


def bu_probes(g: CSR, level, k: int) -> int:
    """Arcs probed by a bottom-up step at level k with early termination."""
    level = np.ascontiguousarray(level, dtype=np.int32)
    return int(lib().oracle_bu_probes(g.n, _p(g.row_ptr), _p(g.col), _p(level), int(k)))
