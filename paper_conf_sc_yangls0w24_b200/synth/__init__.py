"""Seeded synthetic inputs (Graph500 Kronecker, 2D grid, roots) — inputs only.

Shared by bench.py and the tests; holds none of the BFS method's arithmetic.
Recipe: SURVEY.md §8(c) O-1 / O-2 / O-7, restated in DESIGN.md §3.4.  The
paper gives no generator parameters (Tab II); the Graph500
quadrant law A,B,C,D = .57,.19,.19,.05 at edgefactor 16 is reading C-16.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "synth.c")
_LIB = os.path.join(_HERE, "libsynth.so")


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O3", "-std=c11", "-Wall", "-fopenmp", "-shared", "-fPIC",
                               "-o", _LIB, _SRC])
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        i64, i32, u64, f64 = ctypes.c_int64, ctypes.c_int32, ctypes.c_uint64, ctypes.c_double
        L.synth_splitmix64.argtypes = [u64]
        L.synth_splitmix64.restype = u64
        L.synth_uniform.argtypes = [u64, u64, u64, i32]
        L.synth_uniform.restype = f64
        L.synth_perm.argtypes = [u64, i32, u64]
        L.synth_perm.restype = u64
        L.synth_kronecker.argtypes = [i32, u64, i64, i64, i32, P, P]
        L.synth_kronecker.restype = ctypes.c_int
        L.synth_grid_count.argtypes = [i32, i32]
        L.synth_grid_count.restype = i64
        L.synth_grid.argtypes = [i32, i32, u64, i32, f64, P, P, P]
        L.synth_grid.restype = ctypes.c_int
        L.synth_roots.argtypes = [i64, i64, P, P, u64, i64, P]
        L.synth_roots.restype = i64
        _lib = L
    return _lib


def _p(a):
    return a.ctypes.data_as(ctypes.c_void_p)


def _empty(n, dtype, pinned):
    if pinned:
        import torch
        return torch.empty(int(n), dtype={np.uint32: torch.int32}[dtype], pin_memory=True).numpy().view(np.uint32)
    return np.empty(int(n), dtype=dtype)


def kronecker(scale: int, edgefactor: int = 16, seed: int = 1, permute: bool = True,
              e_begin: int = 0, e_end: int | None = None, pinned: bool = False):
    """Graph500 Kronecker tuples [e_begin, e_end) of M = edgefactor * 2^scale.

    Returns (src uint32[m], dst uint32[m], n)."""
    n = 1 << scale
    m_total = edgefactor * n
    e_end = m_total if e_end is None else e_end
    m = e_end - e_begin
    src, dst = _empty(m, np.uint32, pinned), _empty(m, np.uint32, pinned)
    rc = lib().synth_kronecker(scale, seed, e_begin, e_end, int(permute), _p(src), _p(dst))
    if rc != 0:
        raise ValueError("synth_kronecker failed")
    return src, dst, n


def grid(width: int, height: int, seed: int = 1, perm_scale: int = 0, keep_prob: float = 1.0):
    """4-neighbour W x H lattice (O-2).  Returns (src, dst, n)."""
    cap = int(lib().synth_grid_count(width, height))
    src, dst = np.empty(cap, np.uint32), np.empty(cap, np.uint32)
    m = ctypes.c_int64(0)
    rc = lib().synth_grid(width, height, seed, perm_scale, keep_prob, _p(src), _p(dst), ctypes.byref(m))
    if rc != 0:
        raise ValueError("synth_grid failed")
    return src[: m.value].copy(), dst[: m.value].copy(), width * height


def roots(n: int, src, dst, count: int, root_seed: int = 2):
    """O-7 roots: seeded, distinct, each touching a non-self-loop tuple."""
    src = np.ascontiguousarray(src, dtype=np.uint32)
    dst = np.ascontiguousarray(dst, dtype=np.uint32)
    out = np.empty(count, dtype=np.int64)
    got = lib().synth_roots(n, src.shape[0], _p(src), _p(dst), root_seed, count, _p(out))
    if got < 0:
        raise MemoryError("synth_roots")
    return out[:got].copy()


def splitmix64(x: int) -> int:
    return int(lib().synth_splitmix64(x))


def uniform(seed: int, e: int, k: int, scale: int) -> float:
    return float(lib().synth_uniform(seed, e, k, scale))


def perm(seed: int, scale: int, v: int) -> int:
    return int(lib().synth_perm(seed, scale, v))
