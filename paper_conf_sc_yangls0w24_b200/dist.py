"""Multi-GPU XBFS driver (include/xbfs_dist.h): 1D vertex partition, one process
per GPU, torch.distributed for the plumbing (IPC-handle exchange, the 8-counter
all-reduce and the barrier between the two phases of a top-down level).

All per-level compute and the frontier exchange run in libxbfs.so: bottom-up
levels publish their owned next-frontier words straight into every peer's
replica, top-down levels OR remote discoveries into the owner's inbox in peer
memory (north_star "direction switch made on globally reduced
counts").  This module only sequences the calls.
"""
from __future__ import annotations

import ctypes
from dataclasses import dataclass, field

import numpy as np

from . import xbfs as _x

NCOUNTS = 8
IPC_BYTES = 64
BU = _x.BU

_L = _x.lib
_P, _i64, _i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32
_L.xbfs_dist_build.argtypes = [_P, _P, _i64, _i64, _i32, _i32, ctypes.POINTER(_x.BuildOpts), ctypes.POINTER(_P)]
_L.xbfs_dist_info.argtypes = [_P, _P, _P, _P, _P]
_L.xbfs_dist_export.argtypes = [_P, _P]
_L.xbfs_dist_attach.argtypes = [_P, _P]
_L.xbfs_dist_begin.argtypes = [_P, _i64, _P, _P, ctypes.POINTER(_x.RunOpts), _P]
_L.xbfs_dist_level.argtypes = [_P, _i32, _P]
_L.xbfs_dist_advance.argtypes = [_P, _P, _P, _P]
_L.xbfs_dist_levels.argtypes = [_P, _i32, _P, _P, _P, _P, _P]
_L.xbfs_dist_destroy.argtypes = [_P]
_L.xbfs_dist_destroy.restype = None
for _fn in ("xbfs_dist_build", "xbfs_dist_info", "xbfs_dist_export", "xbfs_dist_attach", "xbfs_dist_begin",
            "xbfs_dist_level", "xbfs_dist_advance", "xbfs_dist_levels"):
    getattr(_L, _fn).restype = ctypes.c_int

#: symbols include/xbfs_dist.h declares (checked by tests/test_abi.py)
DIST_EXPORTS = ("xbfs_dist_build", "xbfs_dist_info", "xbfs_dist_export", "xbfs_dist_attach", "xbfs_dist_begin",
                "xbfs_dist_level", "xbfs_dist_advance", "xbfs_dist_levels", "xbfs_dist_destroy")


def partition(n: int, nranks: int, rank: int):
    """Owned range of `rank` (mirrors xbfs_dist_build): blocks of B = 32*ceil(n/(32p))."""
    blk = 32 * ((n + 32 * nranks - 1) // (32 * nranks))
    lo = min(n, rank * blk)
    return lo, max(0, min(blk, n - lo))


@dataclass
class DistStats:
    num_levels: int
    input_edges_traversed: int
    strategy: list = field(default_factory=list)
    frontier_vertices: list = field(default_factory=list)
    frontier_edges: list = field(default_factory=list)
    elapsed_ms: float = 0.0


class _LibBackend:
    """The real per-rank backend: libxbfs.so's xbfs_dist_* entry points."""

    def __init__(self, h):
        self.h = h

    def begin(self, source, level, parent, opts):
        c = np.zeros(NCOUNTS, np.int64)
        _x._check(_L.xbfs_dist_begin(self.h, int(source), _x._ptr(level) if level.numel() else None,
                                     _x._ptr(parent) if parent.numel() else None, ctypes.byref(opts), c.ctypes.data))
        return c

    def level(self, phase):
        c = np.zeros(NCOUNTS, np.int64)
        _x._check(_L.xbfs_dist_level(self.h, phase, c.ctypes.data))
        return c

    def advance(self, g):
        g = np.ascontiguousarray(g, dtype=np.int64)
        s, d = ctypes.c_int32(), ctypes.c_int32()
        _x._check(_L.xbfs_dist_advance(self.h, g.ctypes.data, ctypes.byref(s), ctypes.byref(d)))
        return s.value, bool(d.value)

    def levels(self):
        cap = 1 << 14
        st = np.zeros(cap, np.int8)
        fv = np.zeros(cap, np.int64)
        fe = np.zeros(cap, np.int64)
        nl, m = ctypes.c_int32(), ctypes.c_int64()
        _x._check(_L.xbfs_dist_levels(self.h, cap, st.ctypes.data, fv.ctypes.data, fe.ctypes.data,
                                      ctypes.byref(nl), ctypes.byref(m)))
        k = min(nl.value, cap)
        return DistStats(nl.value, m.value, st[:k].tolist(), fv[:k].tolist(), fe[:k].tolist())


def drive(backend, allreduce, barrier, source, level, parent, opts):
    """The level loop shared by every rank (host-side logic, testable with any
    backend): begin -> all-reduce -> advance, then per level phase 0, and for a
    top-down level a barrier and phase 1, then all-reduce -> advance."""
    g = allreduce(backend.begin(source, level, parent, opts))
    strategy, done = backend.advance(g)
    while not done:
        c = backend.level(0)
        if strategy != BU:
            barrier()               # every remote discovery is in its owner's inbox
            c = backend.level(1)
        g = allreduce(c)            # also orders this level's peer stores before the next level
        strategy, done = backend.advance(g)
    return backend.levels()


class DistGraph:
    """One rank's partition of a graph.  Collective: every rank of `group`
    constructs it with the same full tuple list."""

    def __init__(self, src, dst, num_vertices: int, group=None, device: int | None = None, stream=None):
        import torch
        import torch.distributed as dist
        self.group = group
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        self.device = torch.cuda.current_device() if device is None else device
        if stream is None:
            stream = torch.cuda.current_stream(self.device).cuda_stream
        if isinstance(src, np.ndarray):
            id_bytes, on_dev = src.dtype.itemsize, 0
            src, dst = np.ascontiguousarray(src), np.ascontiguousarray(dst)
        else:
            id_bytes, on_dev = src.element_size(), int(src.is_cuda)
            src, dst = src.contiguous(), dst.contiguous()
        o = _x.BuildOpts(device=self.device, id_bytes=id_bytes, stream=stream, edges_on_device=on_dev,
                         keep_duplicates=0)
        m = int(src.shape[0])
        h = ctypes.c_void_p()
        _x._check(_L.xbfs_dist_build(_x._ptr(src) if m else None, _x._ptr(dst) if m else None, m, num_vertices,
                                     self.world, self.rank, ctypes.byref(o), ctypes.byref(h)))
        self._h = h.value
        first, count, arcs, n = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64()
        _x._check(_L.xbfs_dist_info(self._h, ctypes.byref(first), ctypes.byref(count), ctypes.byref(arcs),
                                    ctypes.byref(n)))
        self.first, self.count, self.local_arcs, self.n = first.value, count.value, arcs.value, n.value
        buf = (ctypes.c_ubyte * IPC_BYTES)()
        _x._check(_L.xbfs_dist_export(self._h, buf))
        handles = [None] * self.world
        dist.all_gather_object(handles, bytes(buf), group=group)
        allh = b"".join(handles)
        _x._check(_L.xbfs_dist_attach(self._h, allh))
        dist.barrier(group=group)
        self._backend = _LibBackend(self._h)
        self._nccl = dist.get_backend(group) == "nccl"

    def _allreduce(self, c):
        import torch
        import torch.distributed as dist
        t = torch.as_tensor(np.asarray(c, dtype=np.int64))
        if self._nccl:
            t = t.cuda(self.device)
        dist.all_reduce(t, group=self.group)
        return t.cpu().numpy()

    def _barrier(self):
        import torch.distributed as dist
        dist.barrier(group=self.group)

    def run(self, source: int, level=None, parent=None, **opts):
        """BFS from global `source`.  Returns (level_local, parent_local, DistStats)
        for this rank's owned range [first, first+count)."""
        import torch
        dev = f"cuda:{self.device}"
        if level is None:
            level = torch.empty(self.count, dtype=torch.int32, device=dev)
        if parent is None:
            parent = torch.empty(self.count, dtype=torch.int32, device=dev)
        st = drive(self._backend, self._allreduce, self._barrier, source, level, parent, _x.make_run_opts(**opts))
        return level, parent, st

    def close(self):
        if getattr(self, "_h", None):
            _L.xbfs_dist_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
