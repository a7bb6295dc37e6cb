"""Multi-GPU XBFS binding (include/xbfs_dist.h): 1D vertex partition, one
process per GPU.  Argument marshalling only: the communicator (a shared-memory
segment on the node, reading R-10), the distributed CSR build with its
peer-memory arc shuffle, and every level of xbfs_run_dist (kernels, peer-memory
frontier exchange, barriers, the per-level counter all-reduce) run inside
libxbfs.so.  torch.distributed is used once, to broadcast the 128-byte unique id
from rank 0 (as one would an ncclUniqueId).
"""
from __future__ import annotations

import ctypes

import numpy as np

from . import xbfs as _x

UNIQUE_ID_BYTES = 128
MAX_RANKS = 16

_L = _x.lib
_P, _i64, _i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32
_L.xbfs_get_unique_id.argtypes = [_P]
_L.xbfs_comm_init.argtypes = [_P, _i32, _i32, ctypes.POINTER(_P)]
_L.xbfs_comm_barrier.argtypes = [_P]
_L.xbfs_comm_allreduce_i64.argtypes = [_P, _P, _P, _i32]
_L.xbfs_comm_destroy.argtypes = [_P]
_L.xbfs_comm_destroy.restype = None
_L.xbfs_build_csr_dist.argtypes = [_P, _P, _P, _i64, _i64, ctypes.POINTER(_x.BuildOpts), ctypes.POINTER(_P)]
_L.xbfs_partition_range.argtypes = [_P, _P, _P]
_L.xbfs_run_dist.argtypes = [_P, _i64, _P, _P, ctypes.POINTER(_x.RunOpts), ctypes.POINTER(_x.RunStats)]
for _fn in ("xbfs_get_unique_id", "xbfs_comm_init", "xbfs_comm_barrier", "xbfs_comm_allreduce_i64",
            "xbfs_build_csr_dist", "xbfs_partition_range", "xbfs_run_dist"):
    getattr(_L, _fn).restype = ctypes.c_int

#: symbols include/xbfs_dist.h declares (checked by tests/test_abi.py)
DIST_EXPORTS = ("xbfs_get_unique_id", "xbfs_comm_init", "xbfs_comm_barrier", "xbfs_comm_allreduce_i64",
                "xbfs_build_csr_dist", "xbfs_partition_range", "xbfs_run_dist", "xbfs_comm_destroy")


def partition(n: int, nranks: int, rank: int):
    """Owned range of `rank` (the library's rule): blocks of B = 32*ceil(n/(32p))."""
    blk = 32 * ((n + 32 * nranks - 1) // (32 * nranks))
    lo = min(n, rank * blk)
    return lo, max(0, min(blk, n - lo))


def tuple_range(m: int, nranks: int, rank: int):
    """The share of the M input tuples rank `rank` generates / passes to the build."""
    return rank * m // nranks, (rank + 1) * m // nranks


def xbfs_get_unique_id() -> bytes:
    buf = (ctypes.c_ubyte * UNIQUE_ID_BYTES)()
    _x._check(_L.xbfs_get_unique_id(buf))
    return bytes(buf)


class Comm:
    """One rank of the node-local communicator.  `uid` must be the same bytes on
    every rank (rank 0's xbfs_get_unique_id)."""

    def __init__(self, uid: bytes, nranks: int, rank: int):
        buf = (ctypes.c_ubyte * UNIQUE_ID_BYTES).from_buffer_copy(uid)
        h = ctypes.c_void_p()
        _x._check(_L.xbfs_comm_init(buf, int(nranks), int(rank), ctypes.byref(h)))
        self._h, self.nranks, self.rank = h.value, int(nranks), int(rank)

    @classmethod
    def from_torch(cls, group=None):
        """Collective over a torch.distributed group: rank 0 makes the id, broadcast it."""
        import torch.distributed as dist
        rank, world = dist.get_rank(group), dist.get_world_size(group)
        obj = [xbfs_get_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(obj, src=0, group=group)
        return cls(obj[0], world, rank)

    def barrier(self):
        _x._check(_L.xbfs_comm_barrier(self._h))

    def allreduce(self, values):
        a = np.ascontiguousarray(np.asarray(values, dtype=np.int64))
        out = np.empty_like(a)
        _x._check(_L.xbfs_comm_allreduce_i64(self._h, a.ctypes.data, out.ctypes.data, int(a.size)))
        return out

    @property
    def handle(self):
        return self._h

    def close(self):
        if getattr(self, "_h", None):
            _L.xbfs_comm_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class DistGraph:
    """This rank's partition of a graph (collective over `comm`).  src/dst: THIS
    rank's share of the input tuples (numpy, or torch tensors on host or device)."""

    def __init__(self, comm: Comm, src, dst, num_vertices: int, device: int | None = None, stream=None):
        import torch
        self.comm = comm
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
        _x._check(_L.xbfs_build_csr_dist(comm.handle, _x._ptr(src) if m else None, _x._ptr(dst) if m else None, m,
                                         int(num_vertices), ctypes.byref(o), ctypes.byref(h)))
        self._h = h.value
        first, count = ctypes.c_int64(), ctypes.c_int64()
        _x._check(_L.xbfs_partition_range(self._h, ctypes.byref(first), ctypes.byref(count)))
        self.first, self.count = first.value, count.value
        self.n, self.arcs, self.m_input, self.max_degree = _x.xbfs_graph_info(self._h)

    def run(self, source: int, level=None, parent=None, stats: bool = True, **opts):
        """BFS from global `source` (xbfs_run_dist).  Returns (level_local,
        parent_local, Stats) for this rank's owned range [first, first+count);
        Stats.elapsed_ms is this rank's device time (take the max over ranks)."""
        import torch
        dev = f"cuda:{self.device}"
        if level is None:
            level = torch.empty(max(self.count, 1), dtype=torch.int32, device=dev)[: self.count]
        if parent is None:
            parent = torch.empty(max(self.count, 1), dtype=torch.int32, device=dev)[: self.count]
        sb = _x._StatsBuf() if stats else None
        _x._check(_L.xbfs_run_dist(self._h, int(source), _x._ptr(level) if self.count else None,
                                   _x._ptr(parent) if self.count else None, ctypes.byref(_x.make_run_opts(**opts)),
                                   ctypes.byref(sb.c) if sb else None))
        return level, parent, (sb.result() if sb else None)

    def close(self):
        if getattr(self, "_h", None):
            _x.xbfs_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
