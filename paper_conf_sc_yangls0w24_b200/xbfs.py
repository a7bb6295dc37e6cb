"""Thin ctypes binding of libxbfs.so (include/xbfs.h).

Argument marshalling only: every step of the BFS runs in the library's CUDA
kernels.  PyTorch supplies device memory (tensors' ``data_ptr()``) and the
stream (``torch.cuda.current_stream().cuda_stream``).  There is no CPU
fallback: if the shared library is missing or was not built for sm_100a,
importing this module raises.

The module-level functions carry the C names (``xbfs_build_csr``, ``xbfs_reorder``,
``xbfs_run`` …); :class:`Graph` is a convenience wrapper over them.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# XBFS_LIB overrides the library path (A/B experiments between builds only).
LIB_PATH = os.environ.get("XBFS_LIB", os.path.join(_HERE, "libxbfs.so"))

XBFS_OK, XBFS_ERR_INVALID_ARG, XBFS_ERR_OUT_OF_MEMORY, XBFS_ERR_CUDA, XBFS_ERR_NCCL, XBFS_ERR_STATE, \
    XBFS_ERR_UNSUPPORTED = range(7)
SF, SS, BU = 0, 1, 2
STRATEGY_NAMES = {SF: "SF", SS: "SS", BU: "BU"}


class XbfsError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"xbfs status {status}: {msg}")
        self.status = status


class BuildOpts(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int32), ("id_bytes", ctypes.c_int32), ("stream", ctypes.c_void_p),
                ("edges_on_device", ctypes.c_int32), ("keep_duplicates", ctypes.c_int32),
                ("directed", ctypes.c_int32)]


class RunOpts(ctypes.Structure):
    _fields_ = [("alpha", ctypes.c_double), ("grow", ctypes.c_double), ("ratio_min", ctypes.c_double),
                ("bu_stay", ctypes.c_double), ("force_strategy", ctypes.c_int32), ("driver", ctypes.c_int32),
                ("small_edges", ctypes.c_int32), ("plan_len", ctypes.c_int32),
                ("plan", ctypes.POINTER(ctypes.c_int8)), ("lookahead", ctypes.c_int32)]


class RunStats(ctypes.Structure):
    _fields_ = [("elapsed_ms", ctypes.c_float), ("num_levels", ctypes.c_int32),
                ("vertices_reached", ctypes.c_int64), ("arcs_traversed", ctypes.c_int64),
                ("input_edges_traversed", ctypes.c_int64), ("kernel_launches", ctypes.c_uint32),
                ("level_capacity", ctypes.c_int32),
                ("strategy", ctypes.POINTER(ctypes.c_int8)), ("frontier_vertices", ctypes.POINTER(ctypes.c_int64)),
                ("frontier_edges", ctypes.POINTER(ctypes.c_int64)), ("unvisited", ctypes.POINTER(ctypes.c_int64)),
                ("bu_probes", ctypes.POINTER(ctypes.c_int64)),
                ("kernel_capacity", ctypes.c_int32), ("num_kernels", ctypes.c_int32),
                ("kernel_id", ctypes.POINTER(ctypes.c_int32)), ("kernel_level", ctypes.POINTER(ctypes.c_int32)),
                ("kernel_ms", ctypes.POINTER(ctypes.c_float)), ("level_ms", ctypes.POINTER(ctypes.c_float)),
                ("lookahead_found", ctypes.POINTER(ctypes.c_int64)),
                ("init_ms", ctypes.c_float)]


#: kernel ids of RunStats.kernel_id (XBFS_K_* in include/xbfs.h)
KERNEL_NAMES = {0: "init_fill", 1: "seed", 2: "generate_pre", 3: "td_expand_sf", 4: "td_expand_ss",
                5: "generate_post", 6: "bu_traverse", 7: "select", 8: "small_sf",
                9: "ss_count"}


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build it with __graft_entry__.build() "
                          "(python -m paper_conf_sc_yangls0w24_b200._build). There is no CPU fallback.")
    L = ctypes.CDLL(LIB_PATH)
    P, i64, i32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32
    L.xbfs_build_csr.argtypes = [P, P, i64, i64, ctypes.POINTER(BuildOpts), ctypes.POINTER(P)]
    L.xbfs_reorder.argtypes = [P, i32]
    L.xbfs_run.argtypes = [P, i64, P, P, ctypes.POINTER(RunOpts), ctypes.POINTER(RunStats)]
    L.xbfs_run_host.argtypes = [P, i64, P, P, ctypes.POINTER(RunOpts), ctypes.POINTER(RunStats)]
    L.xbfs_run_host_batch.argtypes = [P, P, i32, i32, P, P, ctypes.POINTER(RunOpts)]
    L.xbfs_graph_info.argtypes = [P, P, P, P, P]
    L.xbfs_copy_csr.argtypes = [P, P, P]
    L.xbfs_destroy.argtypes = [P]
    L.xbfs_destroy.restype = None
    L.xbfs_last_error.restype = ctypes.c_char_p
    L.xbfs_run_opts_default.argtypes = [ctypes.POINTER(RunOpts)]
    L.xbfs_run_opts_default.restype = None
    L.xbfs_compiled_arch.restype = i32
    for fn in ("xbfs_build_csr", "xbfs_reorder", "xbfs_run", "xbfs_run_host", "xbfs_run_host_batch",
               "xbfs_graph_info", "xbfs_copy_csr"):
        getattr(L, fn).restype = ctypes.c_int
    if L.xbfs_compiled_arch() != 100:
        raise ImportError("libxbfs.so was not built for sm_100a")
    return L


lib = _load()

#: every symbol include/xbfs.h declares (checked by tests/test_abi.py)
EXPORTS = ("xbfs_run_opts_default", "xbfs_build_csr", "xbfs_reorder", "xbfs_run", "xbfs_run_host",
           "xbfs_run_host_batch",
           "xbfs_graph_info", "xbfs_copy_csr", "xbfs_destroy", "xbfs_last_error", "xbfs_compiled_arch")


def _check(rc: int):
    if rc != XBFS_OK:
        raise XbfsError(rc, lib.xbfs_last_error().decode(errors="replace"))


def _ptr(x) -> int:
    """Raw address of a torch tensor or numpy array (contiguous)."""
    if hasattr(x, "data_ptr"):
        assert x.is_contiguous()
        return x.data_ptr()
    assert isinstance(x, np.ndarray) and x.flags["C_CONTIGUOUS"]
    return x.ctypes.data


def xbfs_run_opts_default() -> RunOpts:
    o = RunOpts()
    lib.xbfs_run_opts_default(ctypes.byref(o))
    return o


def xbfs_build_csr(src, dst, num_edges: int, num_vertices: int, opts: BuildOpts | None = None) -> int:
    h = ctypes.c_void_p()
    _check(lib.xbfs_build_csr(_ptr(src) if num_edges else None, _ptr(dst) if num_edges else None,
                              num_edges, num_vertices, ctypes.byref(opts) if opts else None, ctypes.byref(h)))
    return h.value


def xbfs_reorder(g: int, mode: int = 1) -> None:
    _check(lib.xbfs_reorder(g, mode))


def xbfs_run(g: int, source: int, level, parent, opts: RunOpts | None = None, stats: RunStats | None = None):
    _check(lib.xbfs_run(g, source, _ptr(level), _ptr(parent), ctypes.byref(opts) if opts else None,
                        ctypes.byref(stats) if stats else None))


def _check_host_out(level, parent, need: int):
    """The C side DMAs straight into these buffers and cannot bound-check them:
    int32, C-contiguous host arrays of at least `need` elements each."""
    for name, a in (("level", level), ("parent", parent)):
        if not isinstance(a, np.ndarray) or a.dtype != np.int32 or not a.flags["C_CONTIGUOUS"]:
            raise TypeError(f"{name}: need a C-contiguous int32 numpy array (host memory)")
        if a.size < need:
            raise ValueError(f"{name}: {a.size} elements < the {need} the call writes")


def xbfs_run_host(g: int, source: int, level, parent, opts: RunOpts | None = None, stats: RunStats | None = None):
    _check_host_out(level, parent, xbfs_graph_info(g)[0])
    _check(lib.xbfs_run_host(g, source, _ptr(level), _ptr(parent), ctypes.byref(opts) if opts else None,
                             ctypes.byref(stats) if stats else None))


def xbfs_run_host_batch(g: int, sources, level, parent, host_slots: int | None = None,
                        opts: RunOpts | None = None):
    """sources: int64 array of K roots; level/parent: host int32 arrays of host_slots * N
    (host_slots defaults to K); root i's result lands in slot i % host_slots."""
    src = np.ascontiguousarray(np.asarray(sources, dtype=np.int64))
    k = int(src.size)
    slots = k if host_slots is None else int(host_slots)
    if k:
        n = xbfs_graph_info(g)[0]
        _check_host_out(level, parent, max(slots, 1) * n)
    _check(lib.xbfs_run_host_batch(g, src.ctypes.data if k else None, k, max(slots, 1) if k == 0 else slots,
                                   _ptr(level), _ptr(parent), ctypes.byref(opts) if opts else None))


def xbfs_graph_info(g: int):
    n, a, m, d = ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int64(), ctypes.c_int32()
    _check(lib.xbfs_graph_info(g, ctypes.byref(n), ctypes.byref(a), ctypes.byref(m), ctypes.byref(d)))
    return n.value, a.value, m.value, d.value


def xbfs_copy_csr(g: int):
    n, a, _, _ = xbfs_graph_info(g)
    row_ptr = np.empty(n + 1, dtype=np.int64)
    col = np.empty(max(a, 1), dtype=np.int32)
    _check(lib.xbfs_copy_csr(g, row_ptr.ctypes.data, col.ctypes.data))
    return row_ptr, col[:a]


def xbfs_destroy(g: int) -> None:
    lib.xbfs_destroy(g)


def xbfs_last_error() -> str:
    return lib.xbfs_last_error().decode(errors="replace")


# ---------------------------------------------------------------------------
@dataclass
class Stats:
    elapsed_ms: float
    num_levels: int
    vertices_reached: int
    arcs_traversed: int
    input_edges_traversed: int
    kernel_launches: int
    strategy: list = field(default_factory=list)
    frontier_vertices: list = field(default_factory=list)
    frontier_edges: list = field(default_factory=list)
    unvisited: list = field(default_factory=list)
    bu_probes: list = field(default_factory=list)
    kernels: list = field(default_factory=list)   # (name, level, ms) when profiled
    level_ms: list = field(default_factory=list)  # device ms per level (persistent driver)
    lookahead_found: list = field(default_factory=list)  # level-(k+2) vertices set by BU step k
    init_ms: float = 0.0        # persistent driver: kernel entry .. end of init + seed (device time)


class _StatsBuf:
    def __init__(self, cap: int = 1 << 14, kernel_cap: int = 0):
        self.cap = cap
        self.strategy = np.zeros(cap, np.int8)
        self.fv = np.zeros(cap, np.int64)
        self.fe = np.zeros(cap, np.int64)
        self.un = np.zeros(cap, np.int64)
        self.pr = np.zeros(cap, np.int64)
        self.lms = np.zeros(cap, np.float32)
        self.laf = np.zeros(cap, np.int64)
        self.c = RunStats()
        self.c.level_capacity = cap
        P = lambda a, t: a.ctypes.data_as(ctypes.POINTER(t))
        self.c.strategy = P(self.strategy, ctypes.c_int8)
        self.c.frontier_vertices = P(self.fv, ctypes.c_int64)
        self.c.frontier_edges = P(self.fe, ctypes.c_int64)
        self.c.unvisited = P(self.un, ctypes.c_int64)
        self.c.bu_probes = P(self.pr, ctypes.c_int64)
        self.c.level_ms = P(self.lms, ctypes.c_float)
        self.c.lookahead_found = P(self.laf, ctypes.c_int64)
        self.kcap = kernel_cap
        if kernel_cap:
            self.kid = np.zeros(kernel_cap, np.int32)
            self.klv = np.zeros(kernel_cap, np.int32)
            self.kms = np.zeros(kernel_cap, np.float32)
            self.c.kernel_capacity = kernel_cap
            self.c.kernel_id = P(self.kid, ctypes.c_int32)
            self.c.kernel_level = P(self.klv, ctypes.c_int32)
            self.c.kernel_ms = P(self.kms, ctypes.c_float)

    def result(self) -> Stats:
        c = self.c
        nl = min(c.num_levels, self.cap)
        return Stats(c.elapsed_ms, c.num_levels, c.vertices_reached, c.arcs_traversed, c.input_edges_traversed,
                     c.kernel_launches, self.strategy[:nl].tolist(), self.fv[:nl].tolist(), self.fe[:nl].tolist(),
                     self.un[:nl].tolist(), self.pr[:nl].tolist(),
                     [(KERNEL_NAMES[int(self.kid[i])], int(self.klv[i]), float(self.kms[i]))
                      for i in range(min(c.num_kernels, self.kcap))] if self.kcap else [],
                     self.lms[:nl].tolist(), self.laf[:nl].tolist(), c.init_ms)


def make_run_opts(alpha=None, grow=None, ratio_min=None, bu_stay=None, force_strategy=None, driver=None,
                  small_edges=None, plan=None, lookahead=None) -> RunOpts:
    """plan: sequence of per-level strategies (-1 = selector, 0 SF, 1 SS, 2 BU)."""
    o = xbfs_run_opts_default()
    for k, v in dict(alpha=alpha, grow=grow, ratio_min=ratio_min, bu_stay=bu_stay,
                     force_strategy=force_strategy, driver=driver, small_edges=small_edges,
                     lookahead=lookahead).items():
        if v is not None:
            setattr(o, k, v)
    if plan is not None and len(plan):
        arr = (ctypes.c_int8 * len(plan))(*[int(x) for x in plan])
        o._plan_keepalive = arr
        o.plan = ctypes.cast(arr, ctypes.POINTER(ctypes.c_int8))
        o.plan_len = len(plan)
    return o


class Graph:
    """A device-resident CSR graph (owning handle).

    ``src``/``dst``: torch tensors (cuda or cpu) or numpy arrays of uint32/int32
    or int64 vertex ids."""

    def __init__(self, src, dst, num_vertices: int, device: int | None = None, stream=None, reorder: bool = True,
                 directed: bool = False):
        import torch
        if isinstance(src, np.ndarray):
            id_bytes = src.dtype.itemsize
            on_dev = 0
            src = np.ascontiguousarray(src)
            dst = np.ascontiguousarray(dst)
        else:
            id_bytes = src.element_size()
            on_dev = int(src.is_cuda)
            src = src.contiguous()
            dst = dst.contiguous()
        if device is None:
            device = torch.cuda.current_device()
        if stream is None:
            stream = torch.cuda.current_stream(device).cuda_stream
        self.device = device
        o = BuildOpts(device=device, id_bytes=id_bytes, stream=stream, edges_on_device=on_dev, keep_duplicates=0,
                      directed=int(bool(directed)))
        self.directed = bool(directed)
        m = int(src.shape[0])
        self._h = xbfs_build_csr(src, dst, m, num_vertices, o)
        self.n, self.arcs, self.m_input, self.max_degree = xbfs_graph_info(self._h)
        self.reordered = False
        if reorder:
            self.reorder(1)

    def reorder(self, mode: int = 1):
        xbfs_reorder(self._h, mode)
        self.reordered = mode == 1

    def run(self, source: int, level=None, parent=None, stats: bool = False, profile: int = 0, **opts):
        """BFS into device tensors (allocated if not given).  Returns
        (level, parent, Stats or None)."""
        import torch
        if level is None:
            level = torch.empty(self.n, dtype=torch.int32, device=f"cuda:{self.device}")
        if parent is None:
            parent = torch.empty(self.n, dtype=torch.int32, device=f"cuda:{self.device}")
        sb = _StatsBuf(kernel_cap=profile) if (stats or profile) else None
        xbfs_run(self._h, int(source), level, parent, make_run_opts(**opts), sb.c if sb else None)
        return level, parent, (sb.result() if sb else None)

    def run_host(self, source: int, level_host, parent_host, stats: bool = False, **opts):
        sb = _StatsBuf() if stats else None
        xbfs_run_host(self._h, int(source), level_host, parent_host, make_run_opts(**opts), sb.c if sb else None)
        return sb.result() if sb else None

    def run_host_batch(self, sources, level_host, parent_host, host_slots: int | None = None, **opts):
        """Pipelined multi-root BFS into host arrays (xbfs_run_host_batch): D2H of root i
        overlaps the BFS of root i+1."""
        xbfs_run_host_batch(self._h, sources, level_host, parent_host, host_slots, make_run_opts(**opts))

    def csr(self):
        return xbfs_copy_csr(self._h)

    @property
    def handle(self) -> int:
        return self._h

    def close(self):
        if getattr(self, "_h", None):
            xbfs_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
