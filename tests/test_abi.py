"""C-ABI checks that need no GPU: the library loads, exports every symbol
include/xbfs.h declares, was built for sm_100a, and rejects bad arguments
before touching CUDA."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def xb():
    from paper_conf_sc_yangls0w24_b200 import _build
    _build.build_library()
    from paper_conf_sc_yangls0w24_b200 import xbfs
    return xbfs


def _declared(header):
    txt = open(os.path.join(ROOT, "include", header)).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return set(re.findall(r"\b(xbfs_[a-z0-9_]+)\s*\(", txt))


def test_exports_every_declared_symbol(xb):
    from paper_conf_sc_yangls0w24_b200 import dist
    for header, listed in (("xbfs.h", xb.EXPORTS), ("xbfs_dist.h", dist.DIST_EXPORTS)):
        declared = _declared(header)
        assert declared, f"no declarations parsed from {header}"
        for name in declared:
            assert hasattr(xb.lib, name), f"missing export {name}"
        assert declared == set(listed), (header, declared ^ set(listed))


def test_compiled_for_sm100a(xb):
    assert xb.lib.xbfs_compiled_arch() == 100


def test_defaults(xb):
    o = xb.xbfs_run_opts_default()
    assert o.alpha == 0.04 and o.force_strategy == -1   # P:L347 uses 0.1; B200-tuned (reading C-13)


def test_invalid_arguments_do_not_touch_cuda(xb):
    h = ctypes.c_void_p()
    assert xb.lib.xbfs_build_csr(None, None, 0, 10, None, None) == xb.XBFS_ERR_INVALID_ARG
    assert xb.lib.xbfs_build_csr(None, None, 0, 0, None, ctypes.byref(h)) == xb.XBFS_ERR_INVALID_ARG
    assert "num_vertices" in xb.xbfs_last_error()
    assert xb.lib.xbfs_build_csr(None, None, 5, 10, None, ctypes.byref(h)) == xb.XBFS_ERR_INVALID_ARG
    assert xb.lib.xbfs_build_csr(None, None, 0, 1 << 31, None, ctypes.byref(h)) == xb.XBFS_ERR_INVALID_ARG
    assert xb.lib.xbfs_run(None, 0, None, None, None, None) == xb.XBFS_ERR_INVALID_ARG
    assert xb.lib.xbfs_reorder(None, 1) == xb.XBFS_ERR_INVALID_ARG
    assert xb.lib.xbfs_run_host_batch(None, None, 1, 1, None, None, None) == xb.XBFS_ERR_INVALID_ARG
    assert xb.lib.xbfs_graph_info(None, None, None, None, None) == xb.XBFS_ERR_INVALID_ARG
    xb.lib.xbfs_destroy(None)  # NULL-safe
    from paper_conf_sc_yangls0w24_b200 import dist
    uid = (ctypes.c_ubyte * dist.UNIQUE_ID_BYTES).from_buffer_copy(dist.xbfs_get_unique_id())
    assert xb.lib.xbfs_comm_init(uid, 2, 5, ctypes.byref(h)) == xb.XBFS_ERR_INVALID_ARG
    assert xb.lib.xbfs_comm_init(uid, 0, 0, ctypes.byref(h)) == xb.XBFS_ERR_INVALID_ARG
    assert xb.lib.xbfs_comm_init(uid, 17, 0, ctypes.byref(h)) == xb.XBFS_ERR_INVALID_ARG
    junk = (ctypes.c_ubyte * dist.UNIQUE_ID_BYTES)()
    assert xb.lib.xbfs_comm_init(junk, 1, 0, ctypes.byref(h)) == xb.XBFS_ERR_INVALID_ARG
    assert xb.lib.xbfs_build_csr_dist(None, None, None, 0, 10, None, ctypes.byref(h)) == xb.XBFS_ERR_INVALID_ARG
    assert xb.lib.xbfs_run_dist(None, 0, None, None, None, None) == xb.XBFS_ERR_INVALID_ARG
    assert xb.lib.xbfs_partition_range(None, None, None) == xb.XBFS_ERR_INVALID_ARG
    xb.lib.xbfs_comm_destroy(None)
    # a one-rank communicator needs no peers and no GPU
    c = dist.Comm(dist.xbfs_get_unique_id(), 1, 0)
    assert c.allreduce([1, 2, 3]).tolist() == [1, 2, 3]
    c.barrier()
    c.close()


def test_product_path_never_imports_oracle():
    """The CUDA path must not route through the oracle (no CPU fallback)."""
    pkg = os.path.join(ROOT, "paper_conf_sc_yangls0w24_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".c", ".h")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt, f
                assert "oracle.h" not in txt and "liboracle" not in txt, f
