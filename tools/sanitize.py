"""Small BFS workloads for compute-sanitizer (memcheck / racecheck / initcheck):
    compute-sanitizer --tool memcheck python tools/sanitize.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_sc_yangls0w24_b200 import synth  # noqa: E402
from paper_conf_sc_yangls0w24_b200.xbfs import Graph  # noqa: E402

torch.cuda.set_device(0)
for name, (src, dst, n) in {"kron11": synth.kronecker(11, seed=3), "grid": synth.grid(33, 17, seed=1),
                            "kron8": synth.kronecker(8, seed=5)}.items():
    g = Graph(torch.from_numpy(src.view(np.int32)).cuda(), torch.from_numpy(dst.view(np.int32)).cuda(), n)
    for root in synth.roots(n, src, dst, 2, root_seed=4):
        drivers = [int(x) for x in os.environ.get("SANITIZE_DRIVERS", "1,2").split(",")]
        for drv in drivers:
            for opts in (dict(), dict(force_strategy=0), dict(force_strategy=1), dict(force_strategy=2),
                         dict(small_edges=0), dict(plan=[2, 1, 0, 2, 1, 0])):
                if drv == 2 and "plan" in opts:
                    continue
                lv, pa, st = g.run(int(root), stats=True, driver=drv, **opts)
    g.close()
# SANITIZE_PERSIST=1: the persistent driver (3), undirected and directed (f4) graphs,
# including a sink-heavy top-down level
if os.environ.get("SANITIZE_PERSIST") == "1":
    hub, ns = 0, 5000
    sk = np.arange(1, ns + 1)
    ch = np.arange(ns + 1, ns + 40)
    s_src = np.concatenate([np.zeros(ns + ch.size, np.int64), ch[:-1]]).astype(np.uint32)
    s_dst = np.concatenate([sk, ch, ch[1:]]).astype(np.uint32)
    cases = [("kron11", synth.kronecker(11, seed=3), False), ("grid", synth.grid(33, 17, seed=1), False),
             ("kron11d", synth.kronecker(11, seed=3), True), ("sinks", (s_src, s_dst, ns + 40), True)]
    for name, (src, dst, n), directed in cases:
        g = Graph(src, dst, n, directed=directed)
        for root in list(synth.roots(n, src, dst, 2, root_seed=4)) + [0]:
            for opts in (dict(), dict(force_strategy=0), dict(force_strategy=1), dict(force_strategy=2)):
                g.run(int(root), stats=True, driver=3, **opts)
        g.close()
# SANITIZE_DIST=1: the multi-GPU path with one rank (build with its peer-memory shuffle, xbfs_run_dist)
if os.environ.get("SANITIZE_DIST") == "1":
    from paper_conf_sc_yangls0w24_b200.dist import Comm, DistGraph, xbfs_get_unique_id
    c = Comm(xbfs_get_unique_id(), 1, 0)
    for name, (src, dst, n) in {"kron11": synth.kronecker(11, seed=3), "grid": synth.grid(33, 17, seed=1)}.items():
        dg = DistGraph(c, src, dst, n)
        for root in synth.roots(n, src, dst, 2, root_seed=4):
            for opts in (dict(), dict(force_strategy=0), dict(force_strategy=1), dict(force_strategy=2)):
                dg.run(int(root), **opts)
        dg.close()
    c.close()
torch.cuda.synchronize()
print("sanitize workload done")
