"""Multi-GPU path (include/xbfs_dist.h) on the GPU: `world` processes share
cuda:0 (CUDA IPC maps each rank's replicas and inbox into the peers exactly as
across NVLink peers); host plumbing over gloo.  Gathered levels must equal the
oracle bit-exactly and parents must pass Graph500 validation, for the adaptive
selector and for every strategy forced on every level."""
import os
import socket

import numpy as np
import pytest

import oracle
from paper_conf_sc_yangls0w24_b200 import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

MODES = [dict(), dict(force_strategy=0), dict(force_strategy=1), dict(force_strategy=2), dict(alpha=0.02),
         dict(bu_stay=0.0)]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, graph, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        from paper_conf_sc_yangls0w24_b200.dist import DistGraph
        src, dst, n = _graph(graph)
        dg = DistGraph(src, dst, n)
        roots = synth.roots(n, src, dst, 4, root_seed=11).tolist() + [0]
        out = []
        for root in roots:
            for mi, opts in enumerate(MODES):
                lv, pa, st = dg.run(int(root), **opts)
                lvs, pas = [None] * world, [None] * world
                dist.all_gather_object(lvs, lv.cpu().numpy())
                dist.all_gather_object(pas, pa.cpu().numpy())
                if rank == 0:
                    out.append((int(root), mi, np.concatenate(lvs), np.concatenate(pas), st.strategy,
                                st.frontier_vertices, st.input_edges_traversed))
        dg.close()
        q.put((rank, out))
    except Exception as e:
        import traceback
        q.put((rank, f"{type(e).__name__}: {e}\n{traceback.format_exc()}"))
    finally:
        dist.destroy_process_group()


def _graph(name):
    if name == "kron":
        return synth.kronecker(13, seed=6)
    if name == "grid":
        return synth.grid(40, 37, seed=2)
    # odd N and isolated vertices / small components
    rng = np.random.default_rng(3)
    n = 1001
    e = rng.integers(0, 700, (2500, 2)).astype(np.uint32)
    return e[:, 0].copy(), e[:, 1].copy(), n


@pytest.mark.parametrize("world,graph", [(2, "kron"), (3, "kron"), (2, "grid"), (3, "rand"), (1, "kron")])
def test_dist_matches_oracle(world, graph):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, graph, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=600) for _ in range(world))
    for p in procs:
        p.join(timeout=120)
    for r, v in res.items():
        assert not isinstance(v, str), f"rank {r}: {v}"
    src, dst, n = _graph(graph)
    g = oracle.build_csr(n, src, dst)
    for root, mi, lv, pa, strat, fv, m in res[0]:
        ref, _, nl = oracle.bfs(g, root)
        assert np.array_equal(lv, ref), (root, MODES[mi])
        assert oracle.validate(g, src, dst, root, lv, pa) == 0, (root, MODES[mi])
        fs, _ = oracle.level_stats(g, ref)
        assert fv == fs.tolist()
        assert m == oracle.input_edges(src, ref)
        if "force_strategy" in MODES[mi]:
            assert set(strat) == {MODES[mi]["force_strategy"]}
